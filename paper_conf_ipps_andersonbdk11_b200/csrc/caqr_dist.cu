// caqr_dist.cu -- row-sharded multi-GPU TSQR (one process per GPU) over NCCL.
//
// Not in the paper (single GPU); it is the distributed TSQR the paper
// cites mapped onto one NVSwitch node: every rank factors its
// contiguous row shard with the single-GPU TSQR, the n x n local R factors are
// all-gathered over NVLink (one ncclAllGather of n^2 elements per rank), and
// every rank runs the same deterministic structured tree over the P stacked
// R's -- one more tree level whose leaves are GPUs -- so all ranks hold
// bitwise-identical global R and top-level tree vectors (no broadcast).
#include <cuda_runtime.h>
#include <nccl.h>

#include <cstdint>
#include <cstring>
#include <new>

#include "../../include/caqr.h"

struct caqr_dist {
    ncclComm_t comm;
    int nranks;
    int rank;
};

namespace {

// gather (P*n x n, ld = P*n) <- P contiguous column-major n x n blocks.
template <typename T>
__global__ void stack_blocks_kernel(int P, int64_t n, const T* __restrict__ blocks,
                                    T* __restrict__ out, int64_t ld) {
    const int64_t total = (int64_t)P * n * n;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t blk = e / (n * n), rem = e % (n * n);
        const int64_t c = rem / n, r = rem % n;
        out[c * ld + blk * n + r] = blocks[e];
    }
}

template <typename T>
ncclDataType_t nccl_type();
template <>
ncclDataType_t nccl_type<float>() { return ncclFloat32; }
template <>
ncclDataType_t nccl_type<double>() { return ncclFloat64; }

template <typename T>
int dist_factor(caqr_dist* h, int64_t m_local, int64_t n, T* A, int64_t lda, T* R, int64_t ldr,
                void* ws, size_t ws_bytes, T* gather, void* cws, size_t cws_bytes,
                const caqr_opts* opts, cudaStream_t s, int dtype) {
    if (!h) return -1;
    if (n < 0 || n > 256) return -3;
    if (!gather || !cws) return -10;
    const int P = h->nranks;
    // 1. local TSQR of the shard (R lands in R, ldr)
    int rc = dtype == CAQR_F32
                 ? caqr_factor_f32(m_local, n, (float*)A, lda, (float*)R, ldr, ws, ws_bytes, opts, s)
                 : caqr_factor_f64(m_local, n, (double*)A, lda, (double*)R, ldr, ws, ws_bytes,
                                   opts, s);
    if (rc) return rc;
    if (n == 0) return 0;
    if (cws_bytes < caqr_combine_workspace_bytes(P, n, dtype)) return -12;
    // receive area for P contiguous n x n blocks sits after the combine's T blocks
    const size_t blk_elems = (size_t)P * n * n;
    T* recv = reinterpret_cast<T*>(static_cast<char*>(cws) + caqr_combine_workspace_bytes(P, n, dtype) -
                                   blk_elems * sizeof(T));
    // send buffer: my R as a contiguous n x n block (copy if ldr != n)
    T* send = recv + (size_t)h->rank * n * n;  // in-place all-gather
    if (cudaMemcpy2DAsync(send, n * sizeof(T), R, ldr * sizeof(T), n * sizeof(T), n,
                          cudaMemcpyDeviceToDevice, s) != cudaSuccess)
        return CAQR_ERR_CUDA;
    // 2. all-gather of the local R factors over NVLink
    if (ncclAllGather(send, recv, (size_t)n * n, nccl_type<T>(), h->comm, s) != ncclSuccess)
        return CAQR_ERR_NCCL;
    // 3. restack and combine (same bits on every rank)
    const int64_t ld = (int64_t)P * n;
    stack_blocks_kernel<T><<<64, 256, 0, s>>>(P, n, recv, gather, ld);
    if (cudaGetLastError() != cudaSuccess) return CAQR_ERR_CUDA;
    return dtype == CAQR_F32 ? caqr_combine_f32(P, n, (float*)gather, ld, (float*)R, ldr, cws,
                                                cws_bytes, s)
                             : caqr_combine_f64(P, n, (double*)gather, ld, (double*)R, ldr, cws,
                                                cws_bytes, s);
}

}  // namespace

extern "C" {

int caqr_dist_create(caqr_dist** handle, int nranks, int rank, const void* nccl_unique_id) {
    if (nranks < 1) return -1;
    if (rank < 0 || rank >= nranks) return -2;
    if (!handle || !nccl_unique_id) return -3;
    ncclUniqueId id;
    std::memcpy(&id, nccl_unique_id, sizeof(id));
    caqr_dist* h = new (std::nothrow) caqr_dist;
    if (!h) return CAQR_ERR_NCCL;
    h->nranks = nranks;
    h->rank = rank;
    if (ncclCommInitRank(&h->comm, nranks, id, rank) != ncclSuccess) {
        delete h;
        return CAQR_ERR_NCCL;
    }
    *handle = h;
    return 0;
}

void caqr_dist_destroy(caqr_dist* h) {
    if (!h) return;
    ncclCommDestroy(h->comm);
    delete h;
}

int caqr_dist_factor_f32(caqr_dist* h, int64_t m_local, int64_t n, float* A, int64_t lda, float* R,
                         int64_t ldr, void* ws, size_t ws_bytes, float* gather, void* cws,
                         size_t cws_bytes, const caqr_opts* opts, caqr_stream_t stream) {
    return dist_factor<float>(h, m_local, n, A, lda, R, ldr, ws, ws_bytes, gather, cws, cws_bytes,
                              opts, stream, CAQR_F32);
}
int caqr_dist_factor_f64(caqr_dist* h, int64_t m_local, int64_t n, double* A, int64_t lda,
                         double* R, int64_t ldr, void* ws, size_t ws_bytes, double* gather,
                         void* cws, size_t cws_bytes, const caqr_opts* opts,
                         caqr_stream_t stream) {
    return dist_factor<double>(h, m_local, n, A, lda, R, ldr, ws, ws_bytes, gather, cws, cws_bytes,
                               opts, stream, CAQR_F64);
}

/* ncclGetUniqueId wrapper so that the Python side needs no NCCL binding:
 * writes 128 bytes. */
int caqr_dist_unique_id(void* out128) {
    if (!out128) return -1;
    ncclUniqueId id;
    if (ncclGetUniqueId(&id) != ncclSuccess) return CAQR_ERR_NCCL;
    std::memcpy(out128, &id, sizeof(id));
    return 0;
}

}  // extern "C"
