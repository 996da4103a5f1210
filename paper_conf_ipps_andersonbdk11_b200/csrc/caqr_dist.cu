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
#include <algorithm>
#include <chrono>
#include <cstring>
#include <thread>
#include <new>

#include "../../include/caqr.h"

struct caqr_dist {
    ncclComm_t comm;
    int nranks;
    int rank;
    int aborted;
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

// The post-exchange half of the distributed factor: restack P contiguous
// n x n blocks (rank order) into the (P n) x n stack `gather` and run the
// deterministic combine tree on it.  NCCL-free: caqr_dist_factor calls it
// after the all-gather, tests call it directly on one GPU.
template <typename T>
int combine_blocks(int P, int64_t n, const T* blocks, T* gather, int64_t ldg, T* R, int64_t ldr, void* cws,
                   size_t cws_bytes, cudaStream_t s, int dtype) {
    if (P < 1) return -1;
    if (n < 0 || n > 256) return -2;
    if (n == 0) return 0;
    if (!blocks) return -3;
    if (!gather) return -4;
    if (ldg < (int64_t)P * n) return -5;
    if (!R) return -6;
    if (ldr < n) return -7;
    if (!cws) return -8;
    if (cws_bytes < caqr_combine_workspace_bytes(P, n, dtype)) return -9;
    const int64_t total = (int64_t)P * n * n;
    const int blocks_ = (int)std::min<int64_t>(1024, (total + 255) / 256);
    stack_blocks_kernel<T><<<blocks_, 256, 0, s>>>(P, n, blocks, gather, ldg);
    if (cudaGetLastError() != cudaSuccess) return CAQR_ERR_CUDA;
    return dtype == CAQR_F32 ? caqr_combine_f32(P, n, (float*)gather, ldg, (float*)R, ldr, cws, cws_bytes, s)
                             : caqr_combine_f64(P, n, (double*)gather, ldg, (double*)R, ldr, cws, cws_bytes, s);
}

template <typename T>
int dist_factor(caqr_dist* h, int64_t m_local, int64_t n, T* A, int64_t lda, T* R, int64_t ldr,
                void* ws, size_t ws_bytes, T* gather, void* cws, size_t cws_bytes,
                const caqr_opts* opts, cudaStream_t s, int dtype) {
    if (!h) return -1;
    if (h->aborted) return CAQR_ERR_NCCL;
    if (n < 0 || n > 256) return -3;
    if (!gather || !cws) return -10;
    const int P = h->nranks;
    // every argument check before the local factor and the collective: a rank
    // that returned early would leave the others blocked in ncclAllGather
    if (n > 0 && cws_bytes < caqr_combine_workspace_bytes(P, n, dtype)) return -12;
    if (m_local < n) return -2;
    // 1. local TSQR of the shard (R lands in R, ldr)
    int rc = dtype == CAQR_F32
                 ? caqr_factor_f32(m_local, n, (float*)A, lda, (float*)R, ldr, ws, ws_bytes, opts, s)
                 : caqr_factor_f64(m_local, n, (double*)A, lda, (double*)R, ldr, ws, ws_bytes,
                                   opts, s);
    if (rc) return rc;
    if (n == 0) return 0;
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
    return combine_blocks<T>(P, n, recv, gather, (int64_t)P * n, R, ldr, cws, cws_bytes, s, dtype);
}

// ---------------------------------------------------------------------------
// Peer-memory exchange of the local R factors (the alternative to the NCCL
// all-gather; the exchange fused with the restack into the
// combine's input, no collective library on the path).  Rank r's CTA q:
//   1. stores r's n x n R (column-major, contiguous) into slot r of rank q's
//      mailbox buffer (e & 1) -- NVLink peer stores when q is another GPU;
//   2. publishes flags_q[r] = e (system-scope release after a system fence);
//   3. waits for its own flags_r[q] >= e (acquire) and moves the block rank q
//      stored into r's mailbox to rows [q n, (q+1) n) of r's stacked gather
//      (ld = P n), which caqr_combine then factors in place.
// Two mailbox buffers by epoch parity: a sender reuses buffer (e & 1) of a
// peer only after receiving that peer's epoch e-1 block, i.e. after the peer
// finished epoch e-2 (which emptied the same buffer).  Epochs start at 1 and
// increase by one per exchange; flags start at 0.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void st_release_sys(int* p, int v) {
    asm volatile("st.release.sys.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
template <typename T>
__device__ __forceinline__ T ldcg_sys(const T* p) {
    return __ldcg(p);
}
__device__ __forceinline__ int ld_acquire_sys(const int* p) {
    int v;
    asm volatile("ld.acquire.sys.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

template <typename T>
struct PeerArgs {
    int P;
    int64_t n;
    int64_t ldr;
    int epoch;
    const T* R_local;            // this rank's R (single-rank launch)
    T* gather_local;             // this rank's (P n) x n stack, ld = P n
    const T* const* R_arr;       // emulation: device array of the P ranks' R
    T* const* gather_arr;        // emulation: device array of the P ranks' stacks
    T* const* mailbox;           // device array: rank q's mailbox, 2 * P * n * n elements
    int* const* flags;           // device array: rank q's P flags
    int* status;                 // device int: CAQR_ERR_TIMEOUT if a wait timed out (may be null)
    long long timeout_ns;        // 0: wait forever
};

// grid (P, ranks): CTA (q, y) plays rank = rank0 + y, sending to and receiving from q
template <typename T>
__global__ void __launch_bounds__(256) peer_exchange_kernel(PeerArgs<T> a, int rank0) {
    const int q = blockIdx.x, rank = rank0 + blockIdx.y;
    const bool emu = a.R_arr != nullptr;
    const T* R = emu ? a.R_arr[rank] : a.R_local;
    T* g = emu ? a.gather_arr[rank] : a.gather_local;
    const int64_t n = a.n, nn = n * n;
    const int buf = a.epoch & 1;
    // 1. my R -> slot `rank` of q's mailbox buffer (epoch & 1), contiguous n x n
    T* dst = a.mailbox[q] + ((size_t)buf * a.P + rank) * nn;
    for (int64_t e = threadIdx.x; e < nn; e += blockDim.x) {
        const int64_t c = e / n, r = e - c * n;
        dst[e] = R[c * a.ldr + r];
    }
    __syncthreads();
    // 2. publish: a system fence (cumulative over the CTA's stores, ordered by
    //    the barrier) and a system-scope release of the flag
    if (threadIdx.x == 0) {
        __threadfence_system();
        st_release_sys(a.flags[q] + rank, a.epoch);
        // 3. wait for rank q's block in my mailbox (bounded: a rank that never
        //    calls must not hang this GPU forever)
        const int* f = a.flags[rank] + q;
        unsigned long long t0;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        while (ld_acquire_sys(f) < a.epoch) {
            __nanosleep(100);
            if (a.timeout_ns > 0) {
                unsigned long long t;
                asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
                if ((long long)(t - t0) > a.timeout_ns) {
                    if (a.status) atomicExch(a.status, CAQR_ERR_TIMEOUT);
                    break;
                }
            }
        }
    }
    __syncthreads();
    const T* src = a.mailbox[rank] + ((size_t)buf * a.P + q) * nn;
    const int64_t ldg = (int64_t)a.P * n;
    for (int64_t e = threadIdx.x; e < nn; e += blockDim.x) {
        const int64_t c = e / n, r = e - c * n;
        g[c * ldg + (int64_t)q * n + r] = ldcg_sys(src + e);
    }
}

template <typename T>
int peer_exchange(PeerArgs<T> a, int rank, bool emulate, cudaStream_t s) {
    if (a.P < 1) return -1;
    if (!emulate && (rank < 0 || rank >= a.P)) return -2;
    if (a.n < 0 || a.n > 256) return -3;
    if (emulate ? !a.R_arr : !a.R_local) return -4;
    if (a.ldr < std::max<int64_t>(a.n, 1)) return -5;
    if (!a.mailbox) return -6;
    if (!a.flags) return -7;
    if (emulate ? !a.gather_arr : !a.gather_local) return -8;
    if (a.epoch < 1) return -9;
    if (a.n == 0) return 0;
    if (!emulate) {
        peer_exchange_kernel<T><<<dim3(a.P, 1), 256, 0, s>>>(a, rank);
        return cudaGetLastError() == cudaSuccess ? 0 : CAQR_ERR_CUDA;
    }
    // one device, P virtual ranks whose CTAs wait on one another: a cooperative
    // launch guarantees that all P x P CTAs are co-resident
    int rank0 = 0;
    void* args[] = {&a, &rank0};
    const cudaError_t e =
        cudaLaunchCooperativeKernel((const void*)peer_exchange_kernel<T>, dim3(a.P, a.P), dim3(256), args, 0, s);
    return e == cudaSuccess ? 0 : CAQR_ERR_CUDA;
}

}  // namespace

extern "C" {

size_t caqr_peer_mailbox_bytes(int P, int64_t n, int dtype) {
    if (P < 1 || n < 0 || (dtype != CAQR_F32 && dtype != CAQR_F64)) return 0;
    return (size_t)2 * P * n * n * (dtype == CAQR_F32 ? 4 : 8);
}

int caqr_peer_exchange_f32(int P, int rank, int64_t n, const float* R, int64_t ldr, float* const* peer_mailbox,
                           int* const* peer_flags, float* gather, int epoch, int* status, int timeout_ms,
                           caqr_stream_t stream) {
    PeerArgs<float> a{P, n, ldr, epoch, R, gather, nullptr, nullptr, peer_mailbox, peer_flags, status,
                      timeout_ms > 0 ? (long long)timeout_ms * 1000000LL : 0LL};
    return peer_exchange<float>(a, rank, false, reinterpret_cast<cudaStream_t>(stream));
}
int caqr_peer_exchange_f64(int P, int rank, int64_t n, const double* R, int64_t ldr, double* const* peer_mailbox,
                           int* const* peer_flags, double* gather, int epoch, int* status, int timeout_ms,
                           caqr_stream_t stream) {
    PeerArgs<double> a{P, n, ldr, epoch, R, gather, nullptr, nullptr, peer_mailbox, peer_flags, status,
                       timeout_ms > 0 ? (long long)timeout_ms * 1000000LL : 0LL};
    return peer_exchange<double>(a, rank, false, reinterpret_cast<cudaStream_t>(stream));
}
int caqr_peer_exchange_emulate_f32(int P, int64_t n, const float* const* Rs, int64_t ldr, float* const* mailboxes,
                                   int* const* flags, float* const* gathers, int epoch, caqr_stream_t stream) {
    PeerArgs<float> a{P, n, ldr, epoch, nullptr, nullptr, Rs, gathers, mailboxes, flags, nullptr, 0LL};
    return peer_exchange<float>(a, 0, true, reinterpret_cast<cudaStream_t>(stream));
}
int caqr_peer_exchange_emulate_f64(int P, int64_t n, const double* const* Rs, int64_t ldr, double* const* mailboxes,
                                   int* const* flags, double* const* gathers, int epoch, caqr_stream_t stream) {
    PeerArgs<double> a{P, n, ldr, epoch, nullptr, nullptr, Rs, gathers, mailboxes, flags, nullptr, 0LL};
    return peer_exchange<double>(a, 0, true, reinterpret_cast<cudaStream_t>(stream));
}

/* CUDA IPC of a device allocation (the peer pointers of caqr_peer_exchange
 * across processes): handle = 64 opaque bytes. */
int caqr_ipc_handle(const void* dptr, void* out64) {
    if (!dptr) return -1;
    if (!out64) return -2;
    cudaIpcMemHandle_t h;
    if (cudaIpcGetMemHandle(&h, const_cast<void*>(dptr)) != cudaSuccess) return CAQR_ERR_CUDA;
    std::memcpy(out64, &h, sizeof(h));
    return 0;
}
int caqr_ipc_open(const void* handle64, void** dptr) {
    if (!handle64) return -1;
    if (!dptr) return -2;
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle64, sizeof(h));
    return cudaIpcOpenMemHandle(dptr, h, cudaIpcMemLazyEnablePeerAccess) == cudaSuccess ? 0 : CAQR_ERR_CUDA;
}
int caqr_ipc_close(void* dptr) {
    if (!dptr) return -1;
    return cudaIpcCloseMemHandle(dptr) == cudaSuccess ? 0 : CAQR_ERR_CUDA;
}

}  // extern "C"

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
    h->aborted = 0;
    if (ncclCommInitRank(&h->comm, nranks, id, rank) != ncclSuccess) {
        delete h;
        return CAQR_ERR_NCCL;
    }
    *handle = h;
    return 0;
}

void caqr_dist_destroy(caqr_dist* h) {
    if (!h) return;
    if (h->aborted)
        ncclCommAbort(h->comm);
    else
        ncclCommDestroy(h->comm);
    delete h;
}

int caqr_dist_wait(caqr_dist* h, caqr_stream_t stream, int timeout_ms) {
    if (!h) return -1;
    if (h->aborted) return CAQR_ERR_NCCL;
    const auto t0 = std::chrono::steady_clock::now();
    for (;;) {
        const cudaError_t q = cudaStreamQuery(reinterpret_cast<cudaStream_t>(stream));
        if (q == cudaSuccess) return 0;
        if (q != cudaErrorNotReady) return CAQR_ERR_CUDA;
        ncclResult_t async = ncclSuccess;
        if (ncclCommGetAsyncError(h->comm, &async) != ncclSuccess || async != ncclSuccess) {
            ncclCommAbort(h->comm);
            h->aborted = 1;
            return CAQR_ERR_NCCL;
        }
        const auto ms = std::chrono::duration_cast<std::chrono::milliseconds>(std::chrono::steady_clock::now() - t0);
        if (timeout_ms >= 0 && ms.count() > timeout_ms) {
            ncclCommAbort(h->comm);  // unblocks the collective on this rank
            h->aborted = 1;
            return CAQR_ERR_TIMEOUT;
        }
        std::this_thread::sleep_for(std::chrono::microseconds(50));
    }
}

int caqr_dist_combine_blocks_f32(int P, int64_t n, const float* blocks, float* gather, int64_t ldg, float* R,
                                 int64_t ldr, void* cws, size_t cws_bytes, caqr_stream_t stream) {
    return combine_blocks<float>(P, n, blocks, gather, ldg, R, ldr, cws, cws_bytes,
                                 reinterpret_cast<cudaStream_t>(stream), CAQR_F32);
}
int caqr_dist_combine_blocks_f64(int P, int64_t n, const double* blocks, double* gather, int64_t ldg, double* R,
                                 int64_t ldr, void* cws, size_t cws_bytes, caqr_stream_t stream) {
    return combine_blocks<double>(P, n, blocks, gather, ldg, R, ldr, cws, cws_bytes,
                                  reinterpret_cast<cudaStream_t>(stream), CAQR_F64);
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
