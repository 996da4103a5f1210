// xlane_bench.cu -- cross-lane primitive throughput on one SM (design study):
// SHFL.BFLY (independent, 8 chains per warp) and LDS/STS round trips, for
// 1..32 warps per CTA (one CTA per SM).  Reports warp-instructions per cycle
// per SM.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/xlane_bench tools/xlane_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int MODE>
__global__ void k(float* out, int iters, long long* cyc) {
    __shared__ float sm[32 * 9 * 33];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    float v[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = lane * 0.5f + i;
    float* ws = sm + warp * 9 * 33;
    __syncthreads();
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
        if (MODE == 0) {  // 8 independent shuffles per iteration
#pragma unroll
            for (int i = 0; i < 8; ++i) v[i] += __shfl_xor_sync(0xffffffffu, v[i], 1 << (i & 3));
        } else if (MODE == 1) {  // 8 STS + 8 LDS (conflict-free) per iteration
#pragma unroll
            for (int i = 0; i < 8; ++i) ws[i * 33 + lane] = v[i];
            __syncwarp();
#pragma unroll
            for (int i = 0; i < 8; ++i) v[i] += ws[i * 33 + (lane ^ 1)];
            __syncwarp();
        } else if (MODE == 2) {  // 8 independent FFMA per iteration (reference)
#pragma unroll
            for (int i = 0; i < 8; ++i) v[i] = fmaf(v[i], 1.0001f, 0.5f);
        } else {  // 8 shfl.idx broadcasts
#pragma unroll
            for (int i = 0; i < 8; ++i) v[i] += __shfl_sync(0xffffffffu, v[i], i);
        }
    }
    long long t1 = clock64();
    float s = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) s += v[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
    float* out;
    long long* cyc;
    cudaMalloc(&out, 148 * 1024 * sizeof(float));
    cudaMalloc(&cyc, 148 * sizeof(long long));
    const char* names[4] = {"SHFL.BFLY", "STS+LDS", "FFMA", "SHFL.IDX"};
    const int iters = 2000;
    for (int mode = 0; mode < 4; ++mode) {
        for (int nw : {1, 2, 4, 8, 16, 32}) {
            auto f = mode == 0 ? k<0> : mode == 1 ? k<1> : mode == 2 ? k<2> : k<3>;
            f<<<1, nw * 32>>>(out, iters, cyc);
            cudaDeviceSynchronize();
            long long c;
            cudaMemcpy(&c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
            const double ops = (double)iters * 8 * nw * (mode == 1 ? 2 : 1);
            printf("%-10s warps %2d: %8lld cycles, %.3f warp-instr/cycle/SM (%.1f cycles per instr per warp)\n",
                   names[mode], nw, c, ops / c, (double)c / (iters * 8 * (mode == 1 ? 2 : 1)));
        }
    }
    return 0;
}
