// Latency probes on B200 (one warp unless noted): dependent SHFL.BFLY chain,
// 16 interleaved 5-level butterfly reductions, dependent FFMA chain, LDS
// round trip, bar.sync with 8 warps.  Cycles from clock64.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/shfl_bench tools/shfl_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void probe(float* out, unsigned long long* cyc, int n) {
    __shared__ float sm[1024];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    float v = lane * 1.0f + 1.0f;
    sm[threadIdx.x] = v;
    __syncthreads();
    // 1. dependent shuffle chain (one warp)
    if (warp == 0) {
        unsigned long long t0 = clock64();
        for (int i = 0; i < n; ++i) v += __shfl_xor_sync(0xffffffffu, v, 1 + (i & 15));
        unsigned long long t1 = clock64();
        if (lane == 0) cyc[0] = (t1 - t0) / n;
        // 2. 16 interleaved 5-level reductions
        float w[16];
        for (int k = 0; k < 16; ++k) w[k] = v + k;
        t0 = clock64();
        for (int rep = 0; rep < n / 16; ++rep) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1)
#pragma unroll
                for (int k = 0; k < 16; ++k) w[k] += __shfl_xor_sync(0xffffffffu, w[k], o);
        }
        t1 = clock64();
        if (lane == 0) cyc[1] = (t1 - t0) / (n / 16);
        float s = 0;
        for (int k = 0; k < 16; ++k) s += w[k];
        v += s;
        // 3. dependent FFMA chain
        t0 = clock64();
        for (int i = 0; i < n; ++i) v = fmaf(v, 0.999f, 0.5f);
        t1 = clock64();
        if (lane == 0) cyc[2] = (t1 - t0) / n;
        // 4. dependent LDS chain
        int idx = lane;
        t0 = clock64();
        for (int i = 0; i < n; ++i) idx = ((int)sm[idx] + i) & 255;
        t1 = clock64();
        if (lane == 0) cyc[3] = (t1 - t0) / n;
        v += idx;
    }
    __syncthreads();
    // 5. barrier round trip with 8 warps
    unsigned long long t0 = clock64();
    for (int i = 0; i < n; ++i) __syncthreads();
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) cyc[4] = (t1 - t0) / n;
    // 6. one warp, single 5-level reduction chained n times (latency of a full warp_sum)
    if (warp == 0) {
        t0 = clock64();
        for (int i = 0; i < n; ++i) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        }
        t1 = clock64();
        if (lane == 0) cyc[5] = (t1 - t0) / n;
    }
    if (v == 12345.f) out[0] = v;
}

int main() {
    float* o;
    unsigned long long* c;
    cudaMalloc(&o, 64);
    cudaMalloc(&c, 64 * 8);
    probe<<<1, 256>>>(o, c, 4096);
    cudaDeviceSynchronize();
    unsigned long long h[8];
    cudaMemcpy(h, c, sizeof(h), cudaMemcpyDeviceToHost);
    printf("dependent SHFL+FADD: %llu cyc | 16x5-level interleaved reductions: %llu cyc | dependent FFMA: %llu | "
           "dependent LDS: %llu | bar.sync (8 warps): %llu | 5-level warp_sum: %llu  (%s)\n",
           h[0], h[1], h[2], h[3], h[4], h[5], cudaGetErrorString(cudaGetLastError()));
    return 0;
}
