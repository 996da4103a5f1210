// ffma2_bench.cu -- throughput of FFMA vs FFMA2 (sm_100 packed fp32 FMA) on
// B200: 8 independent chains per thread, all SMs busy.  Design study.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ffma2_bench tools/ffma2_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k1(float* out, int n) {
    float a[8];
    for (int i = 0; i < 8; ++i) a[i] = threadIdx.x * 0.001f + i;
    const float b = 0.9999f, c = 0.0001f;
    for (int it = 0; it < n; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) a[i] = fmaf(a[i], b, c);
    float s = 0;
    for (int i = 0; i < 8; ++i) s += a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k2(float* out, int n) {
    float2 a[4];
    for (int i = 0; i < 4; ++i) a[i] = make_float2(threadIdx.x * 0.001f + i, i + 0.5f);
    const float2 b = make_float2(0.9999f, 0.9999f), c = make_float2(0.0001f, 0.0001f);
    for (int it = 0; it < n; ++it)
#pragma unroll
        for (int i = 0; i < 4; ++i) a[i] = __ffma2_rn(a[i], b, c);
    float s = 0;
    for (int i = 0; i < 4; ++i) s += a[i].x + a[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k3(float* out, int n) {  // 8 FFMA2 chains: 16 FMAs per iteration
    float2 a[8];
    for (int i = 0; i < 8; ++i) a[i] = make_float2(threadIdx.x * 0.001f + i, i + 0.5f);
    const float2 b = make_float2(0.9999f, 0.9999f), c = make_float2(0.0001f, 0.0001f);
    for (int it = 0; it < n; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) a[i] = __ffma2_rn(a[i], b, c);
    float s = 0;
    for (int i = 0; i < 8; ++i) s += a[i].x + a[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main() {
    float* out;
    cudaMalloc(&out, 148 * 8 * 1024 * 4);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int n = 1 << 16;
    for (int rep = 0; rep < 2; ++rep) {
        float ms[3];
        for (int v = 0; v < 3; ++v) {
            cudaEventRecord(e0);
            if (v == 0) k1<<<148 * 8, 256>>>(out, n);
            if (v == 1) k2<<<148 * 8, 256>>>(out, n);
            if (v == 2) k3<<<148 * 8, 256>>>(out, n);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&ms[v], e0, e1);
        }
        const double th = 148.0 * 8 * 256;
        printf("FFMA: %.2f TFMA/s  FFMA2 (4 chains): %.2f TFMA/s  FFMA2 (8 chains): %.2f TFMA/s\n",
               th * n * 8 / ms[0] / 1e9, th * n * 8 / ms[1] / 1e9, th * n * 16 / ms[2] / 1e9);
    }
    return 0;
}
