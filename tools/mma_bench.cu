// Microbenchmark: per-SM issue rates of the candidate math paths on B200
// (FFMA, DFMA, mma.sync m16n8k8 TF32, mma.sync m8n8k4 F64).  Prints TFLOP/s.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/mma_bench tools/mma_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

#define ITERS 4096

__global__ void ffma_kernel(float* out, float a, float b) {
    float x[8];
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x + i;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) x[i] = fmaf(x[i], a, b);
    }
    float s = 0;
    for (int i = 0; i < 8; ++i) s += x[i];
    if (s == 12345.f) out[0] = s;
}
__global__ void dfma_kernel(double* out, double a, double b) {
    double x[8];
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x + i;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) x[i] = fma(x[i], a, b);
    }
    double s = 0;
    for (int i = 0; i < 8; ++i) s += x[i];
    if (s == 12345.) out[0] = s;
}
__global__ void mma_tf32_kernel(float* out) {
    unsigned a[4], b[2];
    float d[4][4];
    for (int i = 0; i < 4; ++i) a[i] = __float_as_uint(1.0f + threadIdx.x * 1e-3f + i);
    for (int i = 0; i < 2; ++i) b[i] = __float_as_uint(0.5f + i);
    for (int k = 0; k < 4; ++k)
        for (int i = 0; i < 4; ++i) d[k][i] = 0.f;
    for (int it = 0; it < ITERS / 4; ++it) {
#pragma unroll
        for (int k = 0; k < 4; ++k)
            asm volatile(
                "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
                "{%0,%1,%2,%3};"
                : "+f"(d[k][0]), "+f"(d[k][1]), "+f"(d[k][2]), "+f"(d[k][3])
                : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
    }
    float s = 0;
    for (int k = 0; k < 4; ++k)
        for (int i = 0; i < 4; ++i) s += d[k][i];
    if (s == 12345.f) out[0] = s;
}
__global__ void mma_f64_kernel(double* out) {
    double a = 1.0 + threadIdx.x * 1e-3, b = 0.5;
    double d[4][2];
    for (int k = 0; k < 4; ++k) d[k][0] = d[k][1] = 0;
    for (int it = 0; it < ITERS / 4; ++it) {
#pragma unroll
        for (int k = 0; k < 4; ++k)
            asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                         : "+d"(d[k][0]), "+d"(d[k][1])
                         : "d"(a), "d"(b));
    }
    double s = 0;
    for (int k = 0; k < 4; ++k) s += d[k][0] + d[k][1];
    if (s == 12345.) out[0] = s;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    float* fo;
    double* dout;
    cudaMalloc(&fo, 64);
    cudaMalloc(&dout, 64);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int blocks = sms * 8, threads = 256;
    auto time = [&](auto launch, double flops_per_thread, const char* name) {
        launch();
        cudaDeviceSynchronize();
        cudaEventRecord(e0);
        for (int r = 0; r < 5; ++r) launch();
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        double fl = 5.0 * flops_per_thread * blocks * threads;
        printf("%-22s %8.1f TFLOP/s\n", name, fl / (ms * 1e-3) / 1e12);
    };
    time([&] { ffma_kernel<<<blocks, threads>>>(fo, 1.0001f, 0.5f); }, 2.0 * 8 * ITERS, "FFMA");
    time([&] { dfma_kernel<<<blocks, threads>>>(dout, 1.0001, 0.5); }, 2.0 * 8 * ITERS, "DFMA");
    // per warp per mma: 16*8*8 MACs = 2048 flops -> per thread 64
    time([&] { mma_tf32_kernel<<<blocks, threads>>>(fo); }, 64.0 * 4 * (ITERS / 4), "mma.sync tf32 m16n8k8");
    // m8n8k4: 8*8*4 MACs = 512 flops per warp -> 16 per thread
    time([&] { mma_f64_kernel<<<blocks, threads>>>(dout); }, 16.0 * 4 * (ITERS / 4), "mma.sync f64 m8n8k4");
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
