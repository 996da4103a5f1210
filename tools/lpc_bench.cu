// Microbenchmark: lane-per-column panel factorization (panel_lpc.cuh) vs WB4
// (tsqr_fused.cuh) on 256 x 32 fp32 panels -- cycles per panel for 1 CTA and
// for 2 CTAs per SM, and the max difference of the stored forms / taus.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/lpc_bench tools/lpc_bench.cu
#include <cmath>
#include <cstdio>
#include <cuda_runtime.h>

#include "panel_lpc.cuh"
#include "panel_variants.cuh"

using namespace caqr;

template <int MODE>
__global__ void __launch_bounds__(256, 2) bench(const float* data, int RG, int reps, unsigned long long* cyc,
                                                float* out, float* tout) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int RGP = fused_col_stride<float>(kFusedMaxRows);
    float* P = reinterpret_cast<float*>(smem_raw);
    float* tau_s = P + 32 * RGP;
    float* Tb = tau_s + 32;
    float* scr = Tb + 128;
    unsigned long long total = 0;
    float x[32];
    for (int r = 0; r < reps; ++r) {
        for (int e = threadIdx.x; e < 32 * 256; e += 256) {
            const int c = e / 256, row = e % 256;
            P[c * RGP + row] = row < RG ? data[(blockIdx.x % 4) * 8192 + e] : 0.f;
        }
        if (threadIdx.x < 32) tau_s[threadIdx.x] = 0.f;
        __syncthreads();
        const unsigned long long t0 = clock64();
        if (MODE == 0)
            factor_panel_wb4<float>(Grp{(int)threadIdx.x, 0}, P, RGP, RG, 32, tau_s, Tb, scr);
        else
            factor_panel_lpc<float>(P, RGP, RG, 32, tau_s, scr, x);
        const unsigned long long t1 = clock64();
        total += t1 - t0;
        __syncthreads();
    }
    if (threadIdx.x == 0) cyc[blockIdx.x] = total / reps;
    if (blockIdx.x < 4) {
        float* o = out + blockIdx.x * 8192;
        if (MODE == 0) {
            for (int e = threadIdx.x; e < 8192; e += 256) o[e] = P[(e / 256) * RGP + e % 256];
        } else {
            const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
            for (int i = 0; i < 32; ++i) o[lane * 256 + 32 * warp + i] = x[i];
        }
        if (threadIdx.x < 32) tout[blockIdx.x * 32 + threadIdx.x] = tau_s[threadIdx.x];
    }
}

template <int MODE>
double run(const float* d, int grid, int RG, unsigned long long* cyc, float* out, float* tout, size_t smem) {
    cudaFuncSetAttribute(bench<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    bench<MODE><<<grid, 256, smem>>>(d, RG, 20, cyc, out, tout);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        printf("error %s\n", cudaGetErrorString(e));
        return -1;
    }
    static unsigned long long hc[4096];
    cudaMemcpy(hc, cyc, grid * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < grid; ++i) avg += hc[i];
    return avg / grid;
}

int main() {
    float *d, *o0, *o1, *t0, *t1;
    unsigned long long* cyc;
    cudaMalloc(&d, 4 * 8192 * sizeof(float));
    cudaMalloc(&o0, 4 * 8192 * sizeof(float));
    cudaMalloc(&o1, 4 * 8192 * sizeof(float));
    cudaMalloc(&t0, 128 * sizeof(float));
    cudaMalloc(&t1, 128 * sizeof(float));
    cudaMalloc(&cyc, 4096 * sizeof(unsigned long long));
    static float h[4 * 8192];
    unsigned s = 1;
    for (int i = 0; i < 4 * 8192; ++i) {
        s = s * 1664525u + 1013904223u;
        h[i] = ((s >> 8) & 0xffff) / 32768.f - 1.f;
    }
    cudaMemcpy(d, h, sizeof(h), cudaMemcpyHostToDevice);
    const size_t smem = sizeof(float) * (32 * fused_col_stride<float>(kFusedMaxRows) + 32 + 128 + 8 * (32 * 20 + 16));
    for (int RG : {256, 224, 64}) {
        for (int grid : {1, 296}) {
            const double a = run<0>(d, grid, RG, cyc, o0, t0, smem);
            const double b = run<1>(d, grid, RG, cyc, o1, t1, smem);
            printf("RG %3d grid %4d: WB4 %8.0f cycles/panel  LPC %8.0f cycles/panel (%.2fx)\n", RG, grid, a, b,
                   a / b);
        }
        static float h0[4 * 8192], h1[4 * 8192], ta[128], tb[128];
        cudaMemcpy(h0, o0, sizeof(h0), cudaMemcpyDeviceToHost);
        cudaMemcpy(h1, o1, sizeof(h1), cudaMemcpyDeviceToHost);
        cudaMemcpy(ta, t0, sizeof(ta), cudaMemcpyDeviceToHost);
        cudaMemcpy(tb, t1, sizeof(tb), cudaMemcpyDeviceToHost);
        double md = 0, mx = 0, mt = 0;
        for (int b = 0; b < 4; ++b)
            for (int c = 0; c < 32; ++c)
                for (int r = 0; r < RG; ++r) {
                    const int e = b * 8192 + c * 256 + r;
                    md = fmax(md, fabs(h0[e] - h1[e]));
                    mx = fmax(mx, fabs(h0[e]));
                }
        for (int i = 0; i < 128; ++i) mt = fmax(mt, fabs(ta[i] - tb[i]));
        printf("RG %3d: max |WB4 - LPC| stored form %.3e (max |entry| %.3e), tau %.3e\n", RG, md, mx, mt);
    }
    return 0;
}
