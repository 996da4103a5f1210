// Microbenchmark of the register-resident panel factorization (factor_panel_regs)
// in isolation: cycles per 256x32 panel for 1 CTA and for a full grid.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o tools/panel_bench tools/panel_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

#include "../paper_conf_ipps_andersonbdk11_b200/csrc/tsqr_fused.cuh"

using namespace caqr;

namespace caqr {
template <typename T, int TPC>
__device__ __forceinline__ void factor_panel_timed(T* P, int RGP, int RG, int wp, T* tau_s, unsigned long long* tm) {
    using Lay = PanelLayout<TPC>;
    constexpr int SEG = Lay::SEG, TOPR = Lay::TOPR;
    constexpr int GPW = 32 / TPC;  // column groups per warp
    const int t = threadIdx.x;
    const int c = t / TPC, s = t % TPC;
    const int warp = t >> 5;
    const bool active = c < wp;
    T x[SEG];
    load_col<T, TPC>(P + (size_t)min(c, 31) * RGP, s, x);
#pragma unroll
    for (int i = 0; i < SEG; ++i)
        if (!(active && Lay::row(s, i) < RG)) x[i] = T(0);
    __syncthreads();  // everyone has its registers before P is overwritten with v's

    // Reflector of column j (< 32), run by the whole warp that holds column j
    // (xLARFG, reading S1): beta = -copysign(mu, alpha), tau = 1 + |alpha|/mu
    // == (beta-alpha)/beta, scale = copysign(1/(|alpha|+mu), alpha) == 1/(alpha-beta).
    // The owner group writes v (unit head, zeros above) into P[:, j].
    auto reflector = [&](int j) {
        T s0 = 0, s1 = 0, s2 = 0, s3 = 0, al = 0;
#pragma unroll
        for (int i = 0; i < TOPR; ++i) {
            const int r = s + TPC * i;
            s0 = (r > j) ? fma(x[i], x[i], s0) : s0;
            al = (r == j) ? x[i] : al;
        }
#pragma unroll
        for (int i = TOPR; i < SEG; i += 4) {
            s0 = fma(x[i], x[i], s0);
            if (i + 1 < SEG) s1 = fma(x[i + 1], x[i + 1], s1);
            if (i + 2 < SEG) s2 = fma(x[i + 2], x[i + 2], s2);
            if (i + 3 < SEG) s3 = fma(x[i + 3], x[i + 3], s3);
        }
        T sig = (s0 + s1) + (s2 + s3);
        const bool cr = (t % 32 == 0);
        unsigned long long r0_ = clock64();
#pragma unroll
        for (int o = 1; o < TPC; o <<= 1) {
            sig += __shfl_xor_sync(0xffffffffu, sig, o);
            al += __shfl_xor_sync(0xffffffffu, al, o);
        }
        unsigned long long r1_ = clock64();
        if (cr) tm[5] += r1_ - r0_;
        if (c != j) return;
        T tau = T(0), beta = al, scale = T(1);
        if (j < RG && sig != T(0)) {
            const T ss = fma(al, al, sig);
            const T aa = fabs(al);
            T rmu, mu;
            rsqrt_refined(ss, rmu, mu);  // 1/mu and mu = sqrt(alpha^2 + sigma)
            beta = -copysign(mu, al);
            tau = fma(aa, rmu, T(1));
            scale = copysign(rcp_refined(aa + mu), al);
        }
        unsigned long long r2_ = clock64();
        if (s == 0) tm[6] += r2_ - r1_;
#pragma unroll
        for (int i = 0; i < TOPR; ++i) {
            const int r = s + TPC * i;
            if (r > j) x[i] *= scale;
            if (r == j) x[i] = beta;
        }
#pragma unroll
        for (int i = TOPR; i < SEG; ++i) x[i] *= scale;
        T v[SEG];
#pragma unroll
        for (int i = 0; i < SEG; ++i) v[i] = x[i];
#pragma unroll
        for (int i = 0; i < TOPR; ++i) {
            const int r = s + TPC * i;
            v[i] = r > j ? x[i] : (r == j ? T(1) : T(0));
        }
        unsigned long long r3_ = clock64();
        if (s == 0) tm[7] += r3_ - r2_;
        store_col<T, TPC>(P + (size_t)j * RGP, s, v);
        if (s == 0) tau_s[j] = tau;
    };

    if (warp == 0) reflector(0);
    __syncthreads();
    for (int j = 0; j < wp; ++j) {
        const bool crit = (warp == (j + 1) / GPW) && (t % 32 == 0);
        unsigned long long ta = clock64();
        const T tau = tau_s[j];
        if (warp >= (j + 1) / GPW && tau != T(0)) {  // warps that own some column > j
            T v[SEG];
            load_col<T, TPC>(P + (size_t)j * RGP, s, v);
            T d0 = 0, d1 = 0, d2 = 0, d3 = 0;
#pragma unroll
            for (int i = 0; i < SEG; i += 4) {
                d0 = fma(v[i], x[i], d0);
                if (i + 1 < SEG) d1 = fma(v[i + 1], x[i + 1], d1);
                if (i + 2 < SEG) d2 = fma(v[i + 2], x[i + 2], d2);
                if (i + 3 < SEG) d3 = fma(v[i + 3], x[i + 3], d3);
            }
            const T d0s = (d0 + d1) + (d2 + d3);
            unsigned long long tb_ = clock64();
            if (crit) tm[1] += tb_ - ta;
            const T d = group_sum<TPC>(d0s, 0xffffffffu);
            unsigned long long tc_ = clock64();
            if (crit) tm[2] += tc_ - tb_;
            if (active && c > j) {
                const T st = tau * d;
#pragma unroll
                for (int i = 0; i < SEG; ++i) x[i] = fma(-st, v[i], x[i]);
            }
        }
        unsigned long long td_ = clock64();
        if (j + 1 < wp && warp == (j + 1) / GPW) reflector(j + 1);
        unsigned long long te_ = clock64();
        if (crit) tm[3] += te_ - td_;
        __syncthreads();
        unsigned long long tf_ = clock64();
        if (crit) { tm[4] += tf_ - te_; tm[0] += tf_ - ta; }
    }
    // stored form back into P (R on/above the diagonal, v below)
    if (active) store_col<T, TPC>(P + (size_t)c * RGP, s, x);
    __syncthreads();
}


}

template <int MODE>
__global__ void __launch_bounds__(256, 2) bench(float* data, int RG, int reps, unsigned long long* cyc) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int RGP = fused_col_stride<float>(kFusedMaxRows);
    float* P = reinterpret_cast<float*>(smem_raw);
    float* tau_s = P + 32 * RGP;
    unsigned long long total = 0;
    __shared__ unsigned long long tm[8];
    if (threadIdx.x < 8) tm[threadIdx.x] = 0;
    __syncthreads();
    for (int r = 0; r < reps; ++r) {
        for (int e = threadIdx.x; e < 32 * 256; e += 256) {
            const int c = e / 256, row = e % 256;
            P[c * RGP + padr<float>(row)] = row < RG ? data[(blockIdx.x % 4) * 8192 + e] : 0.f;
        }
        if (threadIdx.x < 32) tau_s[threadIdx.x] = 0.f;
        __syncthreads();
        const unsigned long long t0 = clock64();
        if (MODE == 1) factor_panel_timed<float, 8>(P, RGP, RG, 32, tau_s, tm);
        else if (MODE == 2) factor_panel_wb4<float>(P, RGP, RG, 32, tau_s, tau_s + 32);
        else factor_panel_regs<float, 8>(P, RGP, RG, 32, tau_s);
        const unsigned long long t1 = clock64();
        total += t1 - t0;
        __syncthreads();
    }
    if (threadIdx.x == 0) cyc[blockIdx.x] = total / reps;
    __syncthreads();
    if (MODE == 1 && blockIdx.x == 0 && threadIdx.x < 8) cyc[1024 + threadIdx.x] = tm[threadIdx.x] / reps;
}

int main() {
    float* d;
    unsigned long long* cyc;
    cudaMalloc(&d, 4 * 8192 * sizeof(float));
    cudaMalloc(&cyc, 4096 * sizeof(unsigned long long));
    float h[4 * 8192];
    unsigned s = 1;
    for (int i = 0; i < 4 * 8192; ++i) {
        s = s * 1664525u + 1013904223u;
        h[i] = ((s >> 8) & 0xffff) / 32768.f - 1.f;
    }
    cudaMemcpy(d, h, sizeof(h), cudaMemcpyHostToDevice);
    const size_t smem = sizeof(float) * (32 * fused_col_stride<float>(kFusedMaxRows) + 64 + 256);
    cudaFuncSetAttribute(bench<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    for (int grid : {1, 148, 296}) {
        for (int RG : {64, 256}) {
            bench<0><<<grid, 256, smem>>>(d, RG, 20, cyc);
            cudaDeviceSynchronize();
            unsigned long long hc[4096];
            cudaMemcpy(hc, cyc, grid * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
            double avg = 0;
            for (int i = 0; i < grid; ++i) avg += hc[i];
            avg /= grid;
            printf("grid %4d RG %3d: %8.0f cycles/panel = %6.0f cycles/column  (%s)\n", grid, RG, avg, avg / 32,
                   cudaGetErrorString(cudaGetLastError()));
        }
    }
    cudaFuncSetAttribute(bench<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    for (int grid : {1, 296}) {
        bench<2><<<grid, 256, smem>>>(d, 256, 20, cyc);
        cudaDeviceSynchronize();
        unsigned long long hc2[512];
        cudaMemcpy(hc2, cyc, grid * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < grid; ++i) avg += hc2[i];
        avg /= grid;
        printf("WB4 grid %4d: %8.0f cycles/panel = %6.0f cycles/column (%s)\n", grid, avg, avg / 32,
               cudaGetErrorString(cudaGetLastError()));
    }
    cudaFuncSetAttribute(bench<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    bench<1><<<1, 256, smem>>>(d, 256, 20, cyc);
    cudaDeviceSynchronize();
    unsigned long long hc[1032];
    cudaMemcpy(hc, cyc, sizeof(hc), cudaMemcpyDeviceToHost);
    printf("timed: total/panel %llu | per panel: step %llu, load+dot %llu, shfl %llu, reflector %llu, barrier %llu | refl: shfl %llu sqrt/rcp %llu scale %llu\n",
           hc[0], hc[1024], hc[1025], hc[1026], hc[1027], hc[1028], hc[1029], hc[1030], hc[1031]);
    return 0;
}
