// Microbenchmark of the register-resident panel factorization (factor_panel_regs)
// in isolation: cycles per 256x32 panel for 1 CTA and for a full grid.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o tools/panel_bench tools/panel_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

#include "panel_variants.cuh"

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



template <typename T>
__device__ __forceinline__ void factor_panel_wb4_timed(T* P, int RGP, int RG, int wp, T* tau_s, T* Tb, unsigned long long* tm) {
    T* scr_all = P + 32 * RGP + 1024;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // block blk = 7 - warp: the warp that owns the next block always has the
    // highest warp id among the warps still applying the current one, so the
    // scheduler (highest-id-first) favours the critical path
    const int blk = kWarps - 1 - warp;
    const int cb = 4 * blk;
    const int nc = max(0, min(4, wp - cb));
    T* scr = scr_all + warp * (32 * 20 + 16);
    T x[4][8];
#pragma unroll
    for (int q = 0; q < 4; ++q)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int r = lane + 32 * i;
            x[q][i] = (q < nc && r < RG) ? P[(size_t)(cb + q) * RGP + padr<T>(r)] : T(0);
        }
    __syncthreads();  // all columns are in registers before P gets v's
    const int nblk = (wp + 3) / 4;
    for (int b = 0; b < nblk; ++b) {
        unsigned long long t0 = clock64();
        if (blk == b) {
            T tq[4] = {T(0), T(0), T(0), T(0)};
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                if (q < nc) {
                    const int j = cb + q;
                    unsigned long long q0 = clock64();
                    T sg = T(0);
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const int r = lane + 32 * i;
                        sg = (r > j) ? fma(x[q][i], x[q][i], sg) : sg;
                    }
                    const T al = __shfl_sync(0xffffffffu, x[q][0], j);
                    sg = warp_sum(sg);
                    T tau = T(0), beta = al, scale = T(1);
                    if (j < RG && sg != T(0)) {
                        const T ss = fma(al, al, sg);
                        const T aa = fabs(al);
                        T rmu, mu;
                        rsqrt_refined(ss, rmu, mu);
                        beta = -copysign(mu, al);
                        tau = fma(aa, rmu, T(1));
                        scale = copysign(rcp_refined(aa + mu), al);
                    }
                    tq[q] = tau;
                    unsigned long long q1 = clock64();
                    if (lane == 0) tm[3] += q1 - q0;  // sigma/alpha reduce + rsqrt/rcp
                    T v[8];
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const int r = lane + 32 * i;
                        if (r > j) x[q][i] *= scale;
                        if (r == j) x[q][i] = beta;
                        v[i] = r > j ? x[q][i] : (r == j ? T(1) : T(0));
                        P[(size_t)j * RGP + padr<T>(r)] = v[i];
                    }
                    if (lane == 0) tau_s[j] = tau;
                    unsigned long long q2_ = clock64();
                    if (lane == 0) tm[4] += q2_ - q1;  // scale, v, stores
                    // apply H_j to this warp's later columns (interleaved reductions)
                    if (tau != T(0)) {
                        T d[4] = {T(0), T(0), T(0), T(0)};
#pragma unroll
                        for (int q2 = q + 1; q2 < 4; ++q2)
#pragma unroll
                            for (int i = 0; i < 8; ++i) d[q2] = fma(v[i], x[q2][i], d[q2]);
#pragma unroll
                        for (int o = 16; o > 0; o >>= 1)
#pragma unroll
                            for (int q2 = q + 1; q2 < 4; ++q2) d[q2] += __shfl_xor_sync(0xffffffffu, d[q2], o);
#pragma unroll
                        for (int q2 = q + 1; q2 < 4; ++q2) {
                            const T st = tau * d[q2];
#pragma unroll
                            for (int i = 0; i < 8; ++i) x[q2][i] = fma(-st, v[i], x[q2][i]);
                        }
                    }
                }
            }
            // 4x4 compact-WY factor of the block: g_ab = v_a . v_b (a < b), then
            // T[a][a] = tau_a, T[a][b] = -tau_b sum_{k=a}^{b-1} T[a][k] g_kb.
            T gv[6];
            {
                T vv[4][8];
#pragma unroll
                for (int q = 0; q < 4; ++q)
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const int r = lane + 32 * i, j = cb + q;
                        vv[q][i] = (q < nc) ? (r > j ? x[q][i] : (r == j ? T(1) : T(0))) : T(0);
                    }
                int e = 0;
#pragma unroll
                for (int a = 0; a < 4; ++a)
#pragma unroll
                    for (int bb = a + 1; bb < 4; ++bb, ++e) {
                        T g = T(0);
#pragma unroll
                        for (int i = 0; i < 8; ++i) g = fma(vv[a][i], vv[bb][i], g);
                        gv[e] = g;
                    }
                warp_reduce_many<6>(gv, scr);
            }
            if (lane == 0) {
                // gv index of (a, bb), a < bb: 0:(0,1) 1:(0,2) 2:(0,3) 3:(1,2) 4:(1,3) 5:(2,3)
                T tm[4][4];
#pragma unroll
                for (int a = 0; a < 4; ++a)
#pragma unroll
                    for (int bb = 0; bb < 4; ++bb) tm[a][bb] = T(0);
#pragma unroll
                for (int a = 0; a < 4; ++a) tm[a][a] = tq[a];
                const T g01 = gv[0], g02 = gv[1], g03 = gv[2], g12 = gv[3], g13 = gv[4], g23 = gv[5];
                tm[0][1] = -tq[1] * (tm[0][0] * g01);
                tm[0][2] = -tq[2] * (tm[0][0] * g02 + tm[0][1] * g12);
                tm[1][2] = -tq[2] * (tm[1][1] * g12);
                tm[0][3] = -tq[3] * (tm[0][0] * g03 + tm[0][1] * g13 + tm[0][2] * g23);
                tm[1][3] = -tq[3] * (tm[1][1] * g13 + tm[1][2] * g23);
                tm[2][3] = -tq[3] * (tm[2][2] * g23);
#pragma unroll
                for (int a = 0; a < 4; ++a)
#pragma unroll
                    for (int bb = 0; bb < 4; ++bb) Tb[b * 16 + a * 4 + bb] = tm[a][bb];
            }
        }
        unsigned long long t1 = clock64();
        if (blk == b && lane == 0) tm[0] += t1 - t0;   // owner: 4 reflectors + T
        __syncthreads();
        unsigned long long t2 = clock64();
        if (blk == b + 1 && lane == 0) tm[1] += t2 - t1;   // next owner's barrier wait
        if (blk > b && nc > 0) {
            // X <- X - V_b (T_b^T (V_b^T X)) on this warp's columns
            T vb[4][8];
            const int jb = 4 * b;
#pragma unroll
            for (int a = 0; a < 4; ++a)
#pragma unroll
                for (int i = 0; i < 8; ++i) vb[a][i] = P[(size_t)(jb + a) * RGP + padr<T>(lane + 32 * i)];
            T w[4][4];
#pragma unroll
            for (int a = 0; a < 4; ++a)
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    T acc = T(0);
#pragma unroll
                    for (int i = 0; i < 8; ++i) acc = fma(vb[a][i], x[q][i], acc);
                    w[a][q] = acc;
                }
            {
                T wf[16];
#pragma unroll
                for (int a = 0; a < 4; ++a)
#pragma unroll
                    for (int q = 0; q < 4; ++q) wf[a * 4 + q] = w[a][q];
                warp_reduce_many<16>(wf, scr);
#pragma unroll
                for (int a = 0; a < 4; ++a)
#pragma unroll
                    for (int q = 0; q < 4; ++q) w[a][q] = wf[a * 4 + q];
            }
            T tt[16];
#pragma unroll
            for (int k = 0; k < 16; ++k) tt[k] = Tb[b * 16 + k];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                T w2[4];
#pragma unroll
                for (int a = 0; a < 4; ++a) {
                    T acc = T(0);
#pragma unroll
                    for (int k = 0; k <= a; ++k) acc = fma(tt[k * 4 + a], w[k][q], acc);
                    w2[a] = acc;
                }
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    T xv = x[q][i];
#pragma unroll
                    for (int a = 0; a < 4; ++a) xv = fma(-vb[a][i], w2[a], xv);
                    x[q][i] = xv;
                }
            }
        }
        if (blk == b + 1 && lane == 0) tm[2] += clock64() - t2;  // next owner's apply
    }
    __syncthreads();  // every block applied: P's v columns are no longer read
#pragma unroll
    for (int q = 0; q < 4; ++q)
        if (q < nc)
#pragma unroll
            for (int i = 0; i < 8; ++i) P[(size_t)(cb + q) * RGP + padr<T>(lane + 32 * i)] = x[q][i];
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
    __shared__ __align__(8) uint64_t mbs[32];
    if (threadIdx.x < 32)
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((unsigned)__cvta_generic_to_shared(&mbs[threadIdx.x])) : "memory");
    unsigned par = 0;
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
        else if (MODE == 2) factor_panel_wb4<float>(Grp{(int)threadIdx.x, 0}, P, RGP, RG, 32, tau_s, tau_s + 32, P + 32 * RGP + 1024);
        else if (MODE == 6) {
            NodeRows nr{0, 0, 256, 0, 0, 0, 0};
            factor_panel_pipe<float>(Grp{(int)threadIdx.x, 0}, P, RGP, RG, 32, tau_s, mbs, par, &nr, data + 4 * 8192, 256, 0, 0);
            par ^= 1u;
        }
        else if (MODE == 3) factor_panel_wb4_timed<float>(P, RGP, RG, 32, tau_s, tau_s + 32, tm);
        else factor_panel_regs<float, 8>(P, RGP, RG, 32, tau_s);
        const unsigned long long t1 = clock64();
        total += t1 - t0;
        __syncthreads();
    }
    if (threadIdx.x == 0) cyc[blockIdx.x] = total / reps;
    __syncthreads();
    if ((MODE == 1 || MODE == 3) && blockIdx.x == 0 && threadIdx.x < 8) cyc[1024 + threadIdx.x] = tm[threadIdx.x] / reps;
}

int main() {
    float* d;
    unsigned long long* cyc;
    cudaMalloc(&d, 4 * 8192 * sizeof(float) + 256 * 32 * sizeof(float));
    cudaMalloc(&cyc, 4096 * sizeof(unsigned long long));
    float h[4 * 8192];
    unsigned s = 1;
    for (int i = 0; i < 4 * 8192; ++i) {
        s = s * 1664525u + 1013904223u;
        h[i] = ((s >> 8) & 0xffff) / 32768.f - 1.f;
    }
    cudaMemcpy(d, h, sizeof(h), cudaMemcpyHostToDevice);
    const size_t smem = sizeof(float) * (32 * fused_col_stride<float>(kFusedMaxRows) + 64 + 256 + 1024 + 8 * (32 * 20 + 16));
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
    cudaFuncSetAttribute(bench<6>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    for (int grid : {1, 148, 296}) {
        bench<6><<<grid, 256, smem>>>(d, 256, 20, cyc);
        cudaDeviceSynchronize();
        unsigned long long hc6[512];
        cudaMemcpy(hc6, cyc, grid * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < grid; ++i) avg += hc6[i];
        avg /= grid;
        printf("PIPE grid %4d: %8.0f cycles/panel = %6.0f cycles/column (%s)\n", grid, avg, avg / 32,
               cudaGetErrorString(cudaGetLastError()));
    }
    cudaFuncSetAttribute(bench<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    bench<3><<<1, 256, smem>>>(d, 256, 20, cyc);
    cudaDeviceSynchronize();
    {
        unsigned long long hc3[1032];
        cudaMemcpy(hc3, cyc, sizeof(hc3), cudaMemcpyDeviceToHost);
        printf("WB4 timed: panel %llu | owner(4 refl + T) %llu, next-owner barrier wait %llu, next-owner apply %llu (sums over 8 blocks) | per panel: sigma+sqrt %llu, v/store %llu\n",
               hc3[0], hc3[1024], hc3[1025], hc3[1026], hc3[1027], hc3[1028]);
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
