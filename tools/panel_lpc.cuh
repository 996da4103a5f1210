// panel_lpc.cuh -- "lane per column" Householder panel factorization.
// EXPERIMENT (not used by libcaqr): measured by tools/lpc_bench.cu on a B200 at
// 55k cycles per 256 x 32 panel vs 29k for the library's WB4 scheme (1 CTA),
// so WB4 stays; kept as the record of that negative result.
//
// The paper's fastest apply kernel keeps each thread's data in registers and
// does its reductions serially inside the thread ("register-file serial
// reductions", cyclic column ownership, Fig. 6).  On
// B200 the same idea removes every cross-lane shuffle from the panel's critical
// path: warp w holds gathered rows [32w, 32w + 32) of the panel, lane c holds
// column c of those rows in 32 registers.  Per reflector j (xLARFG, reading S1):
//   1. every lane: partial sigma of its own column over its rows r > j (serial);
//      lane j of each warp publishes its partial (and warp 0 the head alpha);
//   2. CTA barrier; every thread sums the 8 partials and derives beta, tau,
//      scale = 1/(alpha - beta) redundantly (no broadcast needed);
//   3. lane j scales its rows into v (unit head, zeros above) and writes them to
//      the shared panel (the V form the trailing update reads), __syncwarp;
//   4. lanes c > j: partial dot v^T x_c over the warp's rows (serial), published
//      per (warp, column); CTA barrier;
//   5. lanes c > j: s_c = sum of the 8 partials, x_c -= tau s_c v (P:L704-711:
//      the matvec and the rank-1 update).
// Two CTA barriers and no shuffles per column.  Reflector heads (rows j < 32)
// all sit in warp 0.
#pragma once
#include "../paper_conf_ipps_andersonbdk11_b200/csrc/tsqr_kernels.cuh"

namespace caqr {

// Shared scratch: 8 sigma partials + alpha, and 8 x 32 dot partials.
constexpr int kLpcScratch = 16 + 8 * 32;

// P: staged panel (column c at P + c * RGP, rows 0..RG-1, RG <= 256), read into
// registers and overwritten with the V form (unit head, zeros above the head).
// x (out): this lane's column segment in stored form (R on/above the diagonal,
// v below) -- the caller writes it out.  tau_s[j]: reflector scalars.
template <typename T>
__device__ __forceinline__ void factor_panel_lpc(T* P, int RGP, int RG, int wp, T* tau_s, T* scr, T (&x)[32]) {
    static_assert(sizeof(T) == 4, "fp32 panel");
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int rbase = 32 * warp;
    T* sig_s = scr;       // [8] partial sigmas, [8] alpha
    T* dot_s = scr + 16;  // [8][32]
    {
        const T* col = P + (size_t)lane * RGP + rbase;
#pragma unroll
        for (int i = 0; i < 32; i += 4) {
            const float4 q = *reinterpret_cast<const float4*>(col + i);
            x[i] = q.x;
            x[i + 1] = q.y;
            x[i + 2] = q.z;
            x[i + 3] = q.w;
        }
#pragma unroll
        for (int i = 0; i < 32; ++i)
            if (lane >= wp || rbase + i >= RG) x[i] = T(0);
    }
    __syncthreads();  // all columns in registers before P receives v's
    for (int j = 0; j < wp; ++j) {
        // 1. partial sigma over rows > j (warp 0 holds the heads, rows 0..31)
        {
            T s0 = 0, s1 = 0, s2 = 0, s3 = 0, al = 0;
            if (warp == 0) {
#pragma unroll
                for (int i = 0; i < 32; i += 4) {
                    s0 = i > j ? fma(x[i], x[i], s0) : s0;
                    s1 = i + 1 > j ? fma(x[i + 1], x[i + 1], s1) : s1;
                    s2 = i + 2 > j ? fma(x[i + 2], x[i + 2], s2) : s2;
                    s3 = i + 3 > j ? fma(x[i + 3], x[i + 3], s3) : s3;
                }
#pragma unroll
                for (int i = 0; i < 32; ++i) al = i == j ? x[i] : al;
            } else {
#pragma unroll
                for (int i = 0; i < 32; i += 4) {
                    s0 = fma(x[i], x[i], s0);
                    s1 = fma(x[i + 1], x[i + 1], s1);
                    s2 = fma(x[i + 2], x[i + 2], s2);
                    s3 = fma(x[i + 3], x[i + 3], s3);
                }
            }
            if (lane == j) {
                sig_s[warp] = (s0 + s1) + (s2 + s3);
                if (warp == 0) sig_s[8] = al;
            }
        }
        __syncthreads();
        // 2. reflector scalars, redundantly in every thread
        T tau = T(0), beta, scale = T(1);
        {
            const float4 a = *reinterpret_cast<const float4*>(sig_s);
            const float4 b = *reinterpret_cast<const float4*>(sig_s + 4);
            const T al = sig_s[8];
            const T sg = ((a.x + a.y) + (a.z + a.w)) + ((b.x + b.y) + (b.z + b.w));
            beta = al;
            if (j < RG && sg != T(0)) {
                const T ss = fma(al, al, sg);
                const T aa = fabs(al);
                T rmu = rsqrtf(ss);
                {
                    const T h = 0.5f * ss * rmu;
                    rmu = fmaf(-h, rmu, 1.5f) * rmu;
                }
                const T q = ss * rmu;
                const T mu = fmaf(fmaf(-q, q, ss), 0.5f * rmu, q);
                beta = -copysignf(mu, al);
                tau = fmaf(aa, rmu, 1.0f);
                const T d = aa + mu;
                T y = __fdividef(1.0f, d);
                y = fmaf(fmaf(-d, y, 1.0f), y, y);
                scale = copysignf(y, al);
            }
        }
        if (tau == T(0)) {  // H_j = I: v = e_j, nothing to update (uniform branch)
            if (lane == j) {
                T* vc = P + (size_t)j * RGP + rbase;
#pragma unroll
                for (int i = 0; i < 32; i += 4)
                    *reinterpret_cast<float4*>(vc + i) =
                        make_float4(rbase + i == j ? 1.f : 0.f, rbase + i + 1 == j ? 1.f : 0.f,
                                    rbase + i + 2 == j ? 1.f : 0.f, rbase + i + 3 == j ? 1.f : 0.f);
                if (warp == 0) tau_s[j] = T(0);
            }
            __syncthreads();  // sig_s of column j read by all before column j+1 writes it
            continue;
        }
        // 3. lane j: v (unit head, zeros above) into P; stored form kept in x
        if (lane == j) {
            T* vc = P + (size_t)j * RGP + rbase;
            if (warp == 0) {
#pragma unroll
                for (int i = 0; i < 32; ++i) x[i] = i > j ? x[i] * scale : (i == j ? beta : x[i]);
#pragma unroll
                for (int i = 0; i < 32; i += 4) {
                    float4 q;
                    q.x = i > j ? x[i] : (i == j ? 1.f : 0.f);
                    q.y = i + 1 > j ? x[i + 1] : (i + 1 == j ? 1.f : 0.f);
                    q.z = i + 2 > j ? x[i + 2] : (i + 2 == j ? 1.f : 0.f);
                    q.w = i + 3 > j ? x[i + 3] : (i + 3 == j ? 1.f : 0.f);
                    *reinterpret_cast<float4*>(vc + i) = q;
                }
                tau_s[j] = tau;
            } else {
#pragma unroll
                for (int i = 0; i < 32; ++i) x[i] *= scale;
#pragma unroll
                for (int i = 0; i < 32; i += 4)
                    *reinterpret_cast<float4*>(vc + i) = make_float4(x[i], x[i + 1], x[i + 2], x[i + 3]);
            }
        }
        __syncwarp();
        // 4. partial dots of v with the later columns
        T v[32];
        {
            const T* vc = P + (size_t)j * RGP + rbase;
#pragma unroll
            for (int i = 0; i < 32; i += 4) {
                const float4 q = *reinterpret_cast<const float4*>(vc + i);
                v[i] = q.x;
                v[i + 1] = q.y;
                v[i + 2] = q.z;
                v[i + 3] = q.w;
            }
            T d0 = 0, d1 = 0, d2 = 0, d3 = 0;
#pragma unroll
            for (int i = 0; i < 32; i += 4) {
                d0 = fma(v[i], x[i], d0);
                d1 = fma(v[i + 1], x[i + 1], d1);
                d2 = fma(v[i + 2], x[i + 2], d2);
                d3 = fma(v[i + 3], x[i + 3], d3);
            }
            dot_s[warp * 32 + lane] = (d0 + d1) + (d2 + d3);
        }
        __syncthreads();
        // 5. rank-1 update of the later columns
        if (lane > j) {
            T s = T(0);
#pragma unroll
            for (int w = 0; w < 8; ++w) s += dot_s[w * 32 + lane];
            const T st = tau * s;
#pragma unroll
            for (int i = 0; i < 32; ++i) x[i] = fma(-st, v[i], x[i]);
        }
    }
    __syncthreads();  // P holds every v; scratch free
}

}  // namespace caqr
