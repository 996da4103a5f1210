// panel_variants.cuh -- superseded panel-factorization layouts, kept for the
// design-study microbenchmarks in tools/ only (not part of libcaqr):
//   factor_panel_regs  round 1: 8 threads per column, one CTA barrier per column;
//   factor_panel_wb4   round 1-2 default: 4-column blocks, one owner warp per block,
//                      one CTA barrier per block (29.4k cycles per 256 x 32 panel alone,
//                      replaced by factor_panel_pipe: 23.2k; fused kernel 5.93 -> 5.36 ms).
#pragma once
#include "../paper_conf_ipps_andersonbdk11_b200/csrc/tsqr_fused.cuh"

namespace caqr {
// Group reduction over the TPC consecutive lanes that own one column.
template <int TPC, typename T>
__device__ __forceinline__ T group_sum(T v, unsigned mask) {
#pragma unroll
    for (int o = 1; o < TPC; o <<= 1) v += __shfl_xor_sync(mask, v, o);
    return v;
}

// Row layout of a column's TPC owner threads: the top 32 rows (where every
// reflector head of the panel lies) are dealt round-robin, TOPR = 32/TPC rows
// per thread; the remaining rows are contiguous chunks of BULK rows.  Only the
// TOPR top rows ever need per-row "r > j" logic.
template <int TPC>
struct PanelLayout {
    static constexpr int SEG = kFusedMaxRows / TPC;
    static constexpr int TOPR = 32 / TPC;
    static constexpr int BULK = SEG - TOPR;
    __device__ static __forceinline__ int row(int s, int i) {
        return i < TOPR ? s + TPC * i : 32 + BULK * s + (i - TOPR);
    }
};

template <typename T, int TPC>
__device__ __forceinline__ void load_col(const T* col, int s, T (&x)[PanelLayout<TPC>::SEG]) {
    using Lay = PanelLayout<TPC>;
    using V4 = typename Vec4<T>::type;
    constexpr int VN = Vec4<T>::n;
#pragma unroll
    for (int i = 0; i < Lay::TOPR; ++i) x[i] = col[padr<T>(s + TPC * i)];
    if constexpr (Lay::BULK % 4 == 0) {
#pragma unroll
        for (int i = 0; i < Lay::BULK; i += VN) {
            const V4 q = *reinterpret_cast<const V4*>(col + padr<T>(32 + Lay::BULK * s + i));
#pragma unroll
            for (int k = 0; k < VN; ++k) x[Lay::TOPR + i + k] = vget<T>(q, k);
        }
    } else {
#pragma unroll
        for (int i = 0; i < Lay::BULK; ++i) x[Lay::TOPR + i] = col[padr<T>(32 + Lay::BULK * s + i)];
    }
}

template <typename T, int TPC>
__device__ __forceinline__ void store_col(T* col, int s, const T (&x)[PanelLayout<TPC>::SEG]) {
    using Lay = PanelLayout<TPC>;
    using V4 = typename Vec4<T>::type;
    constexpr int VN = Vec4<T>::n;
#pragma unroll
    for (int i = 0; i < Lay::TOPR; ++i) col[padr<T>(s + TPC * i)] = x[i];
    if constexpr (Lay::BULK % 4 == 0) {
#pragma unroll
        for (int i = 0; i < Lay::BULK; i += VN) {
            V4 q;
            T* qq = reinterpret_cast<T*>(&q);
#pragma unroll
            for (int k = 0; k < VN; ++k) qq[k] = x[Lay::TOPR + i + k];
            *reinterpret_cast<V4*>(col + padr<T>(32 + Lay::BULK * s + i)) = q;
        }
    } else {
#pragma unroll
        for (int i = 0; i < Lay::BULK; ++i) col[padr<T>(32 + Lay::BULK * s + i)] = x[Lay::TOPR + i];
    }
}

// ---------------------------------------------------------------------------
// Factor the staged panel P (RG x wp, padded column layout) in registers.
// Thread t owns column c = t / TPC (rows per PanelLayout, s = t % TPC).
// On exit: P holds the stored form (R on/above the diagonal, v below) and
// tau_s[0..wp) the reflector scalars.
// All warp shuffles run with the full mask in warp-uniform control flow (a
// partial mask under divergence compiles to slow WARPSYNC.COLLECTIVE code);
// groups that have nothing to do compute on zeros and discard.
// ---------------------------------------------------------------------------
template <typename T, int TPC>
__device__ __forceinline__ void factor_panel_regs(T* P, int RGP, int RG, int wp, T* tau_s) {
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
#pragma unroll
        for (int o = 1; o < TPC; o <<= 1) {
            sig += __shfl_xor_sync(0xffffffffu, sig, o);
            al += __shfl_xor_sync(0xffffffffu, al, o);
        }
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
        store_col<T, TPC>(P + (size_t)j * RGP, s, v);
        if (s == 0) tau_s[j] = tau;
    };

    if (warp == 0) reflector(0);
    __syncthreads();
    for (int j = 0; j < wp; ++j) {
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
            const T d = group_sum<TPC>((d0 + d1) + (d2 + d3), 0xffffffffu);
            if (active && c > j) {
                const T st = tau * d;
#pragma unroll
                for (int i = 0; i < SEG; ++i) x[i] = fma(-st, v[i], x[i]);
            }
        }
        if (j + 1 < wp && warp == (j + 1) / GPW) reflector(j + 1);
        __syncthreads();
    }
    // stored form back into P (R on/above the diagonal, v below)
    if (active) store_col<T, TPC>(P + (size_t)c * RGP, s, x);
    __syncthreads();
}

// ---------------------------------------------------------------------------
// Panel factorization, 4-column blocks ("WB4").  Warp w owns panel columns
// 4w..4w+3; lane l holds rows l + 32 i (i < 8) of each of them in registers
// (every reflector head, row j < 32, sits in lane j, i = 0).  Block b: warp b
// computes its 4 reflectors warp-locally (shuffle reductions only, no CTA
// barrier), publishes v (V form) into P and its 4x4 compact-WY factor, one CTA
// barrier, then every warp to the right applies the block as
// X <- X - V (T^T (V^T X)) to its own 4 columns.  8 barriers per 32 columns.
// On exit P holds the stored form (R on/above the diagonal, v below) and
// tau_s[0..wp) the reflector scalars.
// ---------------------------------------------------------------------------
template <typename T>
__device__ __forceinline__ void factor_panel_wb4(const Grp& G, T* P, int RGP, int RG, int wp, T* tau_s, T* Tb,
                                                 T* scr_all, const NodeRows* out_nr = nullptr, T* out_A = nullptr,
                                                 int64_t out_lda = 0, int64_t out_c0 = 0, int out_p = 0) {
    const int warp = G.tid >> 5, lane = G.tid & 31;
    // block blk = 7 - warp: the warp that owns the next block always has the
    // highest warp id among the warps still applying the current one, so the
    // scheduler (highest-id-first) favours the critical path
    // (through a shuffle so that the compiler knows blk -- and every branch on
    // it around the warp reductions -- is warp-uniform: no WARPSYNC.COLLECTIVE)
    const int blk = __shfl_sync(0xffffffffu, kWarps - 1 - warp, 0);
    const int cb = 4 * blk;
    const int nc = max(0, min(4, wp - cb));
    T* scr = scr_all + warp * (32 * 20 + 16);  // warp-private reduction scratch
    T x[4][8];
#pragma unroll
    for (int q = 0; q < 4; ++q)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int r = lane + 32 * i;
            x[q][i] = (q < nc && r < RG) ? P[(size_t)(cb + q) * RGP + padr<T>(r)] : T(0);
        }
    gsync(G);  // all columns are in registers before P gets v's
    const int nblk = (wp + 3) / 4;
    for (int b = 0; b < nblk; ++b) {
        if (blk == b) {
            // One 4-value warp reduction per reflector j = cb + q, taken on the
            // UNSCALED column (rows r > j): its squared norm, its dots with the
            // later columns k > q (v^T x_k = x_k[j] + scale * e_k) and with the
            // earlier v_a, a < q (g_aq = v_a[j] + scale * f_a).  So the norm,
            // the block update and the compact-WY Gram entries share one
            // reduction instead of three.
            T tq[4] = {T(0), T(0), T(0), T(0)};
            T gv[6] = {T(0), T(0), T(0), T(0), T(0), T(0)};
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                if (q < nc) {
                    const int j = cb + q;
                    T red[4] = {T(0), T(0), T(0), T(0)};
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const int r = lane + 32 * i;
                        const T xq = r > j ? x[q][i] : T(0);
                        red[0] = fma(xq, xq, red[0]);
#pragma unroll
                        for (int m = 0; m < 3; ++m) {
                            // slot 1 + m: e_{q+1+m} for m < 3 - q, else f_{m-(3-q)}
                            const int k = m < 3 - q ? q + 1 + m : m - (3 - q);
                            red[1 + m] = fma(xq, x[k][i], red[1 + m]);
                        }
                    }
                    warp_reduce_many<4>(red, scr);
                    const T al = __shfl_sync(0xffffffffu, x[q][0], j);
                    T head[3];
#pragma unroll
                    for (int m = 0; m < 3; ++m) {
                        const int k = m < 3 - q ? q + 1 + m : m - (3 - q);
                        head[m] = __shfl_sync(0xffffffffu, x[k][0], j);
                    }
                    const T sg = red[0];
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
#pragma unroll
                    for (int m = 0; m < 3; ++m) {
                        if (m < 3 - q) {  // apply H_j to the later column k
                            const int k = q + 1 + m;
                            const T st = tau * fma(scale, red[1 + m], head[m]);
                            if (tau != T(0))
#pragma unroll
                                for (int i = 0; i < 8; ++i) x[k][i] = fma(-st, v[i], x[k][i]);
                        } else {  // Gram entry g_aq, a < q (index of (a, q), a < q)
                            const int a = m - (3 - q);
                            const int e = a == 0 ? q - 1 : (a == 1 ? q + 1 : 5);
                            gv[e] = fma(scale, red[1 + m], head[m]);
                        }
                    }
                }
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
        gsync(G);
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
            for (int k = 0; k < 16; k += Vec4<T>::n) {
                const typename Vec4<T>::type t4 = *reinterpret_cast<const typename Vec4<T>::type*>(Tb + b * 16 + k);
#pragma unroll
                for (int e = 0; e < Vec4<T>::n; ++e) tt[k + e] = vget<T>(t4, e);
            }
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
    }
    gsync(G);  // every block applied: P's v columns are no longer read
    if (out_A) {
        // epilogue straight from registers: the stored form (R / v, structure
        // masks) to global, the V form (unit head, zeros elsewhere) into P,
        // zero columns beyond wp -- no extra pass over P
        const NodeRows& nr = *out_nr;
        // per row (shared by the 4 columns): segment, absolute row, and the
        // structure test's row key -- r for segment 0 (stored iff r <= jj when
        // it is an R slot), r - n0 - 32p for an upper-triangular segment 1
        // (stored iff key <= jj), -inf-like for a dense one
        int64_t grow[8];
        int key[8];
        bool seg0[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int r = lane + 32 * i;
            seg0[i] = r < nr.n0;
            grow[i] = seg0[i] ? nr.r0 + r : nr.r1 + (r - nr.n0);
            key[i] = seg0[i] ? (nr.seg0_tri ? r : -1) : (nr.seg1_upper ? r - nr.n0 - 32 * out_p : -1);
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int jj = cb + q;
            T* col = out_A + (out_c0 + jj) * out_lda;
            T* pcol = P + (size_t)jj * RGP;
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const int r = lane + 32 * i;
                const bool in = q < nc && r < RG;
                const bool stored = key[i] <= jj;
                if (in && stored) col[grow[i]] = x[q][i];
                T v = T(0);
                if (in) {
                    if (seg0[i]) v = nr.seg0_tri ? (r == jj ? T(1) : T(0)) : (r > jj ? x[q][i] : (r == jj ? T(1) : T(0)));
                    else v = stored ? x[q][i] : T(0);
                }
                pcol[padr<T>(r)] = v;
            }
        }
    } else {
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (q < nc)
#pragma unroll
                for (int i = 0; i < 8; ++i) P[(size_t)(cb + q) * RGP + padr<T>(lane + 32 * i)] = x[q][i];
    }
    gsync(G);
}

}  // namespace caqr
