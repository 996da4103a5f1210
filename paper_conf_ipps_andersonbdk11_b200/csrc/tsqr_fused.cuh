// tsqr_fused.cuh -- the whole TSQR of a panel group in ONE persistent kernel.
//
// Every tree node -- leaf row block ("factor") or merge of two R
// factors ("factor_tree") -- is one task for one CTA.  A task walks
// its <=32-column panels: stage the gathered rows of panel p in shared memory,
// factor it with the panel held in registers (8 threads per column, one CTA
// barrier per column: matvec + rank-1 update of P:L704-711), write R / V and the
// compact-WY T, then apply (I - V T V^T)^T to the node's trailing
// columns block by block (the horizontal update of P:L665-668 done inside the
// node) and publish "slot s, panel p done".  Tasks are handed out by an atomic
// ticket in topological order (leaves, then tree level by level); a merge waits
// only for its children's panel p, so tree levels pipeline behind each other
// panel by panel instead of one launch per level and panel (Fig. 4's host loop).
// Node data are read through L2 (ld.global.cg): a slot written by another SM
// must never come from a stale L1 line.
#pragma once
#include "tsqr_kernels.cuh"

namespace caqr {

// Padded column layout of shared tiles, matched to the panel's thread layout
// (PanelLayout<8>): rows 0..31 plain, then 28-row segments each followed by
// PADS elements of padding, so the 8 segment owners of a column -- and 16-byte
// vector loads by lanes at the same offset of different segments -- hit 8
// different 16-byte bank groups (segment stride = 16 bytes mod 128).
template <typename T>
__host__ __device__ __forceinline__ int padr(int r) {
    constexpr int PADS = sizeof(T) == 4 ? 8 : 6;
    return r < 32 ? r : r + PADS * ((r - 32) / 28);
}
// Column stride for tiles of up to `rows` rows: (stride * sizeof(T)) % 128 == 16.
template <typename T>
__host__ __device__ __forceinline__ int fused_col_stride(int rows) {
    const int r32 = (rows + 31) & ~31;
    int s = padr<T>(r32);
    while ((s * (int)sizeof(T)) % 128 != 16) s += int(16 / sizeof(T));
    return s;
}

constexpr int kFusedMaxRows = 256;  // gathered rows a task may stage (TPC * SEG)

template <typename T>
inline size_t fused_smem_bytes() {
    const int RGP = fused_col_stride<T>(kFusedMaxRows);
    return sizeof(T) * (2 * 32 * (size_t)RGP + 6 * 32 * kTS + 64) + 64;
}

__device__ __forceinline__ int ld_acquire(const int* p) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(int* p, int v) {
    asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

template <typename T>
__device__ __forceinline__ T ldcg(const T* p) {
    return __ldcg(p);
}

// Version a slot's panel flag carries once the node that last writes that slot
// before tree level `level` has finished the panel: 1 = its leaf, l+2 = the
// merge of level l.
__device__ __forceinline__ int expected_version(int64_t slot, int level, int64_t L, int leaves) {
    for (int l = level - 1; l >= 0; --l) {
        const int64_t h = int64_t(1) << l;
        if ((slot & (2 * h - 1)) == 0 && slot + h < L) return l + 2;
    }
    return leaves ? 1 : 0;  // without a leaf phase the slots hold given R factors
}

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
template <typename T>
__device__ __forceinline__ T rcp_rn(T x) {
    if constexpr (sizeof(T) == 4)
        return __frcp_rn(x);
    else
        return __drcp_rn(x);
}

// 1/sqrt(s) and sqrt(s), s > 0.  fp32: hardware approximations plus one
// Newton step (~1 ulp; the reflector stays orthogonal to that level), far
// cheaper on the critical path than the IEEE-rounded sqrt / division
// subroutines.  fp64: IEEE-rounded.
template <typename T>
__device__ __forceinline__ void rsqrt_refined(T s, T& r, T& sq) {
    if constexpr (sizeof(T) == 4) {
        float y = rsqrtf(s);
        const float h = 0.5f * s * y;
        y = fmaf(-h, y, 1.5f) * y;  // y (1.5 - 0.5 s y^2)
        r = y;
        const float q = s * y;      // sqrt(s) ~ s / sqrt(s), one residual correction
        sq = fmaf(fmaf(-q, q, s), 0.5f * y, q);
    } else {
        sq = sqrt(s);
        r = __drcp_rn(sq);
    }
}
template <typename T>
__device__ __forceinline__ T rcp_refined(T d) {
    if constexpr (sizeof(T) == 4) {
        float y = __fdividef(1.0f, d);
        return fmaf(fmaf(-d, y, 1.0f), y, y);  // one Newton step
    } else {
        return __drcp_rn(d);
    }
}

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
__device__ __forceinline__ void factor_panel_wb4(T* P, int RGP, int RG, int wp, T* tau_s, T* Tb) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int cb = 4 * warp;
    const int nc = max(0, min(4, wp - cb));
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
        if (warp == b) {
            T tq[4] = {T(0), T(0), T(0), T(0)};
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                if (q < nc) {
                    const int j = cb + q;
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
#pragma unroll
                for (int o = 16; o > 0; o >>= 1)
#pragma unroll
                    for (int k = 0; k < 6; ++k) gv[k] += __shfl_xor_sync(0xffffffffu, gv[k], o);
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
        __syncthreads();
        if (warp > b && nc > 0) {
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
#pragma unroll
            for (int o = 16; o > 0; o >>= 1)
#pragma unroll
                for (int a = 0; a < 4; ++a)
#pragma unroll
                    for (int q = 0; q < 4; ++q) w[a][q] += __shfl_xor_sync(0xffffffffu, w[a][q], o);
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
    }
    __syncthreads();  // every block applied: P's v columns are no longer read
#pragma unroll
    for (int q = 0; q < 4; ++q)
        if (q < nc)
#pragma unroll
            for (int i = 0; i < 8; ++i) P[(size_t)(cb + q) * RGP + padr<T>(lane + 32 * i)] = x[q][i];
    __syncthreads();
}

// ---------------------------------------------------------------------------
// W(32 x 32) = V^T C over RG rows, V and C padded-column tiles (32 columns).
// 8 warps = 4-way split of the rows x 2 column halves; deterministic reduction.
// ---------------------------------------------------------------------------
template <typename T>
__device__ __forceinline__ void gemm_vtc(const T* Vs, const T* Cs, int RGP, int R32, T* Wp, T* W) {
    using V4 = typename Vec4<T>::type;
    constexpr int VN = Vec4<T>::n;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int ks = warp & 3, ch = warp >> 2;
    const int jg = lane & 7, cg = lane >> 3;
    const int chunk = R32 / 4;
    const int rbeg = ks * chunk, rend = rbeg + chunk;
    T acc[4][4];
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
        for (int b = 0; b < 4; ++b) acc[a][b] = T(0);
    for (int r = rbeg; r < rend; r += VN) {
        const int pr = padr<T>(r);
        V4 vv[4], cc[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) vv[e] = *reinterpret_cast<const V4*>(Vs + (size_t)(jg + 8 * e) * RGP + pr);
#pragma unroll
        for (int e = 0; e < 4; ++e)
            cc[e] = *reinterpret_cast<const V4*>(Cs + (size_t)(16 * ch + cg + 4 * e) * RGP + pr);
#pragma unroll
        for (int q = 0; q < VN; ++q)
#pragma unroll
            for (int a = 0; a < 4; ++a)
#pragma unroll
                for (int b = 0; b < 4; ++b) acc[a][b] = fma(vget<T>(vv[a], q), vget<T>(cc[b], q), acc[a][b]);
    }
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
        for (int b = 0; b < 4; ++b) Wp[(ks * 32 + jg + 8 * a) * kTS + 16 * ch + cg + 4 * b] = acc[a][b];
    __syncthreads();
    for (int e = tid; e < 32 * 32; e += kThreads) {
        const int jj = e >> 5, cc2 = e & 31;
        T sum = Wp[(0 * 32 + jj) * kTS + cc2];
        sum += Wp[(1 * 32 + jj) * kTS + cc2];
        sum += Wp[(2 * 32 + jj) * kTS + cc2];
        sum += Wp[(3 * 32 + jj) * kTS + cc2];
        W[jj * kTS + cc2] = sum;
    }
    __syncthreads();
}

// T (upper triangular, Tt[r*kTS+c] = T[r][c]) from G = V^T V (strict upper
// part in G) and tau (xLARFT forward/columnwise): T[j][j] = tau_j,
// T[0:j,j] = -tau_j T[0:j,0:j] G[0:j,j].  One warp; lane i keeps row i of T in
// registers; 4 independent accumulation chains.
template <typename T>
__device__ __forceinline__ void build_t(const T* G, const T* tau_s, int wp, T* Tt) {
    const int lane = threadIdx.x & 31;
    if (threadIdx.x >= 32) return;
    T row[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) {
        T a0 = 0, a1 = 0, a2 = 0, a3 = 0;
#pragma unroll
        for (int k = 0; k + 3 < j; k += 4) {
            a0 = fma(row[k + 0], G[(k + 0) * kTS + j], a0);
            a1 = fma(row[k + 1], G[(k + 1) * kTS + j], a1);
            a2 = fma(row[k + 2], G[(k + 2) * kTS + j], a2);
            a3 = fma(row[k + 3], G[(k + 3) * kTS + j], a3);
        }
#pragma unroll
        for (int k = j & ~3; k < j; ++k) a0 = fma(row[k], G[k * kTS + j], a0);
        const T tau = j < wp ? tau_s[j] : T(0);
        row[j] = (j == lane) ? tau : (j > lane ? -tau * ((a0 + a1) + (a2 + a3)) : T(0));
    }
#pragma unroll
    for (int j = 0; j < 32; ++j) Tt[lane * kTS + j] = row[j];
}

// C(RG x 32, in Cs) <- C - V (op(T) W) ; written straight to global rows.
template <typename T>
__device__ __forceinline__ void apply_block(const T* Vs, const T* Cs, const T* Tt, T* W, int RGP, int R32,
                                            int RG, int wp, int trans, const NodeRows& nr, T* C,
                                            int64_t ldc, int64_t cb0, int ncb) {
    using V4 = typename Vec4<T>::type;
    constexpr int VN = Vec4<T>::n;
    const int tid = threadIdx.x;
    // W2 = op(T) W: thread (column c, rows jj = jg + 8q); T is zero below its
    // diagonal, so full unrolled sums need no bounds.
    T w2[4];
    {
        const int c = tid & 31, jg = tid >> 5;
#pragma unroll
        for (int q = 0; q < 4; ++q) w2[q] = T(0);
#pragma unroll
        for (int h = 0; h < 32; h += 16) {
            T wc[16];
#pragma unroll
            for (int k = 0; k < 16; ++k) wc[k] = W[(h + k) * kTS + c];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int jj = jg + 8 * q;
                T a0 = 0, a1 = 0;
#pragma unroll
                for (int k = 0; k < 16; k += 2) {
                    if (trans) {
                        a0 = fma(Tt[(h + k) * kTS + jj], wc[k], a0);
                        a1 = fma(Tt[(h + k + 1) * kTS + jj], wc[k + 1], a1);
                    } else {
                        a0 = fma(Tt[jj * kTS + h + k], wc[k], a0);
                        a1 = fma(Tt[jj * kTS + h + k + 1], wc[k + 1], a1);
                    }
                }
                w2[q] += a0 + a1;
            }
        }
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < 4; ++q) W[((tid >> 5) + 8 * q) * kTS + (tid & 31)] = w2[q];
    __syncthreads();
    const int nq = R32 / 4;
    for (int u = tid; u < nq * 4; u += kThreads) {
        const int q = u % nq, cgrp = u / nq;
        const int r = 4 * q, cbase = 8 * cgrp;
        const int pr = padr<T>(r);
        T acc[4][8];
#pragma unroll
        for (int c = 0; c < 8; ++c) {
#pragma unroll
            for (int h = 0; h < 4 / VN; ++h) {
                const V4 t4 = *reinterpret_cast<const V4*>(Cs + (size_t)(cbase + c) * RGP + pr + h * VN);
#pragma unroll
                for (int k = 0; k < VN; ++k) acc[h * VN + k][c] = vget<T>(t4, k);
            }
        }
        for (int jj = 0; jj < wp; ++jj) {
            T vr[4];
#pragma unroll
            for (int h = 0; h < 4 / VN; ++h) {
                const V4 t4 = *reinterpret_cast<const V4*>(Vs + (size_t)jj * RGP + pr + h * VN);
#pragma unroll
                for (int k = 0; k < VN; ++k) vr[h * VN + k] = vget<T>(t4, k);
            }
            T wv[8];
#pragma unroll
            for (int h = 0; h < 8 / VN; ++h) {
                const V4 t4 = *reinterpret_cast<const V4*>(W + jj * kTS + cbase + h * VN);
#pragma unroll
                for (int k = 0; k < VN; ++k) wv[h * VN + k] = vget<T>(t4, k);
            }
#pragma unroll
            for (int c = 0; c < 8; ++c)
#pragma unroll
                for (int i = 0; i < 4; ++i) acc[i][c] = fma(-vr[i], wv[c], acc[i][c]);
        }
        // result back into the staged tile (each element is owned by exactly
        // this thread), then one coalesced pass to global below
#pragma unroll
        for (int c = 0; c < 8; ++c) {
#pragma unroll
            for (int h = 0; h < 4 / VN; ++h) {
                V4 t4;
                T* tt = reinterpret_cast<T*>(&t4);
#pragma unroll
                for (int k = 0; k < VN; ++k) tt[k] = acc[h * VN + k][c];
                *reinterpret_cast<V4*>(const_cast<T*>(Cs) + (size_t)(cbase + c) * RGP + pr + h * VN) = t4;
            }
        }
    }
    __syncthreads();
    {
        const int warp = tid >> 5, lane = tid & 31;
        for (int c = warp; c < ncb; c += kWarps) {
            T* ccol = C + (cb0 + c) * ldc;
            const T* cs = Cs + (size_t)c * RGP;
            for (int r = lane; r < RG; r += 32) ccol[gathered_row(nr, r)] = cs[padr<T>(r)];
        }
    }
    __syncthreads();
}

template <typename T>
__device__ __forceinline__ void stage_cols(T* S, int RGP, int R32, const T* M, int64_t ld, int64_t col0,
                                           int ncol, const NodeRows& nr, int RG, bool mask_panel, int p) {
    // Every thread issues all of its loads before the first store (memory-level
    // parallelism: up to 32 L2/HBM requests in flight per thread), in halves
    // of 16 for fp64 to bound register use.
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    constexpr int NA = sizeof(T) == 4 ? 4 : 2;  // columns per batch per warp
#pragma unroll
    for (int a0 = 0; a0 < 4; a0 += NA) {
        T buf[NA][8];
#pragma unroll
        for (int a = 0; a < NA; ++a) {
            const int jj = warp + 8 * (a0 + a);
            const T* mc = M + (col0 + jj) * ld;
#pragma unroll
            for (int b = 0; b < 8; ++b) {
                const int r = lane + 32 * b;
                T v = T(0);
                if (r < RG && jj < ncol && (!mask_panel || panel_entry_stored(nr, r, jj, p)))
                    v = ldcg(mc + gathered_row(nr, r));
                buf[a][b] = v;
            }
        }
#pragma unroll
        for (int a = 0; a < NA; ++a) {
            T* sc = S + (size_t)(warp + 8 * (a0 + a)) * RGP;
#pragma unroll
            for (int b = 0; b < 8; ++b) {
                const int r = lane + 32 * b;
                if (r < R32) sc[padr<T>(r)] = buf[a][b];
            }
        }
    }
}

// ---------------------------------------------------------------------------
// The persistent dataflow TSQR kernel.
// ---------------------------------------------------------------------------
template <typename T>
__global__ void __launch_bounds__(kThreads, sizeof(T) == 4 ? 2 : 1)
tsqr_fused_kernel(Geom g, T* A, T* __restrict__ Tws, int* __restrict__ sync, int nlevels, int do_leaves,
                  unsigned long long* prof) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int RGP = fused_col_stride<T>(kFusedMaxRows);
    T* P = reinterpret_cast<T*>(smem_raw);
    T* Cs = P + 32 * (size_t)RGP;
    T* Wp = Cs + 32 * (size_t)RGP;
    T* Tt = Wp + 4 * 32 * kTS;
    T* W = Tt + 32 * kTS;
    T* tau_s = W + 32 * kTS;
    __shared__ int s_task;
    int* ticket = sync;
    int* flags = sync + 32;  // [L][npan]
    const int64_t leaf_tasks = do_leaves ? g.P : 0;  // one task per chain of K tiles
    int64_t total = leaf_tasks;
    for (int l = 0; l < nlevels; ++l) {
        const int64_t h = int64_t(1) << l;
        total += (g.P - 1 >= h) ? (g.P - 1 - h) / (2 * h) + 1 : 0;
    }
    // optional phase profile (diagnostics; prof == nullptr in normal use)
    // (accumulators live in shared memory: no registers taken from the math)
    __shared__ unsigned long long pacc[13];
    if (threadIdx.x < 13) pacc[threadIdx.x] = threadIdx.x == 12 ? (unsigned long long)clock64() : 0ull;
#define CAQR_PROF(k)                                              \
    do {                                                          \
        if (prof && threadIdx.x == 0) {                           \
            const unsigned long long t1_ = clock64();             \
            pacc[k] += t1_ - pacc[12];                            \
            pacc[12] = t1_;                                       \
        }                                                         \
    } while (0)
    for (;;) {
        __syncthreads();
        CAQR_PROF(0);
        if (threadIdx.x == 0) s_task = atomicAdd(ticket, 1);
        __syncthreads();
        const int64_t task = s_task;
        if (task >= total) break;
        int level = -1;
        int64_t node = task;
        if (task >= leaf_tasks) {
            node = task - leaf_tasks;
            level = 0;
            for (;;) {
                const int64_t h = int64_t(1) << level;
                const int64_t nm = (g.P - 1 >= h) ? (g.P - 1 - h) / (2 * h) + 1 : 0;
                if (node < nm) break;
                node -= nm;
                ++level;
            }
        }
        int64_t slot_a, slot_b = -1;
        int ver_a = 0, ver_b = 0;
        if (level < 0) {
            slot_a = node;
        } else {
            slot_a = node << (level + 1);
            slot_b = slot_a + (int64_t(1) << level);
            ver_a = expected_version(slot_a, level, g.P, do_leaves);
            ver_b = expected_version(slot_b, level, g.P, do_leaves);
        }
        const int my_ver = level + 2;
        // a chain walks its tiles in order; a merge is one "tile"
        const int64_t ntile = level < 0 ? min(g.K, g.L - node * g.K) : 1;
        for (int kt = 0; kt < ntile; ++kt)
        for (int p = 0; p < g.npan; ++p) {
            const int wp = min(kPW, g.ncols - 32 * p);
            if (level >= 0 && threadIdx.x == 0) {  // children's panel p must be final
                const int* fa = flags + slot_a * g.npan + p;
                const int* fb = flags + slot_b * g.npan + p;
                while (ld_acquire(fa) < ver_a) __nanosleep(64);
                while (ld_acquire(fb) < ver_b) __nanosleep(64);
            }
            __syncthreads();
            CAQR_PROF(1);
            if (prof && threadIdx.x == 0) pacc[level < 0 ? 10 : 11] += 1;
            const NodeRows nr = node_rows(g, level, node, p, wp, kt);
            const int RG = nr.n0 + nr.n1;
            const int R32 = (RG + 31) & ~31;
            const int64_t c0 = g.col0 + 32 * p;
            // ---- panel: stage, factor, store R/V, T ------------------------
            stage_cols(P, RGP, R32, A, g.lda, c0, wp, nr, RG, true, p);
            if (threadIdx.x < 32) tau_s[threadIdx.x] = T(0);
            __syncthreads();
            CAQR_PROF(2);
            factor_panel_wb4<T>(P, RGP, RG, wp, tau_s, Wp);
            CAQR_PROF(3);
            {
                const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
                for (int jj = warp; jj < wp; jj += kWarps) {
                    T* col = A + (c0 + jj) * g.lda;
                    T* pc = P + (size_t)jj * RGP;
                    for (int r = lane; r < R32; r += 32) {
                        const bool in = r < RG;
                        const T val = pc[padr<T>(r)];
                        if (in && panel_entry_stored(nr, r, jj, p)) col[gathered_row(nr, r)] = val;
                        // V form in place: unit head, zeros above, structure masks
                        const T v = in ? v_entry<T>(nr, r, jj, p, val) : T(0);
                        pc[padr<T>(r)] = v;
                    }
                }
                for (int jj = wp + warp; jj < 32; jj += kWarps) {
                    T* pc = P + (size_t)jj * RGP;
                    for (int r = lane; r < R32; r += 32) pc[padr<T>(r)] = T(0);
                }
            }
            __syncthreads();
            CAQR_PROF(4);
            gemm_vtc(P, P, RGP, R32, Wp, W);  // G = V^T V
            build_t(W, tau_s, wp, Tt);
            __syncthreads();
            {
                T* tb = Tws + nr.tblk * (kPW * kPW);
                for (int e = threadIdx.x; e < kPW * kPW; e += kThreads) {
                    const int r = e & 31, c = e >> 5;
                    tb[e] = Tt[r * kTS + c];
                }
            }
            CAQR_PROF(5);
            // ---- trailing columns of this node, 32 at a time -------------------
            const int64_t tfirst = c0 + 32, tend = g.col0 + g.ncols;
            for (int64_t cb0 = tfirst; cb0 < tend; cb0 += 32) {
                const int ncb = (int)(tend - cb0 < 32 ? tend - cb0 : 32);
                stage_cols(Cs, RGP, R32, static_cast<const T*>(A), g.lda, cb0, ncb, nr, RG, false, p);
                __syncthreads();
                CAQR_PROF(6);
                gemm_vtc(P, Cs, RGP, R32, Wp, W);
                CAQR_PROF(7);
                apply_block(P, Cs, Tt, W, RGP, R32, RG, wp, 1, nr, A, g.lda, cb0, ncb);
                CAQR_PROF(8);
            }
            // ---- publish ----------------------------------------------------------
            __threadfence();
            __syncthreads();
            if (threadIdx.x == 0 && kt == ntile - 1)  // the slot's R rows of panel p are final
                st_release(flags + slot_a * g.npan + p, level < 0 ? 1 : my_ver);
            CAQR_PROF(9);
        }
    }
    if (prof && threadIdx.x == 0)
        for (int k = 0; k < 12; ++k) atomicAdd(prof + k, pacc[k]);
#undef CAQR_PROF
}

}  // namespace caqr
