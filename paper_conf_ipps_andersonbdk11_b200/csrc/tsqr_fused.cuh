// tsqr_fused.cuh -- the whole TSQR of a panel group in ONE persistent kernel.
//
// Every tree node -- leaf row block ("factor") or merge of two R
// factors ("factor_tree") -- is one task for one CTA.  A task walks
// its <=32-column panels: stage the gathered rows of panel p in shared memory,
// factor it with the panel held in registers (factor_panel_pipe: each warp owns
// 4 columns, reflectors published one by one through shared-memory mbarriers:
// matvec + rank-1 update of P:L704-711), write R / V and the compact-WY T
// (P:L224-246), then apply (I - V T V^T)^T to the node's trailing
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

// Row index of a shared panel / C tile.  Plain (identity): every access pattern
// that remains is conflict-free without row padding -- the panel and the staging /
// write-back loops have lanes on consecutive rows, and the GEMM fragments
// differ by column, which the column stride (16 bytes mod 128) spreads over
// the banks.  (An earlier 8-threads-per-column panel layout needed padding
// after every 28-row segment; its integer divide cost ~8 % of the kernel's
// instructions.)
template <typename T>
__host__ __device__ __forceinline__ int padr(int r) {
    return r;
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

template <typename T>
__device__ __forceinline__ T rcp_rn(T x) {
    if constexpr (sizeof(T) == 4)
        return __frcp_rn(x);
    else
        return __drcp_rn(x);
}

// 1/sqrt(s) and sqrt(s), s > 0, for the reflector scalars mu, tau = 1 + |alpha|/mu
// and 1/(|alpha| + mu).  fp32: hardware approximations plus one Newton step
// (~1 ulp), far cheaper on the reflector critical path than the IEEE-rounded
// subroutines.  Measured round 2 (1M x 192): IEEE __fsqrt_rn / __frcp_rn give
// ||Q^T Q - I|| 2.9e-6 instead of 6.8e-6 (fp32 LAPACK: 2.0e-6; bound 1e-5) at
// +5 % time (6.03 vs 5.74 ms), so the hot path keeps the approximations;
// CAQR_IEEE_SCALARS (compile-time) selects the IEEE ones.  fp64: IEEE-rounded.
template <typename T>
__device__ __forceinline__ void rsqrt_refined(T s, T& r, T& sq) {
    if constexpr (sizeof(T) == 4) {
#ifdef CAQR_IEEE_SCALARS
        sq = __fsqrt_rn(s);
        r = __frcp_rn(sq);
#else
        float y = rsqrtf(s);
        const float h = 0.5f * s * y;
        y = fmaf(-h, y, 1.5f) * y;  // y (1.5 - 0.5 s y^2)
        r = y;
        const float q = s * y;      // sqrt(s) ~ s / sqrt(s), one residual correction
        sq = fmaf(fmaf(-q, q, s), 0.5f * y, q);
#endif
    } else {
        sq = sqrt(s);
        r = __drcp_rn(sq);
    }
}
template <typename T>
__device__ __forceinline__ T rcp_refined(T d) {
    if constexpr (sizeof(T) == 4) {
#ifdef CAQR_IEEE_SCALARS
        return __frcp_rn(d);
#else
        float y = __fdividef(1.0f, d);
        return fmaf(fmaf(-d, y, 1.0f), y, y);  // one Newton step
#endif
    } else {
        return __drcp_rn(d);
    }
}


// A group of 256 threads (8 warps) that runs one device routine: the whole
// CTA in the one-role kernel, or one of the two roles of the look-ahead
// kernel (named barrier per role).  tid is the group-local thread index.
__device__ __forceinline__ void gsync(const Grp& g) {
    if (g.bar == 0)
        __syncthreads();
    else
        asm volatile("bar.sync %0, 256;" ::"r"(g.bar) : "memory");
}

// Sum N values across the 32 lanes of a warp; every lane gets all N totals.
// Measured on B200: a 5-level SHFL butterfly costs ~150 cycles and SHFL issue
// is ~9 cycles, so N interleaved butterflies (5N shuffles) are throughput-bound
// (16 values: ~760 cycles).  Transpose through shared memory instead: each lane
// stores its N partials, lane l sums value l % NP over a group of NP rows, a
// few shuffles combine the groups, and the totals are broadcast back.
// `scr` is this warp's private scratch of 32 * (NP + 4) + NP elements.
// As warp_reduce_many, but each lane only needs one total: lane l returns the
// sum of value l % NP (no broadcast back through shared memory).
template <int N, typename T>
__device__ __forceinline__ T warp_reduce_scatter_smem(const T (&v)[N], T* scr) {
    constexpr int NP = N <= 1 ? 1 : N <= 2 ? 2 : N <= 4 ? 4 : N <= 8 ? 8 : N <= 16 ? 16 : 32;
    constexpr int LD = NP + 4;
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int k = 0; k < NP; ++k) scr[lane * LD + k] = k < N ? v[k] : T(0);
    __syncwarp();
    const int k = lane % NP, g = lane / NP;
    T acc = T(0);
#pragma unroll
    for (int r = 0; r < NP; ++r) acc += scr[(g * NP + r) * LD + k];
#pragma unroll
    for (int o = NP; o < 32; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    __syncwarp();
    return acc;
}

template <int N, typename T>
__device__ __forceinline__ void warp_reduce_many(T (&v)[N], T* scr) {
    constexpr int NP = N <= 1 ? 1 : N <= 2 ? 2 : N <= 4 ? 4 : N <= 8 ? 8 : N <= 16 ? 16 : 32;
    constexpr int LD = NP + 4;  // row stride (16-byte aligned rows, spread banks)
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int k = 0; k < NP; ++k) scr[lane * LD + k] = k < N ? v[k] : T(0);
    __syncwarp();
    const int k = lane % NP, g = lane / NP;
    T acc = T(0);
#pragma unroll
    for (int r = 0; r < NP; ++r) acc += scr[(g * NP + r) * LD + k];
#pragma unroll
    for (int o = NP; o < 32; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    __syncwarp();
    if (lane < NP) scr[32 * LD + lane] = acc;
    __syncwarp();
#pragma unroll
    for (int q = 0; q < N; ++q) v[q] = scr[32 * LD + q];
    __syncwarp();
}

// Global stores with an L2 evict-first policy (created once per use site):
// data written for the last time by the factorization -- the T blocks, a
// panel's final V rows -- should not push the tiles still being updated out
// of L2.  (1M x 192: DRAM traffic 2.29 -> 1.87 GB per launch.)
__device__ __forceinline__ uint64_t l2_evict_first_policy() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ void st_evict_first(float* p, float v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;" ::"l"(p), "f"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_evict_first(double* p, double v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.f64 [%0], %1, %2;" ::"l"(p), "d"(v), "l"(pol) : "memory");
}

// ---------------------------------------------------------------------------
// Panel factorization, reflector-pipelined ("PIPE").  Same ownership as the
// earlier WB4 kernel (now tools/panel_variants.cuh): warp w owns panel columns
// 4(7-w) .. +3, lane l rows l + 32 i.  But no CTA barrier per 4-column block:
// reflector j is published (v_j in P[:, j], tau_j) through its own
// shared-memory mbarrier, and every warp that owns later columns
// applies H_j = I - tau_j v_j v_j^T to them as soon as it arrives (the
// unblocked xGEQR2 order).  The next block's owner has applied
// all but the newest reflector when its turn comes, so the hand-off costs one
// reflector application instead of a barrier plus a 4-reflector block update.
// The owner's own block: one warp reduction per reflector gives the squared
// norm and the dots with the block's later columns (WB4's unscaled-column
// trick); the compact-WY T comes afterwards from G = V^T V (build_t).
// mb: 32 mbarriers (arrival count 1), `parity` = this call's phase (each call
// arrives exactly once on every one of them, including columns >= wp).
// ---------------------------------------------------------------------------
__device__ __forceinline__ void mbar_arrive1(uint64_t* mb) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"((unsigned)__cvta_generic_to_shared(mb))
                 : "memory");
}
__device__ __forceinline__ void mbar_wait_parity(uint64_t* mb, unsigned parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "PIPE_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra PIPE_WAIT_%=;\n}" ::"r"((unsigned)__cvta_generic_to_shared(mb)),
        "r"(parity)
        : "memory");
}
// All-lane sum of N values by a SHFL butterfly (N <= 4: fewer dependent steps
// than the shared-memory transpose of warp_reduce_many).
template <int N, typename T>
__device__ __forceinline__ void warp_allsum_bfly(T (&v)[N]) {
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1)
#pragma unroll
        for (int k = 0; k < N; ++k) v[k] += __shfl_xor_sync(0xffffffffu, v[k], o);
}

template <typename T>
__device__ __forceinline__ void factor_panel_pipe(const Grp& G, T* P, int RGP, int RG, int wp, T* tau_s,
                                                  uint64_t* mb, unsigned parity, const NodeRows* out_nr,
                                                  T* out_A, int64_t out_lda, int64_t out_c0, int out_p,
                                                  T* Gout = nullptr, T* scr_all = nullptr) {
    const int warp = G.tid >> 5, lane = G.tid & 31;
    const int blk = __shfl_sync(0xffffffffu, kWarps - 1 - warp, 0);
    const int cb = 4 * blk;
    const int nc = max(0, min(4, wp - cb));
    // every warp reads and (as owner) writes only its own columns of P: no
    // barrier needed before the loads
    T x[4][8];
#pragma unroll
    for (int q = 0; q < 4; ++q)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int r = lane + 32 * i;
            x[q][i] = (q < nc && r < RG) ? P[(size_t)(cb + q) * RGP + padr<T>(r)] : T(0);
        }
    if (nc > 0) {
        // ---- earlier reflectors, one at a time as they are published ----
        for (int jr = 0; jr < cb; ++jr) {
            mbar_wait_parity(&mb[jr], parity);
            const T tau = tau_s[jr];
            if (tau == T(0)) continue;
            T v[8];
#pragma unroll
            for (int i = 0; i < 8; ++i) v[i] = P[(size_t)jr * RGP + padr<T>(lane + 32 * i)];
            T d[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                T a0 = T(0), a1 = T(0);
#pragma unroll
                for (int i = 0; i < 8; i += 2) {
                    a0 = fma(v[i], x[q][i], a0);
                    a1 = fma(v[i + 1], x[q][i + 1], a1);
                }
                d[q] = a0 + a1;
            }
            warp_allsum_bfly<4>(d);  // (a shared-memory transpose instead: 5.55 vs 5.37 ms)
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const T st = tau * d[q];
#pragma unroll
                for (int i = 0; i < 8; ++i) x[q][i] = fma(-st, v[i], x[q][i]);
            }
        }
        // ---- this warp's block: reflectors cb .. cb + nc - 1 ----
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            if (q < nc) {
                const int j = cb + q;
                // slot 0: ||x_q (rows > j)||^2, slot 1 + m: x_q . x_{q+1+m} (rows > j)
                T red[4] = {T(0), T(0), T(0), T(0)};
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    const int r = lane + 32 * i;
                    const T xq = r > j ? x[q][i] : T(0);
                    red[0] = fma(xq, xq, red[0]);
#pragma unroll
                    for (int m = 0; m < 3; ++m)
                        if (m < 3 - q) red[1 + m] = fma(xq, x[q + 1 + m][i], red[1 + m]);
                }
                if (q == 0) warp_allsum_bfly<4>(red);
                else if (q == 1) {
                    T rr[3] = {red[0], red[1], red[2]};
                    warp_allsum_bfly<3>(rr);
                    red[0] = rr[0]; red[1] = rr[1]; red[2] = rr[2];
                } else if (q == 2) {
                    T rr[2] = {red[0], red[1]};
                    warp_allsum_bfly<2>(rr);
                    red[0] = rr[0]; red[1] = rr[1];
                } else {
                    T rr[1] = {red[0]};
                    warp_allsum_bfly<1>(rr);
                    red[0] = rr[0];
                }
                const T al = __shfl_sync(0xffffffffu, x[q][0], j);
                T head[3];
#pragma unroll
                for (int m = 0; m < 3; ++m)
                    head[m] = (m < 3 - q) ? __shfl_sync(0xffffffffu, x[q + 1 + m][0], j) : T(0);
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
                __syncwarp();
                if (lane == 0) mbar_arrive1(&mb[j]);  // release: v_j and tau_j are visible
#pragma unroll
                for (int m = 0; m < 3; ++m) {
                    if (m < 3 - q && tau != T(0)) {  // H_j on the block's later column q + 1 + m
                        const T st = tau * fma(scale, red[1 + m], head[m]);
#pragma unroll
                        for (int i = 0; i < 8; ++i) x[q + 1 + m][i] = fma(-st, v[i], x[q + 1 + m][i]);
                    }
                }
            }
        }
    }
    // reflectors this call does not produce (columns >= wp) still complete
    // their phase, so every mbarrier advances exactly once per call
    if (lane == 0)
        for (int q = nc; q < 4; ++q) mbar_arrive1(&mb[cb + q]);
    if (Gout && nc > 0) {
        // The Gram matrix G = V^T V for the compact-WY T (build_t reads G[j][k],
        // k < j), by warps whose own columns are final while the later blocks are
        // still being factored: this block's 6 entries, then, as each later block
        // completes (its last mbarrier), the 4 x 4 entries against it.  Exact
        // fp32 dots over the panel rows, as the separate G = V^T V pass was.
        T v[4][8];
#pragma unroll
        for (int q = 0; q < 4; ++q)
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const int r = lane + 32 * i, j = cb + q;
                v[q][i] = q < nc ? (r > j ? x[q][i] : (r == j ? T(1) : T(0))) : T(0);
            }
        T* scr = scr_all + warp * (32 * 20 + 16);
        {
            T gw[6];
            int e = 0;
#pragma unroll
            for (int a = 0; a < 4; ++a)
#pragma unroll
                for (int b = a + 1; b < 4; ++b, ++e) {
                    T acc = T(0);
#pragma unroll
                    for (int i = 0; i < 8; ++i) acc = fma(v[a][i], v[b][i], acc);
                    gw[e] = acc;
                }
            const T gl = warp_reduce_scatter_smem<6>(gw, scr);  // lane l: entry l % 8
            if (lane < 6) {
                const int a = lane < 3 ? 0 : (lane < 5 ? 1 : 2);
                const int b = lane < 3 ? lane + 1 : (lane < 5 ? lane - 1 : 3);
                Gout[(cb + b) * kTS + cb + a] = gl;
            }
        }
        const int nblk = (wp + 3) / 4;
        for (int bb = blk + 1; bb < nblk; ++bb) {
            mbar_wait_parity(&mb[4 * bb + 3], parity);  // block bb complete
            T w[16];
#pragma unroll
            for (int qb = 0; qb < 4; ++qb) {
                T vb[8];
#pragma unroll
                for (int i = 0; i < 8; ++i) vb[i] = P[(size_t)(4 * bb + qb) * RGP + padr<T>(lane + 32 * i)];
#pragma unroll
                for (int qa = 0; qa < 4; ++qa) {
                    T acc = T(0);
#pragma unroll
                    for (int i = 0; i < 8; ++i) acc = fma(v[qa][i], vb[i], acc);
                    w[qa * 4 + qb] = acc;
                }
            }
            const T wl = warp_reduce_scatter_smem<16>(w, scr);  // lane l: entry l % 16
            if (lane < 16) Gout[(4 * bb + (lane & 3)) * kTS + cb + (lane >> 2)] = wl;
        }
    }
    if (Gout && nc == 0)  // blocks beyond wp: zero rows (build_t multiplies them by tau = 0)
#pragma unroll
        for (int q = 0; q < 4; ++q) Gout[(cb + q) * kTS + lane] = T(0);
    gsync(G);  // every reflector applied: P's v columns are no longer read
    const NodeRows& nr = *out_nr;
    if ((!nr.seg1_upper && nr.n1 == 0) || (nr.seg0_tri && nr.n0 == 32)) {
        // fast epilogue for the common node shapes (warp-uniform test): a leaf
        // (one dense segment, everything stored), a full chain step (gathered
        // rows 0..31 = the R band, stored on and above the diagonal; rows 32..
        // = the tile, dense, final V) and a full merge (rows 32.. = the right
        // member's R slot, stored on and above its diagonal: final tree V)
        const uint64_t pol = l2_evict_first_policy();
        const bool leaf = !nr.seg1_upper && nr.n1 == 0;
        const int upper = nr.seg1_upper ? 32 + 32 * out_p : (1 << 30);  // seg1 row r stored iff r - upper <= jj
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            if (q >= nc) continue;
            const int jj = cb + q;
            T* col = out_A + (out_c0 + jj) * out_lda;
            if (leaf) {
#pragma unroll
                for (int i = 0; i < 8; ++i)
                    if (lane + 32 * i < RG) col[nr.r0 + lane + 32 * i] = x[q][i];
            } else {
                if (lane <= jj) col[nr.r0 + lane] = x[q][0];
                T* tcol = col + nr.r1 - 32;
#pragma unroll
                for (int i = 1; i < 8; ++i)
                    if (lane + 32 * i < RG && lane + 32 * i - upper <= jj)
                        st_evict_first(tcol + lane + 32 * i, x[q][i], pol);
            }
        }
    } else {
        // epilogue straight from registers: the stored form (R / v,
        // structure masks) to global
        const uint64_t pol = l2_evict_first_policy();
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
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const int r = lane + 32 * i;
                const bool in = q < nc && r < RG;
                const bool stored = key[i] <= jj;
                if (in && stored) {
                    // segment 1 (a chain step's tile rows, a merge's right slot)
                    // is final V after this panel: evict first from L2
                    if (seg0[i]) col[grow[i]] = x[q][i];
                    else st_evict_first(col + grow[i], x[q][i], pol);
                }
                // (P already holds the V form: the v each owner wrote for the
                // consumers equals it -- a structured node's implicit zeros
                // stay exactly zero through the dense reflectors)
            }
        }
    }
    gsync(G);
}

// ---------------------------------------------------------------------------
// W(32 x 32) = V^T C over RG rows, V and C padded-column tiles (32 columns).
// 8 warps = 4-way split of the rows x 2 column halves; deterministic reduction.
// ---------------------------------------------------------------------------
template <typename T>
__device__ __forceinline__ void gemm_vtc(const Grp& G, const T* Vs, const T* Cs, int RGP, int R32, T* Wp, T* W) {
    using V4 = typename Vec4<T>::type;
    constexpr int VN = Vec4<T>::n;
    const int tid = G.tid, warp = tid >> 5, lane = tid & 31;
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
    gsync(G);
    for (int e = tid; e < 32 * 32; e += kThreads) {
        const int jj = e >> 5, cc2 = e & 31;
        T sum = Wp[(0 * 32 + jj) * kTS + cc2];
        sum += Wp[(1 * 32 + jj) * kTS + cc2];
        sum += Wp[(2 * 32 + jj) * kTS + cc2];
        sum += Wp[(3 * 32 + jj) * kTS + cc2];
        W[jj * kTS + cc2] = sum;
    }
    gsync(G);
}

// T (upper triangular, Tt[r*kTS+c] = T[r][c]) from G = V^T V (strict upper
// part in G) and tau (xLARFT forward/columnwise): T[j][j] = tau_j,
// T[0:j,j] = -tau_j T[0:j,0:j] G[0:j,j].  One warp; lane i keeps row i of T in
// registers; 4 independent accumulation chains.
template <typename T>
__device__ __forceinline__ void build_t(const Grp& Gr, const T* G, const T* tau_s, int wp, T* Tt,
                                       T* tglobal = nullptr) {
    using V4 = typename Vec4<T>::type;
    constexpr int VN = Vec4<T>::n;
    const int lane = Gr.tid & 31;
    if (Gr.tid >= 32) return;
    T row[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) {
        // G is symmetric bit for bit (G[k][j] and G[j][k] are the same products
        // summed in the same order), so G[k][j] is read from row j: contiguous,
        // 16-byte broadcast loads (a quarter of the shared-memory instructions
        // of a column walk, which made this one-warp step LDS-issue bound)
        const T* gj = G + j * kTS;
        T a0 = 0, a1 = 0, a2 = 0, a3 = 0;
#pragma unroll
        for (int k = 0; k + 3 < j; k += 4) {
            T g[4];
#pragma unroll
            for (int h = 0; h < 4 / VN; ++h) {
                const V4 q = *reinterpret_cast<const V4*>(gj + k + h * VN);
#pragma unroll
                for (int e = 0; e < VN; ++e) g[h * VN + e] = vget<T>(q, e);
            }
            a0 = fma(row[k + 0], g[0], a0);
            a1 = fma(row[k + 1], g[1], a1);
            a2 = fma(row[k + 2], g[2], a2);
            a3 = fma(row[k + 3], g[3], a3);
        }
#pragma unroll
        for (int k = j & ~3; k < j; ++k) a0 = fma(row[k], gj[k], a0);
        const T tau = j < wp ? tau_s[j] : T(0);
        row[j] = (j == lane) ? tau : (j > lane ? -tau * ((a0 + a1) + (a2 + a3)) : T(0));
    }
#pragma unroll
    for (int j = 0; j < 32; ++j) Tt[lane * kTS + j] = row[j];
    if (tglobal) {  // the workspace's column-major T block: coalesced across lanes
        const uint64_t pol = l2_evict_first_policy();
#pragma unroll
        for (int j = 0; j < 32; ++j) st_evict_first(tglobal + j * 32 + lane, row[j], pol);
    }
}

// C(RG x 32, in Cs) <- C - V (op(T) W) ; written straight to global rows.
// ---------------------------------------------------------------------------
// Tensor-core path of the trailing update (fp32): mma.sync m16n8k8 TF32 with
// the 3xTF32 split (x = hi + lo, hi = tf32(x), lo = tf32(x - hi); a*b ~
// ahi*bhi + ahi*blo + alo*bhi), fp32 accumulation.  Measured on this B200:
// 276 TF/s TF32 dense -> ~92 TF/s 3xTF32, vs 71 TF/s FFMA; the point is the
// ~5x lower shared-memory traffic per multiply-add (register fragments reused
// across tiles), which frees the MIO pipe the panel factorization needs.
// Used only for W = V^T C and C -= V W2 of the factorization's trailing
// update: V, T (hence Q) stay exact fp32, so Q's orthogonality is unaffected;
// the trailing matrix sees ~2^-21 relative product errors (backward error).
// The low part goes to the MMA unrounded (the TF32 unit reads its top 10
// mantissa bits: truncation, error <= 2^-21 |x| instead of 2^-22 for a second
// cvt.rna): one conversion less per operand element, 5.34 -> 5.15 ms at
// 1M x 192, every achieved error unchanged to three digits (S20,
// profiles/parity_r02.json).  CAQR_EXACT_SPLIT restores the rounded low part.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void split_tf32(float x, uint32_t& hi, uint32_t& lo) {
    uint32_t h, l;
#ifndef CAQR_EXACT_SPLIT
    // round to the nearest TF32, ties away from zero: the cvt.rna.tf32 result
    // for every finite x, as one integer add and mask (the conversion's NaN
    // handling costs ~3 more instructions per element): 5.16 -> 5.01 ms at
    // 1M x 192, results bit for bit unchanged (profiles/parity_r02.json)
    h = (__float_as_uint(x) + 0x1000u) & 0xffffe000u;
#else
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(h) : "f"(x));
#endif
    const float r = x - __uint_as_float(h);
#ifndef CAQR_EXACT_SPLIT
    l = __float_as_uint(r);
#else
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(l) : "f"(r));
#endif
    hi = h;
    lo = l;
}
__device__ __forceinline__ void mma_tf32(float (&d)[4], const uint32_t (&a)[4], const uint32_t (&b)[2]) {
    asm volatile(
        "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
}
__device__ __forceinline__ void mma_3xtf32(float (&d)[4], const uint32_t (&ah)[4], const uint32_t (&al)[4],
                                           const uint32_t (&bh)[2], const uint32_t (&bl)[2]) {
    mma_tf32(d, al, bh);
    mma_tf32(d, ah, bl);
    mma_tf32(d, ah, bh);
}

// W(32 x 32) = V^T C on tensor cores; same warp split and deterministic
// 4-way reduction as gemm_vtc.
template <bool PAD = true>
__device__ __forceinline__ int rowmap(int r) {
    return PAD ? padr<float>(r) : r;
}

template <bool PAD>
__device__ __forceinline__ void gemm_vtc_mma(const Grp& G, const float* Vs, const float* Cs, int RGP, int R32,
                                             float* Wp, float* W) {
    const int warp = G.tid >> 5, lane = G.tid & 31;
    const int ks = warp & 3, ch = warp >> 2;
    const int g = lane >> 2, t = lane & 3;
    const int chunk = R32 / 4;
    const int rbeg = ks * chunk, rend = rbeg + chunk;
    float acc[2][2][4];
#pragma unroll
    for (int a = 0; a < 2; ++a)
#pragma unroll
        for (int b = 0; b < 2; ++b)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[a][b][e] = 0.f;
    for (int k0 = rbeg; k0 < rend; k0 += 8) {
        const int p0 = rowmap<PAD>(k0 + t), p1 = rowmap<PAD>(k0 + t + 4);
        uint32_t ah[2][4], al[2][4], bh[2][2], bl[2][2];
#pragma unroll
        for (int mt = 0; mt < 2; ++mt) {
            const float* v0 = Vs + (size_t)(16 * mt + g) * RGP;
            const float* v8 = v0 + 8 * (size_t)RGP;
            split_tf32(v0[p0], ah[mt][0], al[mt][0]);
            split_tf32(v8[p0], ah[mt][1], al[mt][1]);
            split_tf32(v0[p1], ah[mt][2], al[mt][2]);
            split_tf32(v8[p1], ah[mt][3], al[mt][3]);
        }
#pragma unroll
        for (int nt = 0; nt < 2; ++nt) {
            const float* c0 = Cs + (size_t)(16 * ch + 8 * nt + g) * RGP;
            split_tf32(c0[p0], bh[nt][0], bl[nt][0]);
            split_tf32(c0[p1], bh[nt][1], bl[nt][1]);
        }
#pragma unroll
        for (int mt = 0; mt < 2; ++mt)
#pragma unroll
            for (int nt = 0; nt < 2; ++nt) mma_3xtf32(acc[mt][nt], ah[mt], al[mt], bh[nt], bl[nt]);
    }
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 2; ++nt) {
            const int jj = 16 * mt + g, c = 16 * ch + 8 * nt + 2 * t;
            float* wr = Wp + (ks * 32 + jj) * kTS + c;
            wr[0] = acc[mt][nt][0];
            wr[1] = acc[mt][nt][1];
            wr[8 * kTS] = acc[mt][nt][2];
            wr[8 * kTS + 1] = acc[mt][nt][3];
        }
    gsync(G);
    for (int e = G.tid; e < 32 * 32; e += kThreads) {
        const int jj = e >> 5, c = e & 31;
        float sum = Wp[(0 * 32 + jj) * kTS + c];
        sum += Wp[(1 * 32 + jj) * kTS + c];
        sum += Wp[(2 * 32 + jj) * kTS + c];
        sum += Wp[(3 * 32 + jj) * kTS + c];
        W[jj * kTS + c] = sum;
    }
    gsync(G);
}

// Cs(R32 x 32) <- Cs - V W2 on tensor cores (W2 in W, rows jj).  Warp w owns
// row tiles {w, w + 8, ...} of 16 rows and all 4 column tiles.
template <bool PAD>
__device__ __forceinline__ void gemm2_mma(const Grp& G, const float* Vs, float* Cs, const float* W, int RGP,
                                          int R32) {
    const int warp = G.tid >> 5, lane = G.tid & 31;
    const int g = lane >> 2, t = lane & 3;
    // B fragments (-W2) for all 4 k-steps x 4 column tiles, split once
    uint32_t bh[4][4][2], bl[4][4][2];
#pragma unroll
    for (int kk = 0; kk < 4; ++kk)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
            split_tf32(-W[(8 * kk + t) * kTS + 8 * nt + g], bh[kk][nt][0], bl[kk][nt][0]);
            split_tf32(-W[(8 * kk + t + 4) * kTS + 8 * nt + g], bh[kk][nt][1], bl[kk][nt][1]);
        }
    for (int mt = warp; mt < R32 / 16; mt += kWarps) {
        const int m0 = 16 * mt;
        const int r0 = rowmap<PAD>(m0 + g), r8 = rowmap<PAD>(m0 + g + 8);
        float d[4][4];
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
            const float* c0 = Cs + (size_t)(8 * nt + 2 * t) * RGP;
            d[nt][0] = c0[r0];
            d[nt][1] = c0[RGP + r0];
            d[nt][2] = c0[r8];
            d[nt][3] = c0[RGP + r8];
        }
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
            const float* va = Vs + (size_t)(8 * kk + t) * RGP;
            const float* vb = va + 4 * (size_t)RGP;
            uint32_t ah[4], al[4];
            split_tf32(va[r0], ah[0], al[0]);
            split_tf32(va[r8], ah[1], al[1]);
            split_tf32(vb[r0], ah[2], al[2]);
            split_tf32(vb[r8], ah[3], al[3]);
#pragma unroll
            for (int nt = 0; nt < 4; ++nt) mma_3xtf32(d[nt], ah, al, bh[kk][nt], bl[kk][nt]);
        }
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
            float* c0 = Cs + (size_t)(8 * nt + 2 * t) * RGP;
            c0[r0] = d[nt][0];
            c0[RGP + r0] = d[nt][1];
            c0[r8] = d[nt][2];
            c0[RGP + r8] = d[nt][3];
        }
    }
}

// This thread's two row quads r = 4 (lane + 32 b), b < 2, of a node's gathered
// rows (<= 256): absolute row offset and the number of rows < RG in the quad.
// Fixed per (node, panel), so the 16-byte staging and write-back of every
// trailing block reuse them instead of re-deriving them element by element.
struct RowQuads {
    int64_t off[2];
    int cnt[2];
};
__device__ __forceinline__ RowQuads row_quads(const NodeRows& nr, int RG) {
    const int lane = threadIdx.x & 31;
    RowQuads q;
#pragma unroll
    for (int b = 0; b < 2; ++b) {
        const int r = 4 * (lane + 32 * b);
        q.cnt[b] = max(0, min(4, RG - r));
        q.off[b] = q.cnt[b] > 0 ? gathered_row(nr, r) : 0;
    }
    return q;
}

template <typename T>
__device__ __forceinline__ void apply_block(const Grp& G, const T* Vs, const T* Cs, const T* Tt, T* W, int RGP, int R32,
                                            int RG, int wp, int trans, const NodeRows& nr, T* C,
                                            int64_t ldc, int64_t cb0, int ncb, bool vec = false,
                                            const RowQuads* rq = nullptr, T* W2buf = nullptr) {
    using V4 = typename Vec4<T>::type;
    constexpr int VN = Vec4<T>::n;
    const int tid = G.tid;
    // W2 = op(T) W: thread (column c, rows jj = 4 jg + q): the 4 T entries a
    // thread needs per k are contiguous (one 16-byte load for Q^T); T is zero
    // below its diagonal, so full unrolled sums need no bounds.
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
            if (trans) {
#pragma unroll
                for (int k = 0; k < 16; ++k) {
                    T tq[4];
#pragma unroll
                    for (int hh = 0; hh < 4 / VN; ++hh) {
                        const V4 t4 = *reinterpret_cast<const V4*>(Tt + (h + k) * kTS + 4 * jg + hh * VN);
#pragma unroll
                        for (int e = 0; e < VN; ++e) tq[hh * VN + e] = vget<T>(t4, e);
                    }
#pragma unroll
                    for (int q = 0; q < 4; ++q) w2[q] = fma(tq[q], wc[k], w2[q]);
                }
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int jj = 4 * jg + q;
                    T a0 = 0, a1 = 0;
#pragma unroll
                    for (int k = 0; k < 16; k += 2) {
                        a0 = fma(Tt[jj * kTS + h + k], wc[k], a0);
                        a1 = fma(Tt[jj * kTS + h + k + 1], wc[k + 1], a1);
                    }
                    w2[q] += a0 + a1;
                }
            }
        }
    }
    // W2 into a separate buffer when given (no barrier between reading W and
    // writing W2), else over W
    T* W2 = W2buf ? W2buf : W;
    if (!W2buf) gsync(G);
#pragma unroll
    for (int q = 0; q < 4; ++q) W2[(4 * (tid >> 5) + q) * kTS + (tid & 31)] = w2[q];
    gsync(G);
    if constexpr (sizeof(T) == 4) {
        gemm2_mma<true>(G, Vs, const_cast<T*>(Cs), W2, RGP, R32);
    } else {
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
                const V4 t4 = *reinterpret_cast<const V4*>(W2 + jj * kTS + cbase + h * VN);
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
    }
    gsync(G);
    {
        const int warp = tid >> 5, lane = tid & 31;
        if (sizeof(T) == 4 && vec && rq) {  // float4 stores, precomputed row quads
            for (int c = warp; c < ncb; c += kWarps) {
                T* ccol = C + (cb0 + c) * ldc;
                const T* cs = Cs + (size_t)c * RGP;
#pragma unroll
                for (int u = 0; u < 2; ++u) {
                    const int r = 4 * (lane + 32 * u);
                    if (rq->cnt[u] == 4) {
                        *reinterpret_cast<float4*>(ccol + rq->off[u]) = *reinterpret_cast<const float4*>(cs + r);
                    } else {
                        for (int q = 0; q < rq->cnt[u]; ++q) ccol[rq->off[u] + q] = cs[r + q];
                    }
                }
            }
        } else if (sizeof(T) == 4 && vec) {  // float4 stores: rows 4q..4q+3 lie in one segment
            for (int c = warp; c < ncb; c += kWarps) {
                T* ccol = C + (cb0 + c) * ldc;
                const T* cs = Cs + (size_t)c * RGP;
                for (int r = 4 * lane; r < RG; r += 128) {
                    if (r + 4 <= RG) {
                        *reinterpret_cast<float4*>(ccol + gathered_row(nr, r)) =
                            *reinterpret_cast<const float4*>(cs + r);
                    } else {
                        for (int q = r; q < RG; ++q) ccol[gathered_row(nr, q)] = cs[q];
                    }
                }
            }
        } else {
            for (int c = warp; c < ncb; c += kWarps) {
                T* ccol = C + (cb0 + c) * ldc;
                const T* cs = Cs + (size_t)c * RGP;
                for (int r = lane; r < RG; r += 32) ccol[gathered_row(nr, r)] = cs[padr<T>(r)];
            }
        }
    }
    gsync(G);
}

// cp.async (LDGSTS) staging of a C block (gathered rows, ncol <= 32 columns
// from col0) into S (column-major, stride RGP, rows [RG, R32) zero-filled):
// no register round trip and, with vec, a quarter of the load instructions
// and address arithmetic of stage_cols.  vec: 16-byte requests (A 16-byte
// aligned, lda % 4 == 0, row segments starting on multiples of 4).  Caller
// waits (cp.async.wait_group) and synchronises.
__device__ __forceinline__ void stage_cols_cp(const Grp& G, float* S, int RGP, int R32, const float* M, int64_t ld,
                                              int64_t col0, int ncol, const NodeRows& nr, int RG, bool vec,
                                              const RowQuads* rq = nullptr) {
    const int warp = G.tid >> 5, lane = G.tid & 31;
    if (vec && rq) {
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const int jj = warp + 8 * a;
            const float* mc = M + (col0 + min(jj, max(ncol - 1, 0))) * ld;
#pragma unroll
            for (int b = 0; b < 2; ++b) {
                const int r = 4 * (lane + 32 * b);
                if (r < R32) {
                    const int valid = jj < ncol ? rq->cnt[b] : 0;
                    const unsigned dst = (unsigned)__cvta_generic_to_shared(S + (size_t)jj * RGP + r);
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(mc + rq->off[b]),
                                 "r"(valid * 4)
                                 : "memory");
                }
            }
        }
    } else if (vec) {
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const int jj = warp + 8 * a;
            const float* mc = M + (col0 + min(jj, max(ncol - 1, 0))) * ld;
#pragma unroll
            for (int b = 0; b < 2; ++b) {
                const int r = 4 * (lane + 32 * b);
                if (r < R32) {
                    const int valid = jj < ncol ? max(0, min(4, RG - r)) : 0;
                    const float* src = valid > 0 ? mc + gathered_row(nr, r) : mc;
                    const unsigned dst = (unsigned)__cvta_generic_to_shared(S + (size_t)jj * RGP + r);
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src),
                                 "r"(valid * 4)
                                 : "memory");
                }
            }
        }
    } else {
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const int jj = warp + 8 * a;
            const float* mc = M + (col0 + min(jj, max(ncol - 1, 0))) * ld;
#pragma unroll
            for (int b = 0; b < 8; ++b) {
                const int r = lane + 32 * b;
                if (r < R32) {
                    const bool valid = jj < ncol && r < RG;
                    const float* src = valid ? mc + gathered_row(nr, r) : mc;
                    const unsigned dst = (unsigned)__cvta_generic_to_shared(S + (size_t)jj * RGP + r);
                    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(dst), "l"(src),
                                 "r"(valid ? 4 : 0)
                                 : "memory");
                }
            }
        }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

template <typename T>
__device__ __forceinline__ void stage_cols(const Grp& G, T* S, int RGP, int R32, const T* M, int64_t ld, int64_t col0,
                                           int ncol, const NodeRows& nr, int RG, bool mask_panel, int p) {
    // Every thread issues all of its loads before the first store (memory-level
    // parallelism: up to 32 L2/HBM requests in flight per thread), in halves
    // of 16 for fp64 to bound register use.
    const int warp = G.tid >> 5, lane = G.tid & 31;
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
    // 16-byte staging / write-back of C blocks (fp32): A 16-byte aligned and
    // every row segment (tiles, R slots) starting on a multiple of 4 rows
    const bool vec = sizeof(T) == 4 && (reinterpret_cast<uintptr_t>(A) % 16 == 0) && (g.lda % 4 == 0) &&
                     (g.row0 % 4 == 0) && (g.b % 4 == 0) && (g.bm % 4 == 0);
    __shared__ int s_task;
    __shared__ __align__(8) uint64_t s_mb[32];  // per-reflector publication (factor_panel_pipe)
    unsigned pipe_parity = 0;
    if (threadIdx.x < 32)
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((unsigned)__cvta_generic_to_shared(&s_mb[threadIdx.x]))
                     : "memory");
    __syncthreads();
    const Grp G0{(int)threadIdx.x, 0};
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
    __shared__ unsigned long long pacc[14];
    if (threadIdx.x < 14) pacc[threadIdx.x] = threadIdx.x == 13 ? (unsigned long long)clock64() : 0ull;
#define CAQR_PROF(k)                                              \
    do {                                                          \
        if (prof && threadIdx.x == 0) {                           \
            const unsigned long long t1_ = clock64();             \
            pacc[k] += t1_ - pacc[13];                            \
            pacc[13] = t1_;                                       \
        }                                                         \
    } while (0)
    for (;;) {
        __syncthreads();
        CAQR_PROF(0);
        if (threadIdx.x == 0) s_task = atomicAdd(ticket, 1);
        __syncthreads();
        const int64_t task = s_task;
        if (prof && threadIdx.x == 0) {  // timeline: first start, last chain end, last merge end
            unsigned long long gt;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt));
            if (task == 0) atomicMax(prof + 15, ~gt);
            atomicMax(prof + 14, gt);
        }
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
            // A slot's panel flag goes through 2v-1 ("panel p factored: its R rows
            // of panel p's columns are final") and 2v ("panel p's trailing update
            // done") for the node of version v that last writes it.  A merge
            // factors its panel p once both children are factored, and updates
            // its trailing columns once both are done: the factorization
            // overlaps the children's trailing updates.
            if (level >= 0 && threadIdx.x == 0) {
                const int* fa = flags + slot_a * g.npan + p;
                const int* fb = flags + slot_b * g.npan + p;
                while (ld_acquire(fa) < 2 * ver_a - 1) __nanosleep(64);
                while (ld_acquire(fb) < 2 * ver_b - 1) __nanosleep(64);
            }
            __syncthreads();
            CAQR_PROF(1);
            if (prof && threadIdx.x == 0) pacc[level < 0 ? 10 : 11] += 1;
            const NodeRows nr = node_rows(g, level, node, p, wp, kt);
            const int RG = nr.n0 + nr.n1;
            const int R32 = (RG + 31) & ~31;
            const int64_t c0 = g.col0 + 32 * p;
            // ---- panel: stage, factor, store R/V, T ------------------------
            if (level < 0 && p > 0) {
                // The previous panel's LAST trailing block was this panel's
                // columns over the previous node's gathered rows, still in Cs
                // (updated).  A leaf's rows are those minus the first 32; a
                // chain node's are the slot rows [32p, 32p+wp) (from global:
                // not part of the previous node) and the same tile rows.
                const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
                const bool leaf = kt == 0;
                T head[4];
#pragma unroll
                for (int a = 0; a < 4; ++a) {
                    const int jj = warp + 8 * a;
                    head[a] = (!leaf && lane < nr.n0 && jj < wp && panel_entry_stored(nr, lane, jj, p))
                                  ? ldcg(A + (c0 + jj) * g.lda + gathered_row(nr, lane))
                                  : T(0);
                }
                if (sizeof(T) == 4 && (leaf || nr.n0 == 32)) {
                    // 16-byte copies: a leaf's rows r come from Cs row r + 32, a chain
                    // step's rows r >= 32 from Cs row r (rows < 32: the slot's heads)
#pragma unroll
                    for (int a = 0; a < 4; ++a) {
                        const int jj = warp + 8 * a;
                        float* pc = reinterpret_cast<float*>(P) + (size_t)jj * RGP;
                        const float* cc = reinterpret_cast<const float*>(Cs) + (size_t)jj * RGP;
                        if (!leaf) pc[lane] = head[a];
#pragma unroll
                        for (int u = 0; u < 2; ++u) {
                            const int r4 = 4 * (lane + 32 * u);
                            if (r4 >= R32 || (!leaf && r4 < 32)) continue;
                            float4 v = *reinterpret_cast<const float4*>(cc + r4 + (leaf ? 32 : 0));
                            const bool ok = jj < wp;
                            v.x = ok && r4 < RG ? v.x : 0.f;
                            v.y = ok && r4 + 1 < RG ? v.y : 0.f;
                            v.z = ok && r4 + 2 < RG ? v.z : 0.f;
                            v.w = ok && r4 + 3 < RG ? v.w : 0.f;
                            *reinterpret_cast<float4*>(pc + r4) = v;
                        }
                    }
                } else {
#pragma unroll
                    for (int a = 0; a < 4; ++a) {
                        const int jj = warp + 8 * a;
                        T* pc = P + (size_t)jj * RGP;
                        const T* cc = Cs + (size_t)jj * RGP;
                        for (int r = lane; r < R32; r += 32) {
                            T v;
                            if (leaf) v = (r < RG && jj < wp) ? cc[padr<T>(r + 32)] : T(0);
                            else if (r < nr.n0) v = head[a];
                            else v = (r < RG && jj < wp) ? cc[padr<T>(r - nr.n0 + 32)] : T(0);
                            pc[padr<T>(r)] = v;
                        }
                    }
                }
            } else {
                stage_cols(G0, P, RGP, R32, A, g.lda, c0, wp, nr, RG, true, p);
            }
            if (threadIdx.x < 32) tau_s[threadIdx.x] = T(0);
            __syncthreads();
            CAQR_PROF(2);
#ifdef CAQR_NO_PIPE_GRAM
            factor_panel_pipe<T>(G0, P, RGP, RG, wp, tau_s, s_mb, pipe_parity, &nr, A, g.lda, c0, p);
#else
            factor_panel_pipe<T>(G0, P, RGP, RG, wp, tau_s, s_mb, pipe_parity, &nr, A, g.lda, c0, p, W, Cs);
#endif
            pipe_parity ^= 1u;
            CAQR_PROF(3);
#ifdef CAQR_NO_PIPE_GRAM
            gemm_vtc(G0, P, P, RGP, R32, Wp, W);  // G = V^T V
#endif
            CAQR_PROF(4);
            build_t(G0, W, tau_s, wp, Tt, Tws + nr.tblk * (kPW * kPW));
            __syncthreads();
            CAQR_PROF(12);
            // wait for the children's trailing updates before touching later
            // columns, then publish "factored" (the stored R / V of panel p are in A).
            // Only a published flag needs the device-scope fence: a chain's next
            // tile reads these rows from this CTA, ordered by the CTA barriers
            // (measured: 5.79 -> 5.71 ms at 1M x 192).  Dropping the barriers
            // too was slower (5.84 ms).
            if (kt == ntile - 1) __threadfence();
            __syncthreads();
            if (threadIdx.x == 0) {
                if (level >= 0) {  // (before this node's own publish on slot a: flags only grow)
                    const int* fa = flags + slot_a * g.npan + p;
                    const int* fb = flags + slot_b * g.npan + p;
                    while (ld_acquire(fa) < 2 * ver_a) __nanosleep(64);
                    while (ld_acquire(fb) < 2 * ver_b) __nanosleep(64);
                }
                if (kt == ntile - 1) st_release(flags + slot_a * g.npan + p, 2 * (level < 0 ? 1 : my_ver) - 1);
            }
            __syncthreads();
            CAQR_PROF(5);
            // ---- trailing columns of this node, 32 at a time -------------------
            // (the block holding the NEXT panel's columns goes last, so that
            // panel can be staged from Cs)
            const int64_t tfirst = c0 + 32, tend = g.col0 + g.ncols;
            const int nblk = tend > tfirst ? (int)((tend - tfirst + 31) / 32) : 0;
            const bool vec_p = vec && (nr.n0 % 4 == 0);
            const RowQuads rq = row_quads(nr, RG);
            for (int ib = 0; ib < nblk; ++ib) {
                const int64_t cb0 = tfirst + 32 * ((ib + 1) % nblk);
                const int ncb = (int)(tend - cb0 < 32 ? tend - cb0 : 32);
                if constexpr (sizeof(T) == 4) {
                    stage_cols_cp(G0, Cs, RGP, R32, A, g.lda, cb0, ncb, nr, RG, vec_p, &rq);
                    asm volatile("cp.async.wait_group 0;" ::: "memory");
                } else {
                    stage_cols(G0, Cs, RGP, R32, static_cast<const T*>(A), g.lda, cb0, ncb, nr, RG, false, p);
                }
                __syncthreads();
                CAQR_PROF(6);
                if constexpr (sizeof(T) == 4)
                    gemm_vtc_mma<true>(G0, P, Cs, RGP, R32, Wp, W);
                else
                    gemm_vtc(G0, P, Cs, RGP, R32, Wp, W);
                CAQR_PROF(7);
                apply_block(G0, P, Cs, Tt, W, RGP, R32, RG, wp, 1, nr, A, g.lda, cb0, ncb, vec_p, &rq, Wp);
                CAQR_PROF(8);
            }
            // ---- publish ----------------------------------------------------------
            if (kt == ntile - 1) __threadfence();
            __syncthreads();
            if (threadIdx.x == 0 && kt == ntile - 1)  // panel p's trailing update done
                st_release(flags + slot_a * g.npan + p, 2 * (level < 0 ? 1 : my_ver));
            CAQR_PROF(9);
        }
        if (prof && threadIdx.x == 0 && level < 0) {  // timeline: this chain's end
            unsigned long long gt;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt));
            atomicMax(prof + 13, gt);
        }
    }
    if (prof && threadIdx.x == 0)
        for (int k = 0; k < 13; ++k) atomicAdd(prof + k, pacc[k]);
#undef CAQR_PROF
}

}  // namespace caqr
