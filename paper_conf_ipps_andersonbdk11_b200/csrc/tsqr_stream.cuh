// tsqr_stream.cuh -- streaming TSQR of a skinny panel (n <= 16): one WARP per
// chain, the chain's R resident in shared memory, tiles double-buffered by
// cp.async, each merge of the binary tree done by the second of its two
// children to arrive (warps inside a CTA, then CTAs).
//
// For the s-step Krylov shape ("millions of rows by less than ten
// columns") the factorization is a stream of A through HBM: read each tile
// once, write its Householder vectors once.  The plan and the implicit-Q
// representation are the block kernels' (node_rows: chains of K tiles, P:L339-341
// "any tree shape", then a binary tree over the chain R's), so
// apply_qt / form_q replay it unchanged.  Per warp:
//   * tile kt+1 is in flight (cp.async.cg, 16 B per lane per request when A is
//     16-byte aligned) while tile kt is factored from registers;
//   * the first tile is a leaf Householder QR ("factor"); every
//     later one a structured QR of [R; tile] whose reflector heads sit in R
//     (v_j = [e_j; y_j]), so R never leaves shared memory inside the chain;
//   * per reflector ONE n-value warp all-reduce gives the squared norm, the dot
//     products with the later columns (matvec of P:L704-711 on the unscaled
//     column) and the Gram entries of the compact-WY T;
//   * then the chains' R's are merged up the binary tree ("factor_tree",
//     P:L658-663): inside the CTA level by level, across CTAs by whichever
//     CTA arrives SECOND at a pair (arrival counter) -- no one spins on a flag.
#pragma once
#include "tsqr_fused.cuh"
#include "umma.cuh"

namespace caqr {

__device__ __forceinline__ int64_t min64(int64_t a, int64_t b) { return a < b ? a : b; }

// All N values summed over the warp; every lane gets all N totals.  Halving
// butterfly (N/2 + N/4 + ... shuffles instead of 5 N), then the distinct
// totals are broadcast through the warp's scratch.
template <int N, typename T>
__device__ __forceinline__ void warp_allreduce(T (&v)[N], T* scr) {
    static_assert(N >= 1 && N <= 32 && (N & (N - 1)) == 0, "N: power of two <= 32");
    const int lane = threadIdx.x & 31;
    int idx = 0;
#pragma unroll
    for (int cnt = N, o = 16; cnt > 1; cnt >>= 1, o >>= 1) {
        const bool up = (lane & o) != 0;
#pragma unroll
        for (int i = 0; i < cnt / 2; ++i) {
            const T keep = up ? v[i + cnt / 2] : v[i];
            const T send = up ? v[i] : v[i + cnt / 2];
            v[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
        }
        idx += up ? cnt / 2 : 0;
    }
    constexpr int kDone = 32 / N;  // lanes [0, kDone) of each group hold one value index
#pragma unroll
    for (int o = kDone / 2; o >= 1; o >>= 1) v[0] += __shfl_xor_sync(0xffffffffu, v[0], o);
    __syncwarp();
    if ((lane & (kDone - 1)) == 0) scr[idx] = v[0];
    __syncwarp();
#pragma unroll
    for (int i = 0; i < N; ++i) v[i] = scr[i];
    __syncwarp();
}

// Householder scalars of one reflector (xLARFG, reading S1):
// alpha = head, sg = squared tail norm.  tau = (beta-alpha)/beta,
// scale = 1/(alpha-beta), beta = -copysign(sqrt(alpha^2 + sg), alpha);
// sg == 0 (or no row) -> H = I.
template <typename T>
__device__ __forceinline__ void householder_scalars(T al, T sg, bool live, T& tau, T& beta, T& scale) {
    tau = T(0);
    beta = al;
    scale = T(1);
    if (live && sg != T(0)) {
        const T ss = fma(al, al, sg);
        const T aa = fabs(al);
        T rmu, mu;
        rsqrt_refined(ss, rmu, mu);
        beta = -copysign(mu, al);
        tau = fma(aa, rmu, T(1));
        scale = copysign(rcp_refined(aa + mu), al);
    }
}

// Per-warp shared state.
// NBUF = 2: double-buffered tile; NBUF = 1: one buffer, refilled as soon as
// the warp has the current tile in registers (halves the shared memory, so
// 16 warps of 256-row tiles fit per SM).
template <typename T, int NC, int B, int NBUF = 2>
struct alignas(16) StreamWarp {
    T buf[NBUF][NC][B];  // tile buffer(s) (column-major, B rows)
    uint64_t mbar[2];  // bulk-copy completion, one per buffer
    T R[NC][NC + 1];   // chain / subtree R, R[j][k] (upper)
    T G[NC][NC + 1];   // Gram entries G[a][j] = v_a^T v_j (a < j)
    T Rs[NC][NC + 1];  // a sibling CTA's R (cross-CTA merges)
    T tau[NC];
    T red[32];         // all-reduce scratch
};

// T (compact WY, xLARFT forward/columnwise) from tau and the Gram entries
// G[a*ldg + j] = v_a^T v_j (a < j); column k of a group (k < NC, on) writes
// row k into the 32x32 column-major slot tb (wp x wp used).
template <typename T, int NC>
__device__ __forceinline__ void stream_write_t(bool on, int k, const T* G, int ldg, const T* tau, int wp, T* tb,
                                               int ldt = kPW) {
    if (on && k < wp) {
        T row[NC];
#pragma unroll
        for (int j = 0; j < NC; ++j) {
            T acc = T(0);
#pragma unroll
            for (int q = 0; q < j; ++q) acc = fma(row[q], G[q * ldg + j], acc);  // row[q] == 0 for q < k
            row[j] = (j == k) ? tau[j] : (j > k ? -tau[j] * acc : T(0));
        }
#pragma unroll
        for (int j = 0; j < NC; ++j)
            if (j < wp) tb[j * ldt + k] = row[j];
    }
}

// cp.async of tile t (h rows, columns [c0, c0 + wp)) into buf (B rows x NC);
// rows >= h and columns >= wp read as zeros.
template <typename T, int NC, int B, bool VEC>
__device__ __forceinline__ void stream_issue_tile(const Geom& g, const T* A, int64_t t, T (*buf)[B]) {
    const int lane = threadIdx.x & 31;
    const int64_t s = g.row0 + t * g.b;
    const int h = (int)min64(g.b, g.mrows - t * g.b);
    const int wp = g.ncols;
    if constexpr (VEC) {
        constexpr int E = 16 / sizeof(T);  // elements per 16-byte request
#pragma unroll
        for (int c = 0; c < NC; ++c) {
#pragma unroll
            for (int u = 0; u < B / (32 * E); ++u) {
                const int r = E * (lane + 32 * u);
                const int valid = c < wp ? max(0, min(E, h - r)) : 0;
                const T* src = A + (g.col0 + min(c, wp - 1)) * g.lda + s + (valid > 0 ? r : 0);
                const unsigned dst = (unsigned)__cvta_generic_to_shared(&buf[c][r]);
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src),
                             "r"(valid * (int)sizeof(T))
                             : "memory");
            }
        }
    } else {
#pragma unroll
        for (int c = 0; c < NC; ++c) {
#pragma unroll
            for (int u = 0; u < B / 32; ++u) {
                const int r = lane + 32 * u;
                const bool valid = c < wp && r < h;
                const T* src = A + (g.col0 + min(c, wp - 1)) * g.lda + s + (valid ? r : 0);
                const unsigned dst = (unsigned)__cvta_generic_to_shared(&buf[c][r]);
                asm volatile("cp.async.ca.shared.global [%0], [%1], %2, %3;" ::"r"(dst), "l"(src),
                             "n"((int)sizeof(T)), "r"(valid ? (int)sizeof(T) : 0)
                             : "memory");
            }
        }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

// A full tile (B rows, 16-byte aligned columns) by the bulk-copy engine:
// lane 0 posts the byte count on the buffer's mbarrier and issues one
// column-sized copy per panel column (columns >= wp of the buffer stay zero).
template <typename T, int NC, int B>
__device__ __forceinline__ void stream_issue_bulk(const Geom& g, const T* A, int64_t t, T (*buf)[B],
                                                  uint64_t* mbar) {
    if ((threadIdx.x & 31) == 0) {
        const int wp = g.ncols;
        constexpr unsigned kBytes = B * sizeof(T);
        const unsigned mb = umma::smem_u32(mbar);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(kBytes * wp)
                     : "memory");
        const T* src = A + g.col0 * g.lda + g.row0 + t * g.b;
        for (int c = 0; c < wp; ++c, src += g.lda)
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                    umma::smem_u32(&buf[c][0])),
                "l"(src), "r"(kBytes), "r"(mb)
                : "memory");
    }
}

// Register layout of a tile: x[c][i] = row 128 (i / 4) + 4 lane + i % 4 of
// column c, so a lane moves 16-byte pieces (LDS.128 from the tile buffer,
// STG.128 of V).  Rows < 16 (R's rows) sit in lanes 0..3, i < 4.
__device__ __forceinline__ int stream_row(int lane, int i) { return 128 * (i >> 2) + 4 * lane + (i & 3); }

// Leaf (kt == 0) or chain step (kt > 0) on the registers x[c][i] (row
// stream_row(lane, i) of column c).  Leaf: R ends in rows < NC of x (and is copied to
// W.R); chain step: reflector heads in W.R, x becomes the dense V.
template <typename T, int NC, int RPL, bool LEAF, int B, int NBUF>
__device__ __forceinline__ void stream_tile_qr(T (&x)[NC][RPL], StreamWarp<T, NC, B, NBUF>& W, int h) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int j = 0; j < NC; ++j) {
        // slot 0: ||x_j||^2 ; slot 1+m (m < NC-1-j): x_j . x_{j+1+m} ; then x_a . x_j (a < j)
        T red[NC];
#pragma unroll
        for (int q = 0; q < NC; ++q) red[q] = T(0);
#pragma unroll
        for (int i = 0; i < RPL; ++i) {
            const T xj = (LEAF && i < 4 && 4 * lane + i <= j) ? T(0) : x[j][i];
            red[0] = fma(xj, xj, red[0]);
#pragma unroll
            for (int q = 1; q < NC; ++q) {
                const int k = q < NC - j ? j + q : q - (NC - j);  // later column, else earlier a
                red[q] = fma(xj, x[k][i], red[q]);
            }
        }
        // heads: leaf -- row j of every column (alpha, the later columns' heads,
        // v_a[j] for a < j); chain step -- row j of R.  Read before the
        // all-reduce (its __syncwarp orders them before lane 0 rewrites row j).
        T hd[NC];
#pragma unroll
        for (int k = 0; k < NC; ++k) {
            if constexpr (LEAF)
                hd[k] = __shfl_sync(0xffffffffu, x[k][j & 3], j >> 2);
            else
                hd[k] = k >= j ? W.R[j][k] : T(0);
        }
        warp_allreduce<NC>(red, W.red);
        const T al = hd[j];
        T tau, beta, scale;
        householder_scalars(al, red[0], !LEAF || j < h, tau, beta, scale);
        // later columns: s_k = head_k + scale * (x_j . x_k); x_k -= tau s_k v_j
#pragma unroll
        for (int q = 1; q < NC; ++q) {
            if (q < NC - j) {
                const int k = j + q;
                const T head = hd[k];
                const T sk = fma(scale, red[q], head);
                const T f = tau * sk;
                const T fs = f * scale;
#pragma unroll
                for (int i = 0; i < RPL; ++i) {
                    if (LEAF && i < 4) {  // rows above the head keep, the head row takes -f
                        const int r = 4 * lane + i;
                        x[k][i] = r < j ? x[k][i] : (r == j ? x[k][i] - f : fma(-fs, x[j][i], x[k][i]));
                    } else {
                        x[k][i] = fma(-fs, x[j][i], x[k][i]);
                    }
                }
                if (!LEAF && lane == 0) W.R[j][k] = head - f;
            } else if (lane == 0) {  // Gram entry (a, j), a < j
                const int a = q - (NC - j);
                W.G[a][j] = LEAF ? fma(scale, red[q], hd[a]) : scale * red[q];
            }
        }
#pragma unroll
        for (int i = 0; i < RPL; ++i) {
            if (LEAF && i < 4) {
                const int r = 4 * lane + i;
                x[j][i] = r < j ? x[j][i] : (r == j ? beta : x[j][i] * scale);
            } else {
                x[j][i] *= scale;
            }
        }
        if (lane == 0) {
            W.tau[j] = tau;
            if (!LEAF) W.R[j][j] = beta;
        }
        __syncwarp();
    }
    if constexpr (LEAF) {  // R = rows < NC of the tile (upper part)
#pragma unroll
        for (int e = 0; e < 4; ++e) {
            const int r = 4 * lane + e;
            if (r < NC)
#pragma unroll
                for (int k = 0; k < NC; ++k) W.R[r][k] = k >= r ? x[k][e] : T(0);
        }
        __syncwarp();
    }
}

// Householder scalars as householder_scalars (sg == 0 -> H = I), computed
// branch-free so that every lane of a warp can evaluate them redundantly.
template <typename T>
__device__ __forceinline__ void householder_scalars_nb(T al, T sg, T& tau, T& beta, T& scale) {
    const T ss = fma(al, al, sg);
    const T aa = fabs(al);
    T rmu, mu;
    rsqrt_refined(ss, rmu, mu);
    const bool z = sg == T(0);
    beta = z ? al : -copysign(mu, al);
    tau = z ? T(0) : fma(aa, rmu, T(1));
    scale = z ? T(1) : copysign(rcp_refined(aa + mu), al);
}

// Merge of two upper-triangular n x n factors [Ra; Rb] (Rb: nb rows) by a
// GROUP of NC lanes, lane k of the group holding column k of both (R[i*ld+k]).
// Reflector j: head Ra[j][j], tail Rb[0..j][j] (structured).
// The pivot column travels by shuffles and every lane computes the squared
// norm and the Householder scalars itself, so a column costs one shuffle
// latency plus the scalar chain (no shared memory, no __syncwarp; 2.1x faster
// than a shared-memory broadcast, tools/merge_bench.cu).
// Out: Ro = new R (may alias Ra or Rb: inputs are read into registers
// first), rb = V_2 column k (rows <= k), G / tau for T.  All lanes of the warp
// call it (full-warp shuffles); lanes with on == false compute nothing useful.
template <typename T, int NC>
__device__ __forceinline__ void merge_group(bool on, int k, const T* Ra, const T* Rb, int ld, int nb, T* Ro,
                                            T (&rb)[NC], T* G, int ldg, T* tau) {
    T ra[NC];
#pragma unroll
    for (int i = 0; i < NC; ++i) {
        ra[i] = on ? Ra[i * ld + k] : T(0);
        rb[i] = (on && i < nb && i <= k) ? Rb[i * ld + k] : T(0);
    }
    __syncwarp();
#pragma unroll
    for (int j = 0; j < NC; ++j) {
        T y[NC];
#pragma unroll
        for (int i = 0; i <= j; ++i) y[i] = __shfl_sync(0xffffffffu, rb[i], j);
        const T al = __shfl_sync(0xffffffffu, ra[j], j);
        T s0 = T(0), s1 = T(0), d0 = T(0), d1 = T(0);  // ||y||^2 and y . rb_k
#pragma unroll
        for (int i = 0; i <= j; i += 2) {
            s0 = fma(y[i], y[i], s0);
            d0 = fma(y[i], rb[i], d0);
            if (i + 1 <= j) {
                s1 = fma(y[i + 1], y[i + 1], s1);
                d1 = fma(y[i + 1], rb[i + 1], d1);
            }
        }
        const T d = d0 + d1;
        T tj, beta, scale;
        householder_scalars_nb(al, s0 + s1, tj, beta, scale);
        // k > j: s_k = Ra[j][k] + v_j . rb_k, v_j tail = scale y; k == j: the
        // reflector itself; k < j: Gram entry v_k . v_j (R_a parts are unit vectors)
        const bool diag = k == j;
        const T f = k > j ? tj * fma(scale, d, ra[j]) : T(0);
        ra[j] = diag ? beta : ra[j] - f;
        const T fs = f * scale;
#pragma unroll
        for (int i = 0; i <= j; ++i) rb[i] = diag ? rb[i] * scale : fma(-fs, y[i], rb[i]);
        if (on && k < j) G[k * ldg + j] = scale * d;
        if (on && diag) tau[j] = tj;
    }
    if (on)
#pragma unroll
        for (int i = 0; i < NC; ++i) Ro[i * ld + k] = i <= k ? ra[i] : T(0);
    __syncwarp();
}

// A merge recorded for write-out after the climb: V_2 (V[k][i], rows i <= k
// of column k), the Gram entries and tau that give its T.
constexpr int kStreamMaxRec = 12;  // >= merges one warp can do (4 in-CTA + 8 cross-CTA levels)
template <typename T, int NC>
struct StreamRec {
    T V[NC][NC];
    T G[NC][NC];
    T tau[NC];
    int64_t sb;
};
template <typename T>
__device__ __forceinline__ void store_v4(T* p, T a, T b, T c, T d) {
    if constexpr (sizeof(T) == 4) {
        *reinterpret_cast<float4*>(p) = make_float4(a, b, c, d);
    } else {
        p[0] = a, p[1] = b, p[2] = c, p[3] = d;
    }
}
template <typename T>
__device__ __forceinline__ void load_v4_cg(const T* p, T (&v)[4]) {
    if constexpr (sizeof(T) == 4) {
        const float4 q = __ldcg(reinterpret_cast<const float4*>(p));
        v[0] = q.x, v[1] = q.y, v[2] = q.z, v[3] = q.w;
    } else {
        for (int e = 0; e < 4; ++e) v[e] = __ldcg(p + e);
    }
}

// Ints of the workspace exchange area holding every CTA's R (NC x NC, 32-aligned).
template <typename T, int NC>
__host__ __device__ inline int64_t stream_rx_ints(int64_t nct) {
    return ((nct * (NC * NC) * (int64_t)sizeof(T) / 4) + 31) & ~int64_t(31);
}

template <typename T, int NC, int RPL, int NW, int NBUF, bool VEC>
__global__ void __launch_bounds__(32 * NW, 1)
tsqr_stream_kernel(Geom g, T* A, T* __restrict__ Tws, int* __restrict__ sync, int nlevels,
                   unsigned long long* prof, int dbg) {
    static_assert((NW & (NW - 1)) == 0, "NW: power of two (in-CTA tree levels)");
    constexpr int B = 32 * RPL;
    constexpr int LDR = NC + 1;
    static_assert(NBUF == 1 || NBUF == 2, "one or two tile buffers");
    static_assert(RPL % 4 == 0, "rows move in 16-byte pieces (stream_row)");
    using SW = StreamWarp<T, NC, B, NBUF>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    SW* Ws = reinterpret_cast<SW*>(smem_raw);
    SW& W = Ws[warp];
    const int64_t base = (int64_t)blockIdx.x * NW;
    const int64_t chain = base + warp;
    // warp-uniform values through a shuffle: the compiler then knows the
    // branches around the warp collectives are uniform (a thread-dependent
    // condition compiles every shuffle to slow WARPSYNC.COLLECTIVE code)
    const bool live = __shfl_sync(0xffffffffu, chain < g.P ? 1 : 0, 0) != 0;
    const int wp = g.ncols;
    // arrival counters of the in-CTA tree levels ([level][leftmost warp])
    constexpr int kInLevels = NW >= 16 ? 4 : NW >= 8 ? 3 : NW >= 4 ? 2 : 1;
    __shared__ int s_cnt[kInLevels * NW];
    for (int i = threadIdx.x; i < kInLevels * NW; i += 32 * NW) s_cnt[i] = 0;
    __syncthreads();

    // optional timestamps (diagnostics, CAQR_PROFILE=1): [0] min chain start,
    // [1] max chain end, [2] root done (ns, globaltimer); [3] sum of chain
    // times; [4] cycles waiting for tiles; [5] last-CTA tree time; [6] merges
    auto gtime = []() {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        return t;
    };
    const unsigned long long tstart = prof ? gtime() : 0ull;
    unsigned long long twait = 0;
    // slot rows of tree leaf sl (top rows of its chain's first tile)
    auto slot_ptr = [&](int64_t sl) { return A + g.col0 * g.lda + g.row0 + sl * g.bm; };
    auto slot_h = [&](int64_t sl) { return min64(g.b, g.mrows - sl * g.bm); };
    // V_2 of a merge into R_b's slot (upper incl. diagonal) and its T
    auto store_merge = [&](bool on, int k, int64_t sb, const T (&rb)[NC], const T* G, const T* tau) {
        const int64_t hb = slot_h(sb);
        if (on && k < wp) {
            T* bb = slot_ptr(sb) + k * g.lda;
#pragma unroll
            for (int i = 0; i < NC; ++i)
                if (i <= k && i < hb) bb[i] = rb[i];
        }
        stream_write_t<T, NC>(on, k, G, LDR, tau, wp, Tws + ((g.L + sb) * g.npan) * (kPW * kPW));
    };

    // ---- the chain: tiles chain*K .., leaf first; R stays in W.R ----------
    if (live) {
        const int64_t t0 = chain * g.K;
        const int ntile = __shfl_sync(0xffffffffu, (int)min64(g.K, g.L - t0), 0);
        // Full tiles of a 16-byte aligned panel come by bulk copy (mbarrier
        // per buffer), the rest -- a ragged last tile, or every tile of an
        // unaligned panel -- by cp.async with zero fill.  Only the matrix's
        // last tile (the last of its chain) can be ragged, so the bulk tiles
        // of a buffer are consecutive uses and the wait parity is kt / NBUF.
        auto bulk = [&](int64_t t) { return VEC && (t + 1) * g.b <= g.mrows; };
        auto issue = [&](int64_t t, int bi) {
            if (bulk(t))
                stream_issue_bulk<T, NC, B>(g, A, t, W.buf[bi], &W.mbar[bi]);
            else
                stream_issue_tile<T, NC, B, VEC>(g, A, t, W.buf[bi]);
        };
        if (VEC) {
            if (lane == 0)
                for (int bi = 0; bi < NBUF; ++bi) umma::mbar_init(&W.mbar[bi], 1);
            for (int bi = 0; bi < NBUF; ++bi)  // columns no bulk copy writes
                for (int c = wp; c < NC; ++c)
                    for (int r = lane; r < B; r += 32) W.buf[bi][c][r] = T(0);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
            umma::fence_async_smem();
            __syncwarp();
        }
        issue(t0, 0);
        for (int kt = 0; kt < ntile; ++kt) {
            const int64_t t = t0 + kt;
            const long long cw0 = prof ? clock64() : 0;
            if (NBUF == 2 && kt + 1 < ntile) issue(t + 1, (kt + 1) % NBUF);
            if (bulk(t))
                umma::mbar_wait(&W.mbar[kt % NBUF], (uint32_t)((kt / NBUF) & 1));
            else
                asm volatile("cp.async.wait_group 0;" ::: "memory");
            if (prof) twait += clock64() - cw0;
            __syncwarp();
            const int h = (int)min64(g.b, g.mrows - t * g.b);
            T x[NC][RPL];
#pragma unroll
            for (int c = 0; c < NC; ++c)
#pragma unroll
                for (int u = 0; u < RPL / 4; ++u) {
                    const T* p = &W.buf[kt % NBUF][c][128 * u + 4 * lane];
                    if constexpr (sizeof(T) == 4) {
                        const float4 q = *reinterpret_cast<const float4*>(p);
                        x[c][4 * u] = q.x, x[c][4 * u + 1] = q.y, x[c][4 * u + 2] = q.z, x[c][4 * u + 3] = q.w;
                    } else {
#pragma unroll
                        for (int e = 0; e < 4; ++e) x[c][4 * u + e] = p[e];
                    }
                }
            __syncwarp();  // the buffer is refilled (tile kt + NBUF) after this point
            if (NBUF == 1 && kt + 1 < ntile) issue(t + 1, 0);
            if (kt == 0)
                stream_tile_qr<T, NC, RPL, true, B, NBUF>(x, W, h);
            else
                stream_tile_qr<T, NC, RPL, false, B, NBUF>(x, W, h);
            // V (and a leaf's R) back over the tile; T into its slot
            const int64_t s = g.row0 + t * g.b;
#pragma unroll
            for (int c = 0; c < NC; ++c) {
                if (c < wp) {
                    T* col = A + (g.col0 + c) * g.lda + s;
#pragma unroll
                    for (int u = 0; u < RPL / 4; ++u) {
                        const int r = 128 * u + 4 * lane;
                        if (VEC && sizeof(T) == 4 && r + 4 <= h) {
                            store_v4<T>(col + r, x[c][4 * u], x[c][4 * u + 1], x[c][4 * u + 2], x[c][4 * u + 3]);
                        } else {
#pragma unroll
                            for (int e = 0; e < 4; ++e)
                                if (r + e < h) col[r + e] = x[c][4 * u + e];
                        }
                    }
                }
            }
            stream_write_t<T, NC>(lane < NC, lane, &W.G[0][0], LDR, W.tau, wp, Tws + (t * g.npan) * (kPW * kPW));
            __syncwarp();
        }
        if (prof && lane == 0) {
            const unsigned long long te = gtime();
            atomicMin(prof + 0, tstart);
            atomicMax(prof + 1, te);
            atomicAdd(prof + 3, te - tstart);
            atomicAdd(prof + 4, twait);
        }
    }

    // ---- the binary tree over the chain R's -------------------
    // A merge's V_2 and T are not needed by the levels above it (only its new
    // R is), so they are recorded in the merging warp's free tile buffers and
    // written out after the climb, by all warps of the CTA together.
    // (as many as fit: all of them for n <= 8; merges beyond the capacity
    // store at once)
    using Rec = StreamRec<T, NC>;
    constexpr int kRecFit = (int)(sizeof(T) * NBUF * NC * B / sizeof(Rec));
    constexpr int kRecCap = kRecFit < kStreamMaxRec ? kRecFit : kStreamMaxRec;
    static_assert(NC > 8 || kRecCap == kStreamMaxRec, "n <= 8: every merge record fits in the tile buffers");
    __shared__ int s_nrec[NW];
    int nrec = 0;
    auto merge_rec = [&](const T* Ra, const T* Rb, int nb, T* Ro, int64_t sb) {
        T rb[NC];
        merge_group<T, NC>(lane < NC, lane, Ra, Rb, LDR, nb, Ro, rb, &W.G[0][0], LDR, W.tau);
        if (nrec >= kRecCap) {
            store_merge(lane < NC, lane, sb, rb, &W.G[0][0], W.tau);
            return;
        }
        Rec& r = reinterpret_cast<Rec*>(&W.buf[0][0][0])[nrec++];
        if (lane < NC) {
#pragma unroll
            for (int i = 0; i < NC; ++i) {
                r.V[lane][i] = rb[i];
                r.G[i][lane] = W.G[i][lane];
            }
            r.tau[lane] = W.tau[lane];
        }
        if (lane == 0) r.sb = sb;
        __syncwarp();
    };
    // The climb: every level's pair is merged by whichever member arrives
    // SECOND (an arrival counter per pair; the first stops).  Inside the CTA
    // a subtree's R lives in the shared R of the warp of its leftmost chain
    // and the counters are shared-memory atomics; across CTAs the R travels
    // through the workspace exchange area.  No barrier: the critical path is
    // the last chain's own merges.  Release/acquire on the counters (one
    // lane, after __syncwarp) publishes the R written by the whole warp.
    // (root path stamps, CAQR_PROFILE=1: [8] tree start, [9] in-CTA levels
    // done, [10..13] sums of publish / ticket / sibling load / merge, [14]
    // cross-CTA merges, [15] root done)
    unsigned long long tp[6] = {0, 0, 0, 0, 0, 0};
    if (prof) tp[0] = gtime();
    auto store_r = [&](const T* R, int64_t sl) {  // R (upper) into the slot's top rows
        const int64_t hs = slot_h(sl);
        if (lane < NC && lane < wp) {
            T* col = slot_ptr(sl) + lane * g.lda;
#pragma unroll
            for (int i = 0; i < NC; ++i)
                if (i <= lane && i < hs) col[i] = R[i * LDR + lane];
        }
    };
    if (live) {
        int64_t cur = chain;  // leftmost chain of this warp's subtree
        bool root = true;
        int l = 0;
        for (; (2 << l) <= NW && l < nlevels; ++l) {
            const int hl = 1 << l;
            const int64_t sa = cur & ~int64_t(2 * hl - 1), sb = sa + hl;
            if (sb >= g.P) continue;  // no right member at this level: pass up
            __syncwarp();
            int old = 0;
            if (lane == 0)
                asm volatile("atom.acq_rel.cta.shared::cta.add.s32 %0, [%1], 1;"
                             : "=r"(old)
                             : "r"(umma::smem_u32(&s_cnt[l * NW + (int)(sa - base)]))
                             : "memory");
            old = __shfl_sync(0xffffffffu, old, 0);
            if (old == 0) {  // the sibling merges
                root = false;
                break;
            }
            __syncwarp();
            T* Ra = &Ws[sa - base].R[0][0];
            merge_rec(Ra, &Ws[sb - base].R[0][0], (int)min64(NC, slot_h(sb)), Ra, sb);
            cur = sa;
        }
        if (prof) tp[1] = gtime();
        if (root && l >= nlevels) {  // the whole tree fitted in this CTA
            store_r(&Ws[0].R[0][0], base);
        } else if (root) {
            // ---- across CTAs -------------------------------------------------
            const int nct = (int)gridDim.x;
            constexpr int NQ = NC * NC / 4;  // float4's per R
            T* Rx = reinterpret_cast<T*>(sync + 64);          // [nct][NC][NC]
            int* cnt = sync + 64 + stream_rx_ints<T, NC>(nct);  // [levels][nct]
            const int l0 = l;
            int64_t cc = blockIdx.x;  // CTA whose slot (cc * NW) this R belongs to
            T* Rm = &Ws[0].R[0][0];
            T* Rs = &W.Rs[0][0];
            int nx = 0;
            // Poll every level above at once (lane q: level l0 + q, acquire):
            // where the sibling subtree has already arrived, this CTA is the
            // second at that pair whatever happens below, so it merges there
            // without publishing its R or taking a ticket.  (The last CTA to
            // finish finds all its siblings done: one round trip for the poll
            // instead of a publish + ticket per level.)
            unsigned ready = 0;
            {
                int v = 0;
                const int lq = l0 + lane;
                if (lq < nlevels && lq < 31) {
                    const int64_t hl = int64_t(1) << lq;
                    const int64_t sa = base & ~(2 * hl - 1), sb = sa + hl;
                    if (sb < g.P)
                        asm volatile("ld.acquire.gpu.global.s32 %0, [%1];"
                                     : "=r"(v)
                                     : "l"(cnt + (int64_t)(lq - l0) * nct + sa / NW)
                                     : "memory");
                }
                ready = __ballot_sync(0xffffffffu, v != 0);
                __syncwarp();
            }
            for (; l < nlevels; ++l) {
                const int64_t hl = int64_t(1) << l;
                const int64_t slot = cc * NW;
                const bool left = ((slot >> l) & 1) == 0;
                const int64_t sa = left ? slot : slot - hl, sb = sa + hl;
                if (sb >= g.P) continue;  // no right member at this level: pass up
                unsigned long long c0 = prof ? gtime() : 0ull;
                if (!((ready >> (l - l0)) & 1u)) {  // publish, then the ticket decides
                    for (int q = lane; q < NQ; q += 32) {
                        const int i = (4 * q) / NC, c = (4 * q) % NC;
                        const T* rr = Rm + i * LDR + c;
                        store_v4<T>(Rx + cc * NC * NC + 4 * q, rr[0], rr[1], rr[2], rr[3]);
                    }
                    __syncwarp();
                    if (prof) { const unsigned long long c1 = gtime(); tp[2] += c1 - c0; c0 = c1; }
                    int old = 0;
                    if (lane == 0)
                        asm volatile("atom.acq_rel.gpu.global.add.s32 %0, [%1], 1;"
                                     : "=r"(old)
                                     : "l"(cnt + (int64_t)(l - l0) * nct + sa / NW)
                                     : "memory");
                    old = __shfl_sync(0xffffffffu, old, 0);
                    if (prof) { const unsigned long long c1 = gtime(); tp[3] += c1 - c0; c0 = c1; }
                    if (old == 0) {  // the sibling merges
                        root = false;
                        break;
                    }
                }
                __syncwarp();
                const int64_t other = (left ? sb : sa) / NW;
                for (int q = lane; q < NQ; q += 32) {
                    const int i = (4 * q) / NC, c = (4 * q) % NC;
                    T v[4];
                    load_v4_cg<T>(Rx + other * NC * NC + 4 * q, v);
#pragma unroll
                    for (int e = 0; e < 4; ++e) Rs[i * LDR + c + e] = v[e];
                }
                __syncwarp();
                if (prof) { const unsigned long long c1 = gtime(); tp[4] += c1 - c0; c0 = c1; }
                merge_rec(left ? Rm : Rs, left ? Rs : Rm, (int)min64(NC, slot_h(sb)), Rm, sb);
                if (prof) { tp[5] += gtime() - c0; ++nx; }
                cc = sa / NW;
            }
            if (root) {
                store_r(Rm, 0);  // the root R into A's top rows
                if (prof && lane == 0) {
                    const unsigned long long te = gtime();
                    atomicMax(prof + 2, te);
                    for (int q = 0; q < 6; ++q) prof[8 + q] = tp[q];
                    prof[14] = nx;
                    prof[15] = te;
                }
            }
        }
    }
    // ---- write out every recorded merge (V_2 into R_b's slot, T), CTA-wide
    if (lane == 0) s_nrec[warp] = nrec;
    __syncthreads();
    {
        int idx = 0;
        for (int w = 0; w < NW; ++w) {
            const int nw = s_nrec[w];
            const Rec* rs = reinterpret_cast<const Rec*>(&Ws[w].buf[0][0][0]);
            for (int r = 0; r < nw; ++r, ++idx) {
                if (idx % NW != warp) continue;
                const Rec& rc = rs[r];
                const int64_t sb = rc.sb;
                const int k = lane;
                const int64_t hb = slot_h(sb);
                if (k < NC && k < wp) {
                    T* bb = slot_ptr(sb) + k * g.lda;
#pragma unroll
                    for (int i = 0; i < NC; ++i)
                        if (i <= k && i < hb) bb[i] = rc.V[k][i];
                }
                stream_write_t<T, NC>(k < NC, k, &rc.G[0][0], NC, rc.tau, wp,
                                      Tws + ((g.L + sb) * g.npan) * (kPW * kPW));
            }
        }
    }
}

template <typename T, int NC, int RPL, int NW, int NBUF = 2>
inline size_t stream_smem_bytes(int64_t /*nct*/) {
    return sizeof(StreamWarp<T, NC, 32 * RPL, NBUF>) * NW;
}

}  // namespace caqr
