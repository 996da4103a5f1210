// tsqr_kernels.cuh -- sm_100a device code of the TSQR / CAQR hot path.
//
// Two kernels carry the whole method:
//
//  panel_factor_kernel   Householder QR of one <=32-column panel of one tree
//                        node (a leaf row block -- the paper's "factor",
//                        or a stacked pair of R factors -- its
//                        "factor_tree"), entirely in shared memory,
//                        one CTA per node.  Per column: warp-shuffle norm,
//                        reflector, warp-shuffle dot products s = A^T v and the
//                        rank-1 update A -= tau v s^T (Fig. 5), then
//                        the compact-WY factor T from the inner products of the
//                        vectors.
//  panel_update_kernel   C <- (I - V T V^T)^T C (or without ^T) for one node and
//                        one 32-column block of C: W = V^T C, W = T^T W,
//                        C -= V W -- the blocked trailing update
//                        used horizontally across leaves ("apply_qt_h",
//                        P:L665-668) and on the gathered rows of tree nodes
//                        ("apply_qt_tree", Fig. 3(c,d)).
//
// A tree node's rows are "gathered": a leaf is one contiguous row segment; a
// merge of R_a and R_b (binary tree) is the segment holding R_a's
// rows of the current panel followed by the segment holding R_b's top rows.
// Masks keep the stacked-triangle structure ("possibly exploiting
// the sparsity pattern") and keep the leaves' vectors that share those rows
// untouched (tree vectors overwrite exactly the R slots).
#pragma once
#include <cooperative_groups.h>
#include <cstdint>
#include <cuda_runtime.h>

namespace caqr {

constexpr int kPW = 32;        // max reflectors per panel step (panel width)
constexpr int kThreads = 256;  // 8 warps
constexpr int kWarps = kThreads / 32;
constexpr int kTS = 36;        // stride of 32x32 scratch tiles (16-byte aligned rows)

// Geometry of one TSQR panel group (a column panel of width ncols <= 256 that
// starts at row0 = col0 of A; the grid redrawn "nb rows lower").
// Rows are cut into L tiles of b rows (the last one ragged).  Consecutive
// tiles form chains of K tiles (a flat tree, "any tree shape" P:L339-341): the
// first tile of a chain is a leaf QR, each later tile a structured QR of
// [chain R; tile].  The P chain R factors are reduced by a binary tree.
struct Geom {
    int64_t lda;
    int64_t row0;   // first row of the group
    int64_t mrows;  // rows of the group (m - row0)
    int64_t col0;   // first column of the group
    int64_t b;      // tile (leaf) height
    int64_t L;      // number of tiles
    int64_t K;      // tiles per chain
    int64_t P;      // chains = leaves of the binary tree
    int64_t bm;     // rows per chain (K * b): stride of the tree's R slots
    int32_t ncols;  // group width
    int32_t npan;   // ceil(ncols / 32)
};

// The gathered rows of one node for panel p.  level < 0: tile kt of chain
// `node` (kt == 0: leaf); level >= 0: merge `node` of that tree level.
struct NodeRows {
    int64_t r0, r1;      // first absolute row of segment 0 / segment 1
    int32_t n0, n1;      // rows in segment 0 / 1
    int32_t seg0_tri;    // 1: segment 0 is an R slot (heads on its diagonal, v = e_j there)
    int32_t seg1_upper;  // 1: segment 1 is an upper-triangular R slot (merge); 0: dense
    int64_t tblk;        // index of this (node, panel)'s 32x32 T block in the workspace
};

__device__ __forceinline__ NodeRows node_rows(const Geom& g, int level, int64_t node, int p, int wp,
                                              int kt) {
    NodeRows nr;
    if (level < 0) {
        const int64_t t = node * g.K + kt;  // tile index
        const int64_t s = g.row0 + t * g.b;
        const int64_t h = t < g.L ? min(g.b, g.mrows - t * g.b) : 0;
        nr.tblk = t * g.npan + p;
        nr.seg1_upper = 0;
        if (kt == 0) {  // leaf
            nr.r0 = s + 32 * p;
            nr.n0 = (int32_t)(h - 32 * p > 0 ? h - 32 * p : 0);
            nr.r1 = 0;
            nr.n1 = 0;
            nr.seg0_tri = 0;
        } else {  // [chain R; tile]
            nr.r0 = g.row0 + node * g.bm + 32 * p;
            nr.n0 = h > 0 ? wp : 0;
            nr.r1 = s;
            nr.n1 = (int32_t)h;
            nr.seg0_tri = 1;
        }
    } else {
        const int64_t a = node << (level + 1);
        const int64_t bb = a + (int64_t(1) << level);
        const int64_t hb = min(g.b, g.mrows - bb * g.bm);
        nr.r0 = g.row0 + a * g.bm + 32 * p;
        nr.n0 = wp;
        nr.r1 = g.row0 + bb * g.bm;
        nr.n1 = (int32_t)(32 * p + wp < hb ? 32 * p + wp : hb);
        nr.seg0_tri = 1;
        nr.seg1_upper = 1;
        nr.tblk = (g.L + bb) * g.npan + p;  // merges: indexed by the right member's slot
    }
    return nr;
}

// Absolute row of gathered row r.
__device__ __forceinline__ int64_t gathered_row(const NodeRows& nr, int r) {
    return r < nr.n0 ? nr.r0 + r : nr.r1 + (r - nr.n0);
}

// Is entry (gathered row r, panel column jj) of the panel stored in A for this
// node?  Leaves and dense tiles: every entry (R on/above the diagonal, v
// below).  An R-slot segment 0 holds R on and above the diagonal only (below it
// sit leaf vectors); a merge's R_b segment holds an upper-triangular R (factor
// input) / V_2 (tree vectors) only -- local row i <= 32p + jj.
__device__ __forceinline__ bool panel_entry_stored(const NodeRows& nr, int r, int jj, int p) {
    if (r < nr.n0) return !nr.seg0_tri || r <= jj;
    return !nr.seg1_upper || (r - nr.n0) <= 32 * p + jj;
}

// Householder vector entry (gathered row r, panel column jj) given the stored
// value: unit head, zeros above it, the structure's zeros.
template <typename T>
__device__ __forceinline__ T v_entry(const NodeRows& nr, int r, int jj, int p, T stored) {
    if (r < nr.n0) {
        if (nr.seg0_tri) return r == jj ? T(1) : T(0);
        return r > jj ? stored : (r == jj ? T(1) : T(0));
    }
    if (nr.seg1_upper) return (r - nr.n0) <= 32 * p + jj ? stored : T(0);
    return stored;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Column stride (elements) of a column-major shared tile with >= rows rows:
// rows rounded up to 32, plus 16 bytes, so that 16-byte vector loads by lanes
// reading 8 different columns at the same rows hit 8 disjoint bank groups.
template <typename T>
__host__ __device__ __forceinline__ int smem_col_stride(int rows) {
    const int r32 = (rows + 31) & ~31;
    return r32 + int(16 / sizeof(T));
}

// ---------------------------------------------------------------------------
// Reflector of panel column j (xLARFG, reading S1), computed by ONE
// warp: alpha = P[j][j], sigma = sum_{r>j} P[r][j]^2 (warp-shuffle reduction),
// beta = -copysign(sqrt(alpha^2+sigma), alpha), tau = (beta-alpha)/beta,
// v = P[j+1:, j] / (alpha - beta); P[j][j] <- beta.  sigma == 0 -> tau = 0.
// ---------------------------------------------------------------------------
template <typename T>
__device__ __forceinline__ void make_reflector(T* P, int RGP, int RG, int j, T* tau_s, int lane) {
    T* col = P + (size_t)j * RGP;
    const T alpha = (j < RG) ? col[j] : T(0);
    T sigma = T(0);
    for (int r = j + 1 + lane; r < RG; r += 32) {
        const T x = col[r];
        sigma = fma(x, x, sigma);
    }
    sigma = warp_sum(sigma);
    T tau = T(0);
    if (j < RG && sigma != T(0)) {
        const T mu = sqrt(fma(alpha, alpha, sigma));
        const T beta = -copysign(mu, alpha);
        tau = (beta - alpha) / beta;
        const T scale = T(1) / (alpha - beta);
        for (int r = j + 1 + lane; r < RG; r += 32) col[r] *= scale;
        __syncwarp();
        if (lane == 0) col[j] = beta;
    }
    if (lane == 0) tau_s[j] = tau;
    __syncwarp();
}

// ---------------------------------------------------------------------------
// panel_factor_kernel: grid = nodes of this level, block = 256 threads.
// Shared: P (wp columns x RGP), G (32x33), Tm (32x33), tau (32).
// ---------------------------------------------------------------------------
template <typename T>
__global__ void __launch_bounds__(kThreads)
panel_factor_kernel(Geom g, T* A, T* __restrict__ Tws, int level, int p, int kt) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int wp = min(kPW, g.ncols - 32 * p);
    const NodeRows nr = node_rows(g, level, blockIdx.x, p, wp, kt);
    const int RG = nr.n0 + nr.n1;
    const int RGP = smem_col_stride<T>(RG);
    T* P = reinterpret_cast<T*>(smem_raw);
    T* G = P + (size_t)wp * RGP;
    T* Tm = G + kPW * kTS;
    T* tau_s = Tm + kPW * kTS;
    const int64_t c0 = g.col0 + 32 * p;

    // ---- stage: coalesced column loads (lanes along rows) with structure masks
    for (int jj = warp; jj < wp; jj += kWarps) {
        const T* col = A + (c0 + jj) * g.lda;
        T* pc = P + (size_t)jj * RGP;
        for (int r = lane; r < RG; r += 32)
            pc[r] = panel_entry_stored(nr, r, jj, p) ? col[gathered_row(nr, r)] : T(0);
    }
    __syncthreads();

    // ---- unblocked Householder over the panel columns ----------
    // Column c is owned by warp c % 8.  After reflector j is published, each
    // warp applies it to its columns c > j (dot via shuffles, rank-1 update);
    // the owner of column j+1 builds reflector j+1 right after updating it, so
    // one CTA barrier per column suffices.
    if (warp == 0) make_reflector(P, RGP, RG, 0, tau_s, lane);
    __syncthreads();
    for (int j = 0; j < wp; ++j) {
        const T tau = tau_s[j];
        const T* v = P + (size_t)j * RGP;
        int c = j + 1 + ((warp - (j + 1)) % kWarps + kWarps) % kWarps;  // first owned c > j
        for (; c < wp; c += kWarps) {
            T* a = P + (size_t)c * RGP;
            if (tau != T(0)) {
                T s = T(0);
                for (int r = j + 1 + lane; r < RG; r += 32) s = fma(v[r], a[r], s);
                s = warp_sum(s);
                s = (s + a[j]) * tau;
                __syncwarp();
                for (int r = j + 1 + lane; r < RG; r += 32) a[r] = fma(-s, v[r], a[r]);
                if (lane == 0) a[j] -= s;
                __syncwarp();
            }
            if (c == j + 1) make_reflector(P, RGP, RG, c, tau_s, lane);
        }
        __syncthreads();
    }

    // ---- compact-WY T (LAPACK xLARFT, forward/columnwise) -------
    // G[i][j] = v_i . v_j (i < j) with unit heads; T[j][j] = tau_j,
    // T[0:j, j] = -tau_j T[0:j, 0:j] G[0:j, j].
    for (int j = warp; j < wp; j += kWarps) {
        const T* vj = P + (size_t)j * RGP;
        for (int i = 0; i < j; ++i) {
            const T* vi = P + (size_t)i * RGP;
            T s = T(0);
            for (int r = j + 1 + lane; r < RG; r += 32) s = fma(vi[r], vj[r], s);
            s = warp_sum(s);
            if (lane == 0) G[i * kTS + j] = s + (j < RG ? vi[j] : T(0));
        }
    }
    __syncthreads();
    if (warp == 0 && lane < wp) {
        const int i = lane;
        Tm[i * kTS + i] = tau_s[i];
        for (int j = i + 1; j < wp; ++j) {
            T t = T(0);
            for (int k = i; k < j; ++k) t = fma(Tm[i * kTS + k], G[k * kTS + j], t);
            Tm[i * kTS + j] = -tau_s[j] * t;
        }
    }
    __syncthreads();

    // ---- write back: panel (masked) to A, T (32x32 column-major) to ws ------
    for (int jj = warp; jj < wp; jj += kWarps) {
        T* col = A + (c0 + jj) * g.lda;
        const T* pc = P + (size_t)jj * RGP;
        for (int r = lane; r < RG; r += 32)
            if (panel_entry_stored(nr, r, jj, p)) col[gathered_row(nr, r)] = pc[r];
    }
    T* tb = Tws + nr.tblk * (kPW * kPW);
    for (int e = threadIdx.x; e < kPW * kPW; e += kThreads) {
        const int r = e & 31, c = e >> 5;
        tb[e] = (r <= c && c < wp) ? Tm[r * kTS + c] : T(0);
    }
}

template <typename T>
inline size_t panel_factor_smem(int wp, int RGmax) {
    return sizeof(T) * ((size_t)wp * smem_col_stride<T>(RGmax) + 2 * kPW * kTS + kPW);
}

// ---------------------------------------------------------------------------
// panel_update_kernel: C[gathered rows, block] <- op(I - V T V^T) C.
// grid.x = nodes, grid.y = 32-column blocks of C's [cfirst, cfirst+ccount).
// trans = 1: Q^T (W = T^T V^T C), trans = 0: Q (W = T V^T C).
// Shared: Vs, Cs (32 columns x RGP, column-major, rows zero-padded to 32),
// Wp (4 K-split partials of 32x33), Tt (32x33), W (32x33).
// ---------------------------------------------------------------------------
template <typename T>
struct Vec4;  // 16-byte vector of T
template <>
struct Vec4<float> {
    using type = float4;
    static constexpr int n = 4;
};
template <>
struct Vec4<double> {
    using type = double2;
    static constexpr int n = 2;
};

template <typename T>
__device__ __forceinline__ T vget(const float4& v, int i) {
    return i == 0 ? v.x : i == 1 ? v.y : i == 2 ? v.z : v.w;
}
template <typename T>
__device__ __forceinline__ T vget(const double2& v, int i) {
    return i == 0 ? v.x : v.y;
}

// The mma (3xTF32 tensor-core) version of the two GEMMs, for the factor
// path's CAQR trailing update only (apply_qt / apply_q / form_q use FFMA).
struct Grp {
    int tid;
    int bar;  // 0: __syncthreads over the CTA; >0: bar.sync bar, 256
};
template <bool PAD>
__device__ __forceinline__ void gemm_vtc_mma(const Grp& G, const float* Vs, const float* Cs, int RGP, int R32,
                                             float* Wp, float* W);
template <bool PAD>
__device__ __forceinline__ void gemm2_mma(const Grp& G, const float* Vs, float* Cs, const float* W, int RGP,
                                          int R32);

// One (node, panel p) of the implicit Q applied to column blocks [blk_beg,
// blk_end) of C: C <- (I - V T V^T)^T C (trans) or (I - V T V^T) C, on the node's
// gathered rows (the horizontal / tree updates).  A device routine
// so that one launch can walk a whole chain (chain_update_kernel) as well as
// one launch per (level, panel) (panel_update_kernel).
template <typename T, bool MMA>
__device__ __forceinline__ void update_node(const Geom& g, const T* A, const T* __restrict__ Tws, int level,
                                            int64_t node, int p, int kt, T* C, int64_t ldc, int64_t cfirst,
                                            int64_t ccount, int trans, int64_t blk_beg, int64_t blk_end,
                                            unsigned char* smem_raw) {
    using V4 = typename Vec4<T>::type;
    constexpr int VN = Vec4<T>::n;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int wp = min(kPW, g.ncols - 32 * p);
    const NodeRows nr = node_rows(g, level, node, p, wp, kt);
    const int RG = nr.n0 + nr.n1;
    if (RG == 0) return;
    __syncthreads();  // a previous call's readers of the shared tiles are done
    // 16-byte C stores: C aligned, ldc % 4 == 0 and every gathered-row segment
    // (R slots, tiles) starting on a multiple of 4 rows
    const bool vec_p = sizeof(T) == 4 && (reinterpret_cast<uintptr_t>(C) % 16 == 0) && (ldc % 4 == 0) &&
                       (g.row0 % 4 == 0) && (g.b % 4 == 0) && (g.bm % 4 == 0) && (nr.r0 % 4 == 0) &&
                       (nr.r1 % 4 == 0) && (nr.n0 % 4 == 0);
    const int R32 = (RG + 31) & ~31;
    const int RGP = smem_col_stride<T>(RG);
    T* Vs = reinterpret_cast<T*>(smem_raw);
    T* Cs = Vs + 32 * (size_t)RGP;
    T* Wp = Cs + 32 * (size_t)RGP;  // 4 x 32 x kTS
    T* Tt = Wp + 4 * 32 * kTS;
    T* W = Tt + 32 * kTS;
    const int64_t c0 = g.col0 + 32 * p;

    // ---- stage V (implicit unit heads, structure masks) and C ---------------
    // Each thread issues its loads in batches (4 columns x up to 9 row groups)
    // before storing: one outstanding load per element would serialize the
    // L2/HBM latency.
    int64_t cb0 = 0;
    int ncb = 0;
    auto stage = [&](int pass) {
        T buf[4][9];
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const int jj = warp + kWarps * a;
            const T* acol = A + (c0 + jj) * g.lda;
            const T* ccol = C + (cb0 + jj) * ldc;
#pragma unroll
            for (int i = 0; i < 9; ++i) {
                const int r = lane + 32 * i;
                T val = T(0);
                if (r < RG) {
                    if (pass == 0) {
                        if (jj < wp) {
                            const bool st = panel_entry_stored(nr, r, jj, p) && (r >= nr.n0 || !nr.seg0_tri) &&
                                            !(r < nr.n0 && r <= jj);
                            val = st ? acol[gathered_row(nr, r)] : T(0);
                        }
                    } else if (jj < ncb) {
                        val = ccol[gathered_row(nr, r)];
                    }
                }
                buf[a][i] = val;
            }
        }
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const int jj = warp + kWarps * a;
            T* dst = (pass == 0 ? Vs : Cs) + (size_t)jj * RGP;
#pragma unroll
            for (int i = 0; i < 9; ++i) {
                const int r = lane + 32 * i;
                if (r < R32) {
                    T val = buf[a][i];
                    if (pass == 0) val = (r < RG && jj < wp) ? v_entry<T>(nr, r, jj, p, val) : T(0);
                    dst[r] = val;
                }
            }
        }
    };
    stage(0);  // V once per CTA
    {
        const T* tb = Tws + nr.tblk * (kPW * kPW);
        // only the wp x wp part of a T block is meaningful (the skinny kernel
        // writes nothing else)
        for (int e = tid; e < kPW * kPW; e += kThreads)
            Tt[(e & 31) * kTS + (e >> 5)] = ((e & 31) < wp && (e >> 5) < wp) ? tb[e] : T(0);
    }
    for (int64_t blk = blk_beg; blk < blk_end; ++blk) {
    cb0 = cfirst + 32 * blk;
    ncb = (int)(cfirst + ccount - cb0 < 32 ? cfirst + ccount - cb0 : 32);
    __syncthreads();  // the previous block's readers of Cs are done
    if constexpr (sizeof(T) == 4) {
        if (vec_p) {
            // 16-byte loads of 4 consecutive gathered rows (one segment, aligned):
            // a quarter of the load instructions, all issued before the stores
            const int nq4 = R32 >> 2;  // <= 72
            float4 b4[9];
#pragma unroll
            for (int u = 0; u < 9; ++u) {
                const int e = tid + kThreads * u;
                const int jj = e / nq4, r = 4 * (e - jj * nq4);
                float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
                if (jj < ncb && r < RG) {
                    const float* src = reinterpret_cast<const float*>(C) + (cb0 + jj) * ldc + gathered_row(nr, r);
                    if (r + 4 <= RG) {
                        v = __ldcg(reinterpret_cast<const float4*>(src));
                    } else {
                        v.x = src[0];
                        if (r + 1 < RG) v.y = src[1];
                        if (r + 2 < RG) v.z = src[2];
                    }
                }
                b4[u] = v;
            }
#pragma unroll
            for (int u = 0; u < 9; ++u) {
                const int e = tid + kThreads * u;
                const int jj = e / nq4, r = 4 * (e - jj * nq4);
                if (jj < 32) *reinterpret_cast<float4*>(reinterpret_cast<float*>(Cs) + (size_t)jj * RGP + r) = b4[u];
            }
        } else {
            stage(1);
        }
    } else {
        stage(1);
    }
    __syncthreads();

    if constexpr (MMA) {
        gemm_vtc_mma<false>(Grp{tid, 0}, Vs, Cs, RGP, R32, Wp, W);
    } else {
    // ---- W = V^T C : 4-way split over rows x 2 column halves per warp -------
    {
        const int ks = warp & 3, ch = warp >> 2;
        const int jg = lane & 7, cg = lane >> 3;  // jj = jg + 8e (e<4), c = 16ch + cg + 4e (e<4)
        const int chunk = R32 / 4;                // multiple of 8
        const int rbeg = ks * chunk, rend = rbeg + chunk;
        T acc[4][4];
#pragma unroll
        for (int a = 0; a < 4; ++a)
#pragma unroll
            for (int b2 = 0; b2 < 4; ++b2) acc[a][b2] = T(0);
        for (int r = rbeg; r < rend; r += VN) {
            V4 vv[4], cc[4];
#pragma unroll
            for (int e = 0; e < 4; ++e)
                vv[e] = *reinterpret_cast<const V4*>(Vs + (size_t)(jg + 8 * e) * RGP + r);
#pragma unroll
            for (int e = 0; e < 4; ++e)
                cc[e] = *reinterpret_cast<const V4*>(Cs + (size_t)(16 * ch + cg + 4 * e) * RGP + r);
#pragma unroll
            for (int q = 0; q < VN; ++q)
#pragma unroll
                for (int a = 0; a < 4; ++a)
#pragma unroll
                    for (int b2 = 0; b2 < 4; ++b2)
                        acc[a][b2] = fma(vget<T>(vv[a], q), vget<T>(cc[b2], q), acc[a][b2]);
        }
#pragma unroll
        for (int a = 0; a < 4; ++a)
#pragma unroll
            for (int b2 = 0; b2 < 4; ++b2)
                Wp[(ks * 32 + jg + 8 * a) * kTS + 16 * ch + cg + 4 * b2] = acc[a][b2];
    }
    __syncthreads();
    // reduce the 4 partials (fixed order: deterministic)
    for (int e = tid; e < 32 * 32; e += kThreads) {
        const int jj = e >> 5, c = e & 31;
        T s = Wp[(0 * 32 + jj) * kTS + c];
        s += Wp[(1 * 32 + jj) * kTS + c];
        s += Wp[(2 * 32 + jj) * kTS + c];
        s += Wp[(3 * 32 + jj) * kTS + c];
        W[jj * kTS + c] = s;
    }
    __syncthreads();
    }
    // ---- W2 = T^T W (Q^T) or T W (Q); T upper triangular (Tt[r][c] = T[r][c])
    // thread (column c, rows jj = 4 jg + q): its 4 T entries per k are one
    // 16-byte load (Q^T); unrolled, T's zeros need no bounds
    T w2[4];
    {
        const int c = tid & 31, jg = tid >> 5;
#pragma unroll
        for (int q = 0; q < 4; ++q) w2[q] = T(0);
#pragma unroll
        for (int h = 0; h < 32; h += 8) {
            T wc[8];
#pragma unroll
            for (int k2 = 0; k2 < 8; ++k2) wc[k2] = W[(h + k2) * kTS + c];
            if (trans) {
#pragma unroll
                for (int k2 = 0; k2 < 8; ++k2) {
                    T tq[4];
#pragma unroll
                    for (int hh = 0; hh < 4 / VN; ++hh) {
                        const V4 t4 = *reinterpret_cast<const V4*>(Tt + (h + k2) * kTS + 4 * jg + hh * VN);
#pragma unroll
                        for (int e = 0; e < VN; ++e) tq[hh * VN + e] = vget<T>(t4, e);
                    }
#pragma unroll
                    for (int q = 0; q < 4; ++q) w2[q] = fma(tq[q], wc[k2], w2[q]);
                }
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int jj = 4 * jg + q;
                    T acc = T(0);
#pragma unroll
                    for (int k2 = 0; k2 < 8; ++k2) acc = fma(Tt[jj * kTS + h + k2], wc[k2], acc);
                    w2[q] += acc;
                }
            }
        }
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < 4; ++q) W[(4 * (tid >> 5) + q) * kTS + (tid & 31)] = w2[q];
    __syncthreads();

    if constexpr (MMA) {
        gemm2_mma<false>(Grp{tid, 0}, Vs, Cs, W, RGP, R32);
        __syncthreads();
        for (int c = warp; c < ncb; c += kWarps) {
            T* ccol = C + (cb0 + c) * ldc;
            const T* cs = Cs + (size_t)c * RGP;
            if (vec_p) {  // rows 4q..4q+3: one segment, 16-byte aligned
                for (int r = 4 * lane; r < RG; r += 128) {
                    if (r + 4 <= RG)
                        *reinterpret_cast<float4*>(reinterpret_cast<float*>(ccol) + gathered_row(nr, r)) =
                            *reinterpret_cast<const float4*>(reinterpret_cast<const float*>(cs) + r);
                    else
                        for (int q = r; q < RG; ++q) ccol[gathered_row(nr, q)] = cs[q];
                }
            } else {
                for (int r = lane; r < RG; r += 32) ccol[gathered_row(nr, r)] = cs[r];
            }
        }
    } else {
    // ---- C -= V W2 : thread = (4 consecutive rows, 8 consecutive columns) ---
    const int nq = R32 / 4;
    for (int u = tid; u < nq * 4; u += kThreads) {
        const int q = u % nq, cgrp = u / nq;
        const int r = 4 * q, cbase = 8 * cgrp;
        T acc[4][8];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int c = 0; c < 8; ++c) acc[i][c] = Cs[(size_t)(cbase + c) * RGP + r + i];
        for (int jj = 0; jj < wp; ++jj) {
            T vr[4];
#pragma unroll
            for (int h = 0; h < 4 / VN; ++h) {
                const V4 t4 = *reinterpret_cast<const V4*>(Vs + (size_t)jj * RGP + r + h * VN);
#pragma unroll
                for (int q = 0; q < VN; ++q) vr[h * VN + q] = vget<T>(t4, q);
            }
#pragma unroll
            for (int c = 0; c < 8; ++c) {
                const T wv = W[jj * kTS + cbase + c];
#pragma unroll
                for (int i = 0; i < 4; ++i) acc[i][c] = fma(-vr[i], wv, acc[i][c]);
            }
        }
        const bool v4 = sizeof(T) == 4 && vec_p && r + 4 <= RG;  // rows r..r+3: one segment, 16-byte aligned
#pragma unroll
        for (int c = 0; c < 8; ++c) {
            if (cbase + c >= ncb) break;
            T* ccol = C + (cb0 + cbase + c) * ldc;
            if constexpr (sizeof(T) == 4) {
                if (v4) {
                    *reinterpret_cast<float4*>(ccol + gathered_row(nr, r)) =
                        make_float4(acc[0][c], acc[1][c], acc[2][c], acc[3][c]);
                    continue;
                }
            }
#pragma unroll
            for (int i = 0; i < 4; ++i)
                if (r + i < RG) ccol[gathered_row(nr, r + i)] = acc[i][c];
        }
    }
    }
    }  // column blocks of this CTA
}

template <typename T, bool MMA = false>
__global__ void __launch_bounds__(kThreads)
panel_update_kernel(Geom g, const T* A, const T* __restrict__ Tws, int level, int p, int kt, T* C,
                    int64_t ldc, int64_t cfirst, int64_t ccount, int trans, int cpb) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int64_t nblk = (ccount + 31) / 32;
    const int64_t blk_beg = (int64_t)blockIdx.y * cpb, blk_end = min(nblk, blk_beg + cpb);
    update_node<T, MMA>(g, A, Tws, level, blockIdx.x, p, kt, C, ldc, cfirst, ccount, trans, blk_beg, blk_end,
                        smem_raw);
}

// Every step of node blockIdx.x in one launch.  level < 0: chain blockIdx.x --
// Q^T applies tile 0 (the leaf) .. K-1, each panel 0 .. npan-1 (the order of
// the factorization), Q the reverse; level >= 0: merge blockIdx.x of that tree
// level, all its panels.  The nodes of one level touch disjoint rows, so no two
// CTAs ever need each other's results: one launch per tree level (plus one for
// all chains) instead of one per (level or tile, panel).
template <typename T, bool MMA = false>
__global__ void __launch_bounds__(kThreads)
node_update_kernel(Geom g, const T* A, const T* __restrict__ Tws, int level, T* C, int64_t ldc, int64_t cfirst,
                   int64_t ccount, int trans, int cpb) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int64_t node = blockIdx.x;
    const int ntile = level < 0 ? (int)min(g.K, g.L - node * g.K) : 1;
    const int64_t nblk = (ccount + 31) / 32;
    const int64_t blk_beg = (int64_t)blockIdx.y * cpb, blk_end = min(nblk, blk_beg + cpb);
    const int steps = ntile * g.npan;
    for (int s = 0; s < steps; ++s) {
        const int kt = trans ? s / g.npan : ntile - 1 - s / g.npan;
        const int p = trans ? s % g.npan : g.npan - 1 - s % g.npan;
        update_node<T, MMA>(g, A, Tws, level, node, p, kt, C, ldc, cfirst, ccount, trans, blk_beg, blk_end,
                            smem_raw);
    }
}

// Q^T C / Q C of a whole group in ONE launch (the device
// steps through the tree levels instead of the host, cf. the early start of
// P:L356-360).  The phases -- the chains (level -1) and the tree levels, in
// execution order (bottom-up for Q^T, top-down for Q) -- are cut into tasks
// (node, group of 32-column blocks) exactly as node_update_kernel's grid;
// a cooperative grid of resident CTAs strides over each phase's tasks and
// meets at a grid barrier between phases (no scratch memory: the apply calls
// take the workspace read-only).  Each node runs the same update_node calls
// in the same order as the per-level launches: the results are bitwise equal
// (tests/test_gpu_parity.py).
constexpr int kMaxApplyPhases = 40;
struct ApplyPhases {
    int n;                          // phases
    int level[kMaxApplyPhases];     // -1: the chains
    int nodes[kMaxApplyPhases];     // nodes of the phase
    int cpb[kMaxApplyPhases];       // 32-column blocks per task
    int start[kMaxApplyPhases + 1]; // first task of each phase (prefix sums)
};

template <typename T>
__global__ void __launch_bounds__(kThreads, sizeof(T) == 4 ? 2 : 1)  // fp32: node_update_kernel's 2 CTAs/SM
node_update_all_kernel(Geom g, const T* A, const T* __restrict__ Tws, T* C, int64_t ldc, int64_t cfirst,
                       int64_t ccount, int trans, ApplyPhases ph) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    cooperative_groups::grid_group grid = cooperative_groups::this_grid();
    const int64_t nblk = (ccount + 31) / 32;
    for (int q = 0; q < ph.n; ++q) {
        if (q > 0) grid.sync();  // phase q-1 done everywhere (and its C stores visible)
        const int level = ph.level[q];
        const int ntask = ph.start[q + 1] - ph.start[q];
        for (int local = blockIdx.x; local < ntask; local += gridDim.x) {
            const int64_t node = local % ph.nodes[q];
            const int64_t blk_beg = (int64_t)(local / ph.nodes[q]) * ph.cpb[q];
            const int64_t blk_end = min(nblk, blk_beg + ph.cpb[q]);
            const int ntile = level < 0 ? (int)min(g.K, g.L - node * g.K) : 1;
            const int steps = ntile * g.npan;
            for (int s = 0; s < steps; ++s) {
                const int kt = trans ? s / g.npan : ntile - 1 - s / g.npan;
                const int p = trans ? s % g.npan : g.npan - 1 - s % g.npan;
                update_node<T, false>(g, A, Tws, level, node, p, kt, C, ldc, cfirst, ccount, trans, blk_beg,
                                      blk_end, smem_raw);
            }
        }
    }
}

template <typename T>
inline size_t panel_update_smem(int RGmax) {
    return sizeof(T) * (64 * (size_t)smem_col_stride<T>(RGmax) + 6 * 32 * kTS);
}

// R (n x n, ldr) <- triu(A[0:n, 0:n]).
template <typename T>
__global__ void extract_r_kernel(int64_t n, const T* __restrict__ A, int64_t lda,
                                 T* __restrict__ R, int64_t ldr) {
    const int64_t c = blockIdx.y;
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n;
         r += (int64_t)gridDim.x * blockDim.x)
        R[c * ldr + r] = r <= c ? A[c * lda + r] : T(0);
}

// Q (m x n, ldq) <- [I_n; 0].
template <typename T>
__global__ void set_identity_kernel(int64_t m, int64_t n, T* __restrict__ Q, int64_t ldq) {
    const int64_t c = blockIdx.y;
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < m;
         r += (int64_t)gridDim.x * blockDim.x)
        Q[c * ldq + r] = r == c ? T(1) : T(0);
}

}  // namespace caqr
