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

// Padded column layout of shared tiles: 16 bytes of padding after every 32
// rows, so that threads owning different 32-row segments of a column (and
// 16-byte vector loads of 8 different columns) hit disjoint bank groups.
template <typename T>
__host__ __device__ __forceinline__ int padr(int r) {
    return r + (r >> 5) * int(16 / sizeof(T));
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

// ---------------------------------------------------------------------------
// Factor the staged panel P (RG x wp, padded column layout) in registers.
// Thread t owns column c = t / TPC and rows [s*SEG, s*SEG+SEG), s = t % TPC.
// On exit: P holds the stored form (R on/above the diagonal, v below) and
// tau_s[0..wp) the reflector scalars.
// ---------------------------------------------------------------------------
template <typename T, int TPC>
__device__ __forceinline__ void factor_panel_regs(T* P, int RGP, int RG, int wp, T* tau_s) {
    constexpr int SEG = kFusedMaxRows / TPC;
    static_assert(SEG % 4 == 0, "SEG");
    using V4 = typename Vec4<T>::type;
    constexpr int VN = Vec4<T>::n;
    const int t = threadIdx.x;
    const int c = t / TPC, s = t % TPC, r0 = s * SEG;
    const int lane = t & 31;
    const unsigned gmask = TPC == 32 ? 0xffffffffu : (((1u << TPC) - 1u) << (lane & ~(TPC - 1)));
    const bool active = c < wp;
    T x[SEG];
    {
        const T* pc = P + (size_t)min(c, 31) * RGP + padr<T>(r0);
#pragma unroll
        for (int i = 0; i < SEG; i += VN) {
            const V4 q = *reinterpret_cast<const V4*>(pc + i);
#pragma unroll
            for (int k = 0; k < VN; ++k) x[i + k] = (active && r0 + i + k < RG) ? vget<T>(q, k) : T(0);
        }
    }
    __syncthreads();  // everyone has its registers before P is overwritten with v's

    // Reflector of column j by its owner group (xLARFG, reading S1).  Writes the
    // v column (unit head, zeros above) into P[:, j] for the other groups.
    auto reflector = [&](int j) {
        T sig = T(0), al = T(0);
#pragma unroll
        for (int i = 0; i < SEG; ++i) {
            const int r = r0 + i;
            sig = (r > j) ? fma(x[i], x[i], sig) : sig;
            al = (r == j) ? x[i] : al;
        }
        sig = group_sum<TPC>(sig, gmask);
        al = group_sum<TPC>(al, gmask);
        T tau = T(0), beta = al, scale = T(0);
        if (j < RG && sig != T(0)) {
            const T mu = sqrt(fma(al, al, sig));
            beta = -copysign(mu, al);
            tau = (beta - al) / beta;
            scale = T(1) / (al - beta);
        }
        T* pj = P + (size_t)j * RGP + padr<T>(r0);
#pragma unroll
        for (int i = 0; i < SEG; i += VN) {
            V4 q;
            T* qq = reinterpret_cast<T*>(&q);
#pragma unroll
            for (int k = 0; k < VN; ++k) {
                const int r = r0 + i + k;
                if (r > j) x[i + k] = (tau != T(0)) ? x[i + k] * scale : x[i + k];
                if (r == j) x[i + k] = beta;
                qq[k] = r > j ? x[i + k] : (r == j ? T(1) : T(0));
            }
            *reinterpret_cast<V4*>(pj + i) = q;
        }
        if (s == 0) tau_s[j] = tau;
    };

    if (c == 0) reflector(0);
    __syncthreads();
    for (int j = 0; j < wp; ++j) {
        const T tau = tau_s[j];
        if (active && c > j) {
            if (tau != T(0)) {
                const T* pj = P + (size_t)j * RGP + padr<T>(r0);
                T d0 = 0, d1 = 0, d2 = 0, d3 = 0;
#pragma unroll
                for (int i = 0; i < SEG; i += 4) {
                    T v4[4];
#pragma unroll
                    for (int h = 0; h < 4 / VN; ++h) {
                        const V4 q = *reinterpret_cast<const V4*>(pj + i + h * VN);
#pragma unroll
                        for (int k = 0; k < VN; ++k) v4[h * VN + k] = vget<T>(q, k);
                    }
                    d0 = fma(v4[0], x[i + 0], d0);
                    d1 = fma(v4[1], x[i + 1], d1);
                    d2 = fma(v4[2], x[i + 2], d2);
                    d3 = fma(v4[3], x[i + 3], d3);
                }
                T d = group_sum<TPC>((d0 + d1) + (d2 + d3), gmask);
                const T st = tau * d;
#pragma unroll
                for (int i = 0; i < SEG; i += VN) {
                    const V4 q = *reinterpret_cast<const V4*>(pj + i);
#pragma unroll
                    for (int k = 0; k < VN; ++k) x[i + k] = fma(-st, vget<T>(q, k), x[i + k]);
                }
            }
            if (c == j + 1) reflector(j + 1);
        }
        __syncthreads();
    }
    // stored form back into P (R on/above the diagonal, v below)
    if (active) {
        T* pc = P + (size_t)c * RGP + padr<T>(r0);
#pragma unroll
        for (int i = 0; i < SEG; i += VN) {
            V4 q;
            T* qq = reinterpret_cast<T*>(&q);
#pragma unroll
            for (int k = 0; k < VN; ++k) qq[k] = x[i + k];
            *reinterpret_cast<V4*>(pc + i) = q;
        }
    }
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

// T (upper triangular, Tt[r*kTS+c] = T[r][c]) from G = V^T V (in G) and tau
// (xLARFT forward/columnwise): T[j][j] = tau_j, T[0:j,j] = -tau_j T[0:j,0:j] G[0:j,j].
// One warp; lane i keeps row i of T in registers.
template <typename T>
__device__ __forceinline__ void build_t(const T* G, const T* tau_s, int wp, T* Tt) {
    const int lane = threadIdx.x & 31;
    if (threadIdx.x >= 32) return;
    T row[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) {
        T tj = T(0);
        if (j < wp) {
            T a0 = 0, a1 = 0;
#pragma unroll
            for (int k = 0; k < j; k += 2) {
                a0 = fma(row[k], G[k * kTS + j], a0);
                if (k + 1 < j) a1 = fma(row[k + 1], G[(k + 1) * kTS + j], a1);
            }
            const T tau = tau_s[j];
            tj = (j == lane) ? tau : (j > lane ? -tau * (a0 + a1) : T(0));
        }
        row[j] = tj;
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
    T w2[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int e = tid + q * kThreads;
        const int jj = e >> 5, c = e & 31;
        T s = T(0);
        if (trans) {
            for (int k = 0; k <= jj; ++k) s = fma(Tt[k * kTS + jj], W[k * kTS + c], s);
        } else {
            for (int k = jj; k < 32; ++k) s = fma(Tt[jj * kTS + k], W[k * kTS + c], s);
        }
        w2[q] = s;
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int e = tid + q * kThreads;
        W[(e >> 5) * kTS + (e & 31)] = w2[q];
    }
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
#pragma unroll
            for (int c = 0; c < 8; ++c) {
                const T wv = W[jj * kTS + cbase + c];
#pragma unroll
                for (int i = 0; i < 4; ++i) acc[i][c] = fma(-vr[i], wv, acc[i][c]);
            }
        }
#pragma unroll
        for (int c = 0; c < 8; ++c) {
            if (cbase + c >= ncb) break;
            T* ccol = C + (cb0 + cbase + c) * ldc;
#pragma unroll
            for (int i = 0; i < 4; ++i)
                if (r + i < RG) ccol[gathered_row(nr, r + i)] = acc[i][c];
        }
    }
    __syncthreads();
}

// Stage gathered rows of 32 columns [col0, col0+ncol) of M into a padded tile
// (columns >= ncol and rows >= RG zero).  mask_panel: apply the merge-node
// structure masks of panel p (panel_entry_stored).
template <typename T>
__device__ __forceinline__ void stage_cols(T* S, int RGP, int R32, const T* M, int64_t ld, int64_t col0,
                                           int ncol, const NodeRows& nr, int RG, bool mask_panel, int p) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int jj = warp; jj < 32; jj += kWarps) {
        T* sc = S + (size_t)jj * RGP;
        const T* mc = M + (col0 + jj) * ld;
        for (int r = lane; r < R32; r += 32) {
            T v = T(0);
            if (jj < ncol && r < RG && (!mask_panel || panel_entry_stored(nr, r, jj, p)))
                v = ldcg(mc + gathered_row(nr, r));
            sc[padr<T>(r)] = v;
        }
    }
}

// ---------------------------------------------------------------------------
// The persistent dataflow TSQR kernel.
// ---------------------------------------------------------------------------
template <typename T>
__global__ void __launch_bounds__(kThreads, sizeof(T) == 4 ? 2 : 1)
tsqr_fused_kernel(Geom g, T* A, T* __restrict__ Tws, int* __restrict__ sync, int nlevels, int do_leaves) {
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
    const int64_t leaf_tasks = do_leaves ? g.L : 0;
    int64_t total = leaf_tasks;
    for (int l = 0; l < nlevels; ++l) {
        const int64_t h = int64_t(1) << l;
        total += (g.L - 1 >= h) ? (g.L - 1 - h) / (2 * h) + 1 : 0;
    }
    for (;;) {
        __syncthreads();
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
                const int64_t nm = (g.L - 1 >= h) ? (g.L - 1 - h) / (2 * h) + 1 : 0;
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
            ver_a = expected_version(slot_a, level, g.L, do_leaves);
            ver_b = expected_version(slot_b, level, g.L, do_leaves);
        }
        const int my_ver = level + 2;
        for (int p = 0; p < g.npan; ++p) {
            const int wp = min(kPW, g.ncols - 32 * p);
            if (level >= 0 && threadIdx.x == 0) {
                const int* fa = flags + slot_a * g.npan + p;
                const int* fb = flags + slot_b * g.npan + p;
                while (ld_acquire(fa) < ver_a) __nanosleep(64);
                while (ld_acquire(fb) < ver_b) __nanosleep(64);
            }
            __syncthreads();
            const NodeRows nr = node_rows(g, level, node, p, wp);
            const int RG = nr.n0 + nr.n1;
            const int R32 = (RG + 31) & ~31;
            const int64_t c0 = g.col0 + 32 * p;
            // ---- panel: stage, factor, store R/V, T ------------------------
            stage_cols(P, RGP, R32, A, g.lda, c0, wp, nr, RG, true, p);
            if (threadIdx.x < 32) tau_s[threadIdx.x] = T(0);
            __syncthreads();
            if (wp <= 8)
                factor_panel_regs<T, 32>(P, RGP, RG, wp, tau_s);
            else
                factor_panel_regs<T, 8>(P, RGP, RG, wp, tau_s);
            {
                const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
                for (int jj = warp; jj < wp; jj += kWarps) {
                    T* col = A + (c0 + jj) * g.lda;
                    T* pc = P + (size_t)jj * RGP;
                    for (int r = lane; r < R32; r += 32) {
                        const bool in = r < RG;
                        const T val = pc[padr<T>(r)];
                        if (in && panel_entry_stored(nr, r, jj, p)) col[gathered_row(nr, r)] = val;
                        // V form in place: unit head, zeros above, merge masks
                        T v = T(0);
                        if (in) {
                            if (!nr.merge)
                                v = r > jj ? val : (r == jj ? T(1) : T(0));
                            else if (r < nr.n0)
                                v = (r == jj) ? T(1) : T(0);
                            else
                                v = (r - nr.n0) <= 32 * p + jj ? val : T(0);
                        }
                        pc[padr<T>(r)] = v;
                    }
                }
                for (int jj = wp + warp; jj < 32; jj += kWarps) {
                    T* pc = P + (size_t)jj * RGP;
                    for (int r = lane; r < R32; r += 32) pc[padr<T>(r)] = T(0);
                }
            }
            __syncthreads();
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
            // ---- trailing columns of this node, 32 at a time -------------------
            const int64_t tfirst = c0 + 32, tend = g.col0 + g.ncols;
            for (int64_t cb0 = tfirst; cb0 < tend; cb0 += 32) {
                const int ncb = (int)(tend - cb0 < 32 ? tend - cb0 : 32);
                stage_cols(Cs, RGP, R32, static_cast<const T*>(A), g.lda, cb0, ncb, nr, RG, false, p);
                __syncthreads();
                gemm_vtc(P, Cs, RGP, R32, Wp, W);
                apply_block(P, Cs, Tt, W, RGP, R32, RG, wp, 1, nr, A, g.lda, cb0, ncb);
            }
            // ---- publish ----------------------------------------------------------
            __threadfence();
            __syncthreads();
            if (threadIdx.x == 0) st_release(flags + slot_a * g.npan + p, level < 0 ? 1 : my_ver);
        }
    }
}

}  // namespace caqr
