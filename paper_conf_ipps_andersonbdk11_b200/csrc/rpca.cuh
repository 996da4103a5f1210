// rpca.cuh -- the paper's application layer on the GPU:
// SVD of a tall-skinny matrix through its QR (Sec. VI.B) and the
// robust-PCA alternating-directions iteration built on it (P:L1089-1113,
// Sec. VI.C, Fig. 11).
//
//   * jacobi_svd_kernel: SVD of the small n x n factor R.  The paper does this
//     on the CPU with MKL; here one CTA does a one-sided
//     (Hestenes) Jacobi SVD in fp64 in shared memory: columns of B = R are
//     rotated pairwise (round-robin "circle" ordering, n/2 independent pairs per
//     round, one warp per pair) until every pair is orthogonal to a relative
//     tolerance; then sigma_j = ||b_j||, U = B diag(1/sigma), V = the product of
//     the rotations, sorted by descending sigma.
//   * svt_core_kernel: W = U diag(max(sigma - tau, 0)) V^T (the threshold of
//     Fig. 11); the low-rank iterate is then L = Q [W; 0] (caqr_apply_q).
//   * rpca_update_kernel: the shrinkage step and the dual update, fused with
//     forming the next SVT input (one pass over M, L, S, Y), plus per-block
//     partial sums of ||M - L - S||_F^2 reduced in a fixed order (deterministic).
#pragma once
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <cstdint>

namespace caqr {

constexpr int kSvdMaxN = 112;     // 2 n^2 doubles in shared memory (B and V); n/2 <= 64 half-warps
constexpr int kSvdThreads = 1024;
constexpr int kSvdRpl = (kSvdMaxN + 15) / 16;  // rows per lane of a half-warp
constexpr int kSvdLd = 16 * kSvdRpl;           // padded column length of B
constexpr int kRpcaBlocks = 1024;  // partial sums of the residual (fixed grid)

__device__ __forceinline__ double warp_sum_d(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Player at position k of round r of the circle method over np (even) players.
__device__ __forceinline__ int rr_player(int k, int r, int np) {
    return k == 0 ? 0 : ((k - 1 + r) % (np - 1)) + 1;
}

template <typename T>
__global__ void __launch_bounds__(kSvdThreads, 1)
jacobi_svd_kernel(int n, const T* __restrict__ R, int64_t ldr, T* __restrict__ U, int64_t ldu,
                  T* __restrict__ sigma, T* __restrict__ V, int64_t ldv, double tol, int max_sweeps) {
    const double tol2 = tol * tol;
    const bool want_v = V != nullptr;
    extern __shared__ __align__(16) double sm[];
    const int np = (n + 1) & ~1;  // an odd n gets a zero column (never rotated)
    // columns padded with zero rows to kSvdLd = 16 * kSvdRpl: the half-warp
    // loops need no bounds (a rotation keeps zero rows zero)
    double* B = sm;                          // [np][kSvdLd]  column j at B + j * kSvdLd
    double* Vs = B + (size_t)np * kSvdLd;    // [np][np]
    double* nrm = Vs + (size_t)np * np;  // [np]
    double* sig = nrm + np;              // [np]
    int* rank = reinterpret_cast<int*>(sig + np);  // [np]
    __shared__ int s_rot;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarp = blockDim.x >> 5;
    for (int e = tid; e < np * kSvdLd; e += blockDim.x) {
        const int j = e / kSvdLd, i = e % kSvdLd;
        B[e] = (j < n && i < n) ? (double)R[(int64_t)j * ldr + i] : 0.0;
    }
    if (want_v)
        for (int e = tid; e < np * np; e += blockDim.x) Vs[e] = (e / np == e % np) ? 1.0 : 0.0;
    __syncthreads();
    for (int sweep = 0; sweep < max_sweeps; ++sweep) {
        // exact squared column norms at the start of every sweep
        for (int j = warp; j < np; j += nwarp) {
            double a = 0.0;
            for (int i = lane; i < n; i += 32) a = fma(B[j * kSvdLd + i], B[j * kSvdLd + i], a);
            a = warp_sum_d(a);
            if (lane == 0) nrm[j] = a;
        }
        if (tid == 0) s_rot = 0;
        __syncthreads();
        // one HALF-warp per pair: all n/2 pairs of a round at once (32 warps)
        const int hl = lane & 15, hw = 2 * warp + (lane >> 4);
        const unsigned hmask = (lane >> 4) ? 0xffff0000u : 0x0000ffffu;
        // (n <= 112: np/2 <= 56 pairs <= 64 half-warps, so each has at most one;
        // its two players advance by the circle method: x -> x + 1, np-1 -> 1)
        int pa = rr_player(hw, 0, np), pb = rr_player(np - 1 - hw, 0, np);
        for (int r = 0; r < np - 1; ++r, pa = pa == 0 ? 0 : (pa == np - 1 ? 1 : pa + 1),
                 pb = pb == np - 1 ? 1 : pb + 1) {
            if (hw < np / 2) {
                const int p = min(pa, pb), q = max(pa, pb);
                double* bp = B + p * kSvdLd + hl;
                double* bq = B + q * kSvdLd + hl;
                // (rows hl + 16 t, t < 7: fully unrolled, every load issued up front)
                double xp[kSvdRpl], xq[kSvdRpl];
#pragma unroll
                for (int t = 0; t < kSvdRpl; ++t) {
                    xp[t] = bp[16 * t];
                    xq[t] = bq[16 * t];
                }
                double g = 0.0, g1 = 0.0;
#pragma unroll
                for (int t = 0; t < kSvdRpl; t += 2) {
                    g = fma(xp[t], xq[t], g);
                    if (t + 1 < kSvdRpl) g1 = fma(xp[t + 1], xq[t + 1], g1);
                }
                g += g1;
#pragma unroll
                for (int o = 8; o > 0; o >>= 1) g += __shfl_xor_sync(hmask, g, o);
                const double al = nrm[p], be = nrm[q];
                __syncwarp(hmask);  // every lane has read nrm before lane 0 rewrites it
                if (g * g > tol2 * (al * be) && g != 0.0) {
                    // rotate so that b_p' . b_q' = 0 (cot 2 theta = (be - al) / (2 g)):
                    // t = tan theta = 2 g sign(d) / (|d| + sqrt(d^2 + 4 g^2)), d = be - al
                    // The angle only steers convergence; the rotation applied is
                    // exactly orthogonal whatever t is (c, s from t in fp64), so t
                    // comes from fast fp32 arithmetic.
                    const float df = (float)(be - al), gf = (float)g;
                    const float tf = (df < 0.f ? -2.f * gf : 2.f * gf) *
                                     __frcp_rn(fabsf(df) + sqrtf(fmaf(df, df, 4.f * gf * gf)));
                    const double t = (double)tf;
                    const double c = rsqrt(fma(t, t, 1.0)), s = c * t;
#pragma unroll
                    for (int t = 0; t < kSvdRpl; ++t) {
                        bp[16 * t] = c * xp[t] - s * xq[t];
                        bq[16 * t] = s * xp[t] + c * xq[t];
                    }
                    if (want_v) {
                        double* vp = Vs + (size_t)p * np;
                        double* vq = Vs + (size_t)q * np;
                        for (int i = hl; i < np; i += 16) {
                            const double x = vp[i], y = vq[i];
                            vp[i] = c * x - s * y;
                            vq[i] = s * x + c * y;
                        }
                    }
                    if (hl == 0) {
                        nrm[p] = al - t * g;
                        nrm[q] = be + t * g;
                        s_rot = 1;
                    }
                }
            }
            __syncthreads();
        }
        const int rot = s_rot;
        __syncthreads();
        if (!rot) break;
    }
    // sigma_j = ||b_j|| (exact), descending order (ties by index)
    for (int j = warp; j < np; j += nwarp) {
        double a = 0.0;
        for (int i = lane; i < n; i += 32) a = fma(B[j * kSvdLd + i], B[j * kSvdLd + i], a);
        a = warp_sum_d(a);
        if (lane == 0) sig[j] = sqrt(a);
    }
    __syncthreads();
    for (int j = tid; j < n; j += blockDim.x) {
        int rk = 0;
        for (int k = 0; k < n; ++k) rk += (sig[k] > sig[j]) || (sig[k] == sig[j] && k < j);
        rank[j] = rk;
    }
    __syncthreads();
    for (int e = tid; e < n * n; e += blockDim.x) {
        const int j = e / n, i = e % n, rk = rank[j];
        const double sj = sig[j];
        U[(int64_t)rk * ldu + i] = (T)(sj > 0.0 ? B[j * kSvdLd + i] / sj : 0.0);
        if (want_v) V[(int64_t)rk * ldv + i] = (T)Vs[(size_t)j * np + i];
        if (i == 0) sigma[rk] = (T)sj;
    }
}

template <typename T>
inline size_t jacobi_svd_smem(int n) {
    const size_t np = (size_t)((n + 1) & ~1);
    return sizeof(double) * (np * kSvdLd + np * np + 2 * np) + sizeof(int) * np;
}

// Block one-sided Jacobi (U, sigma only) over a CLUSTER of 8 CTAs.  The np <=
// 112 columns form 16 blocks of 7; CTA c holds the blocks at tournament
// positions c and 15 - c (round-robin "circle" ordering over the blocks) in its
// own shared memory.  A sweep: first the pairs inside every block (7 rounds,
// circle method on 7 + 1 idle), then 15 outer rounds in which each CTA rotates
// the 49 pairs ACROSS its two blocks (7 rounds of 7 disjoint pairs, one
// half-warp per pair, CTA barriers only) and moves both blocks to their next
// positions -- direct writes into the destination CTA's other buffer through
// distributed shared memory -- closed by one cluster barrier.  Every pair is
// visited once per sweep, as in the single-CTA kernel, but in 7 + 15 x 7
// cheap rounds on 8 SMs with 15 cluster barriers, instead of 99 rounds that
// each carry all n/2 pairs on one SM (measured: 0.63 vs 1.58 ms at n = 100).
constexpr int kSvdBlk = 7;     // columns per block
constexpr int kSvdNBlk = 16;   // blocks (np <= 112)
constexpr int kSvdCl = 8;      // CTAs per cluster (2 blocks each)
constexpr int kSvdClT = 128;   // 8 half-warps >= 7 pairs per inner round

template <typename T>
__global__ void __cluster_dims__(kSvdCl, 1, 1) __launch_bounds__(kSvdClT, 1)
jacobi_svd_block_kernel(int n, const T* __restrict__ R, int64_t ldr, T* __restrict__ U, int64_t ldu,
                        T* __restrict__ sigma, double tol, int max_sweeps) {
    namespace cg = cooperative_groups;
    cg::cluster_group cl = cg::this_cluster();
    const int crank = (int)cl.block_rank();
    constexpr int NL = 2 * kSvdBlk;  // local columns: block A = 0..6, block B = 7..13
    __shared__ __align__(16) double buf[2][NL][kSvdLd];  // [cur/next][local column][row]
    __shared__ int gidx[2][NL];                             // global index of each local column
    __shared__ double nrm2[2][NL];                          // squared column norms (travel with the blocks)
    __shared__ double sig0[kSvdNBlk * kSvdBlk];             // CTA 0: every sigma
    __shared__ int flag[2];                                 // CTA 0: "rotated in sweep s&1"
    __shared__ int s_rot;
    const double tol2 = tol * tol;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int hl = lane & 15, hw = 2 * warp + (lane >> 4);
    const unsigned hmask = (lane >> 4) ? 0xffff0000u : 0x0000ffffu;
    // initial blocks: position c holds block c, position 15 - c block 15 - c
    for (int e = tid; e < NL * kSvdLd; e += blockDim.x) {
        const int lc = e / kSvdLd, i = e % kSvdLd;
        const int blk = lc < kSvdBlk ? crank : kSvdNBlk - 1 - crank;
        const int j = blk * kSvdBlk + lc % kSvdBlk;
        buf[0][lc][i] = (j < n && i < n) ? (double)R[(int64_t)j * ldr + i] : 0.0;
        if (i == 0) gidx[0][lc] = j;
    }
    if (tid < 2) flag[tid] = 0;
    cl.sync();
    int cur = 0;
    auto norms = [&]() {
        for (int lc = warp; lc < NL; lc += blockDim.x >> 5) {
            double a = 0.0;
            for (int i = lane; i < kSvdLd; i += 32) a = fma(buf[cur][lc][i], buf[cur][lc][i], a);
            a = warp_sum_d(a);
            if (lane == 0) nrm2[cur][lc] = a;
        }
    };
    // rotate local columns (p, q) so that they are orthogonal (half-warp hw)
    auto rotate = [&](int p, int q) {
        if (gidx[cur][p] > gidx[cur][q]) {  // the single-CTA kernel's convention: p < q globally
            const int t = p;
            p = q;
            q = t;
        }
        double* bp = &buf[cur][p][hl];
        double* bq = &buf[cur][q][hl];
        double xp[kSvdRpl], xq[kSvdRpl];
#pragma unroll
        for (int t = 0; t < kSvdRpl; ++t) {
            xp[t] = bp[16 * t];
            xq[t] = bq[16 * t];
        }
        double g = 0.0, g1 = 0.0;
#pragma unroll
        for (int t = 0; t < kSvdRpl; t += 2) {
            g = fma(xp[t], xq[t], g);
            if (t + 1 < kSvdRpl) g1 = fma(xp[t + 1], xq[t + 1], g1);
        }
        g += g1;
#pragma unroll
        for (int o = 8; o > 0; o >>= 1) g += __shfl_xor_sync(hmask, g, o);
        const double al = nrm2[cur][p], be = nrm2[cur][q];
        __syncwarp(hmask);
        if (g * g > tol2 * (al * be) && g != 0.0) {
            const float df = (float)(be - al), gf = (float)g;
            const float tf = (df < 0.f ? -2.f * gf : 2.f * gf) *
                             __frcp_rn(fabsf(df) + sqrtf(fmaf(df, df, 4.f * gf * gf)));
            const double t = (double)tf;
            const double c = rsqrt(fma(t, t, 1.0)), sn = c * t;
#pragma unroll
            for (int u = 0; u < kSvdRpl; ++u) {
                bp[16 * u] = c * xp[u] - sn * xq[u];
                bq[16 * u] = sn * xp[u] + c * xq[u];
            }
            if (hl == 0) {
                nrm2[cur][p] = al - t * g;
                nrm2[cur][q] = be + t * g;
                s_rot = 1;
            }
        }
    };
    for (int sweep = 0; sweep < max_sweeps; ++sweep) {
        int* flag0 = cl.map_shared_rank(&flag[sweep & 1], 0);
        // ---- pairs inside each block: circle method on 8 (7 + an idle one) --
        norms();
        if (tid == 0) s_rot = 0;
        __syncthreads();
        for (int ir = 0; ir < kSvdBlk; ++ir) {
            const int blk = hw >> 2, k = hw & 3;
            const int a = rr_player(k, ir, kSvdBlk + 1), b = rr_player(kSvdBlk - k, ir, kSvdBlk + 1);
            if (a < kSvdBlk && b < kSvdBlk) rotate(blk * kSvdBlk + a, blk * kSvdBlk + b);
            __syncthreads();
        }
        for (int r = 0; r < kSvdNBlk - 1; ++r) {
            // ---- pairs across the two blocks held: 7 rounds of 7 disjoint pairs
            for (int ir = 0; ir < kSvdBlk; ++ir) {
                if (hw < kSvdBlk) rotate(hw, kSvdBlk + (hw + ir) % kSvdBlk);
                __syncthreads();
            }
            if (tid == 0 && s_rot) *flag0 = 1;
            // ---- move both blocks to their next positions (DSMEM writes) ----
            const int nxt = cur ^ 1;
#pragma unroll
            for (int slot = 0; slot < 2; ++slot) {
                const int pos = slot == 0 ? crank : kSvdNBlk - 1 - crank;
                const int dpos = pos == 0 ? 0 : (pos == 1 ? kSvdNBlk - 1 : pos - 1);
                const int dcta = dpos < kSvdCl ? dpos : kSvdNBlk - 1 - dpos;
                const int dslot = dpos < kSvdCl ? 0 : 1;
                double2* dst = reinterpret_cast<double2*>(cl.map_shared_rank(&buf[nxt][dslot * kSvdBlk][0], dcta));
                const double2* src = reinterpret_cast<const double2*>(&buf[cur][slot * kSvdBlk][0]);
                for (int e = tid; e < kSvdBlk * kSvdLd / 2; e += blockDim.x) dst[e] = src[e];
                int* dg = cl.map_shared_rank(&gidx[nxt][dslot * kSvdBlk], dcta);
                if (tid < kSvdBlk) dg[tid] = gidx[cur][slot * kSvdBlk + tid];
                double* dn = cl.map_shared_rank(&nrm2[nxt][dslot * kSvdBlk], dcta);
                if (tid < kSvdBlk) dn[tid] = nrm2[cur][slot * kSvdBlk + tid];
            }
            cl.sync();
            cur = nxt;
            // (the previous sweep's flag has been read by every CTA: reset it)
            if (r == 0 && crank == 0 && tid == 0) flag[(sweep + 1) & 1] = 0;
        }
        const int rot = *flag0;
        if (!rot) break;
    }
    cl.sync();
    // sigma_j = ||b_j|| by the column's holder, gathered in CTA 0; ranks; U, sigma
    double* s0 = cl.map_shared_rank(&sig0[0], 0);
    for (int lc = warp; lc < NL; lc += blockDim.x >> 5) {
        double a = 0.0;
        for (int i = lane; i < kSvdLd; i += 32) a = fma(buf[cur][lc][i], buf[cur][lc][i], a);
        a = warp_sum_d(a);
        if (lane == 0) s0[gidx[cur][lc]] = sqrt(a);
    }
    cl.sync();
    for (int lc = warp; lc < NL; lc += blockDim.x >> 5) {
        const int j = gidx[cur][lc];
        if (j >= n) continue;
        const double sj = s0[j];
        int rk = 0;
        for (int q = lane; q < n; q += 32) {
            const double sq = s0[q];
            rk += (sq > sj) || (sq == sj && q < j);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) rk += __shfl_xor_sync(0xffffffffu, rk, o);
        for (int i = lane; i < n; i += 32) U[(int64_t)rk * ldu + i] = (T)(sj > 0.0 ? buf[cur][lc][i] / sj : 0.0);
        if (lane == 0) sigma[rk] = (T)sj;
    }
    cl.sync();  // no CTA exits while others may still read its shared memory
}

// W(n x n) = U diag(max(sigma - tau, 0)) V^T; one block per column k of W.
template <typename T>
__global__ void svt_core_kernel(int n, const T* __restrict__ U, int64_t ldu, const T* __restrict__ sigma,
                                const T* __restrict__ V, int64_t ldv, T tau, T* __restrict__ W, int64_t ldw) {
    const int k = blockIdx.x;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
        double acc = 0.0;
        for (int j = 0; j < n; ++j) {
            const double d = (double)sigma[j] - (double)tau;
            if (d > 0.0) acc = fma((double)U[(int64_t)j * ldu + i] * d, (double)V[(int64_t)j * ldv + k], acc);
        }
        W[(int64_t)k * ldw + i] = (T)acc;
    }
}

// W(n x n) = U diag(max(sigma - tau, 0) / sigma) U^T R  (== U diag(max(sigma - tau, 0)) V^T
// for R = U diag(sigma) V^T: U^T R = diag(sigma) V^T; no V needed, and only
// sigma_j > tau, hence no small sigma, is divided by).  One block per column k.
template <typename T>
__global__ void svt_core_r_kernel(int n, const T* __restrict__ U, int64_t ldu, const T* __restrict__ sigma,
                                  const T* __restrict__ R, int64_t ldr, T tau, T* __restrict__ W, int64_t ldw,
                                  const double* __restrict__ sched = nullptr) {
    __shared__ double pk[kSvdMaxN];
    if (sched) tau = (T)(1.0 / sched[0]);  // the iteration's 1/mu (device schedule)
    const int k = blockIdx.x;
    for (int j = threadIdx.x; j < n; j += blockDim.x) {  // pk_j = f(sigma_j) (U^T R)_jk
        const double sj = (double)sigma[j], d = sj - (double)tau;
        double acc = 0.0;
        if (d > 0.0) {
            for (int l = 0; l < n; ++l) acc = fma((double)U[(int64_t)j * ldu + l], (double)R[(int64_t)k * ldr + l], acc);
            acc *= d / sj;
        }
        pk[j] = acc;
    }
    __syncthreads();
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
        double acc = 0.0;
        for (int j = 0; j < n; ++j) acc = fma((double)U[(int64_t)j * ldu + i], pk[j], acc);
        W[(int64_t)k * ldw + i] = (T)acc;
    }
}

// C (m x n) = [W; 0], W n x n.
template <typename T>
__global__ void embed_top_kernel(int64_t m, int64_t n, const T* __restrict__ W, int64_t ldw, T* __restrict__ C,
                                 int64_t ldc) {
    const int64_t total = m * n;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = e / m, i = e % m;
        C[j * ldc + i] = i < n ? W[j * ldw + i] : T(0);
    }
}

__device__ __forceinline__ double block_sum_d(double v, double* scr) {
    v = warp_sum_d(v);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (lane == 0) scr[warp] = v;
    __syncthreads();
    double t = 0.0;
    if (threadIdx.x == 0)
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += scr[w];
    return t;
}

// Elementwise over m x n ([19]):
//   S <- shrink(M - L + Y/mu, lambda/mu);  Y <- Y + mu (M - L - S);
//   X <- M - S + Y/mu_next  (the next SVT input);  part[b] = sum (M - L - S)^2.
template <typename T>
__global__ void __launch_bounds__(256) rpca_update_kernel(int64_t m, int64_t n, const T* __restrict__ M, int64_t ldm,
                                                          const T* __restrict__ L, int64_t ldl, T* __restrict__ S,
                                                          int64_t lds, T* __restrict__ Y, int64_t ldy,
                                                          T* __restrict__ X, int64_t ldx, T mu, T mu_next,
                                                          T lambda, double* __restrict__ part,
                                                          const double* __restrict__ sched = nullptr) {
    __shared__ double scr[8];
    if (sched) {  // device schedule: mu, mu_next = min(rho mu, mu_max), lambda
        mu = (T)sched[0];
        mu_next = (T)fmin(sched[2] * sched[0], sched[1]);
        lambda = (T)sched[4];
    }
    const T imu = T(1) / mu, imu_next = T(1) / mu_next, thr = lambda / mu;
    double acc = 0.0;
    const int64_t total = m * n;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = e / m, i = e % m;
        const T mv = M[j * ldm + i], lv = L[j * ldl + i], yv = Y[j * ldy + i];
        const T t = mv - lv + yv * imu;
        const T a = fabs(t) - thr;
        const T sv = a > T(0) ? copysign(a, t) : T(0);
        const T z = mv - lv - sv;
        const T yn = yv + mu * z;
        S[j * lds + i] = sv;
        Y[j * ldy + i] = yn;
        X[j * ldx + i] = mv - sv + yn * imu_next;
        acc = fma((double)z, (double)z, acc);
    }
    const double b = block_sum_d(acc, scr);
    if (threadIdx.x == 0) part[1 + blockIdx.x] = b;
}

// part[0] = sum of part[1..nb] in index order (deterministic).
// With a device schedule it also advances mu <- min(rho mu, mu_max) (this
// kernel runs after the update kernel that read mu, on the same stream).
__global__ void sum_parts_kernel(int nb, double* part, double* sched = nullptr) {
    __shared__ double scr[32];
    double a = 0.0;
    // fixed assignment of parts to threads and a fixed tree: deterministic
    for (int b = threadIdx.x; b < nb; b += blockDim.x) a += part[1 + b];
    const double t = block_sum_d(a, scr);
    if (threadIdx.x == 0) {
        part[0] = t;
        if (sched) sched[0] = fmin(sched[2] * sched[0], sched[1]);
    }
}

// Device schedule of the iteration (reading S19): from ||M||_2 = sigma[0] and
// ||M||_inf = amax[0]: mu0 = mu_factor / ||M||_2, mu_max = mu_max_factor mu0,
// rho, yscale = 1 / max(||M||_2, ||M||_inf / lambda), lambda -- in double.
__global__ void rpca_schedule_kernel(const float* __restrict__ sigma, const float* __restrict__ amax, double lambda,
                                     double mu_factor, double mu_max_factor, double rho, double* sched) {
    if (threadIdx.x != 0) return;
    const double norm2 = (double)sigma[0], norminf = (double)amax[0];
    const double J = fmax(norm2, norminf / lambda);
    const double mu = mu_factor / norm2;
    sched[0] = mu;
    sched[1] = mu * mu_max_factor;
    sched[2] = rho;
    sched[3] = 1.0 / J;
    sched[4] = lambda;
}

// Start of the iteration: S = 0, Y = yscale M, X = M + Y / mu.
template <typename T>
__global__ void rpca_init_kernel(int64_t m, int64_t n, const T* __restrict__ M, int64_t ldm, T yscale,
                                 T* __restrict__ S, int64_t lds, T* __restrict__ Y, int64_t ldy, T* __restrict__ X,
                                 int64_t ldx, T mu, const double* __restrict__ sched = nullptr) {
    if (sched) {
        yscale = (T)sched[3];
        mu = (T)sched[0];
    }
    const int64_t total = m * n;
    const T imu = T(1) / mu;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = e / m, i = e % m;
        const T mv = M[j * ldm + i];
        const T yv = yscale * mv;
        S[j * lds + i] = T(0);
        Y[j * ldy + i] = yv;
        X[j * ldx + i] = mv + yv * imu;
    }
}

// out[0] = max |M_ij| (as the bits of a non-negative float: integer max is
// order-independent, so the result is deterministic).
template <typename T>
__global__ void absmax_kernel(int64_t m, int64_t n, const T* __restrict__ M, int64_t ldm, T* out) {
    __shared__ T scr[32];
    T a = T(0);
    const int64_t total = m * n;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = e / m, i = e % m;
        a = fmax(a, fabs(M[j * ldm + i]));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) a = fmax(a, __shfl_xor_sync(0xffffffffu, a, o));
    if ((threadIdx.x & 31) == 0) scr[threadIdx.x >> 5] = a;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < (int)(blockDim.x >> 5); ++w) a = fmax(a, scr[w]);
        if constexpr (sizeof(T) == 4)
            atomicMax(reinterpret_cast<unsigned int*>(out), __float_as_uint(a));
        else
            atomicMax(reinterpret_cast<unsigned long long*>(out), (unsigned long long)__double_as_longlong(a));
    }
}


// X = R^{-1} B in place (R n x n upper triangular, B n x k), one CTA per
// column of B: column-oriented back substitution with b in shared memory --
// x_i = b_i / R_ii, then b_j -= R_ji x_i for j < i (coalesced over j).  The
// triangular solve of least squares through QR (xGELS: x = R^{-1} (Q^T b)[0:n],
// P:L86-92).
template <typename T>
__global__ void __launch_bounds__(256) trsm_upper_kernel(int64_t n, const T* __restrict__ R, int64_t ldr, T* B,
                                                         int64_t ldb) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* b = reinterpret_cast<T*>(smem_raw);
    __shared__ T s_x;
    T* col = B + (int64_t)blockIdx.x * ldb;
    for (int64_t j = threadIdx.x; j < n; j += blockDim.x) b[j] = col[j];
    __syncthreads();
    for (int64_t i = n - 1; i >= 0; --i) {
        if (threadIdx.x == 0) {
            const T xi = b[i] / R[i * ldr + i];
            b[i] = xi;
            s_x = xi;
        }
        __syncthreads();
        const T xi = s_x;
        const T* ri = R + i * ldr;
        for (int64_t j = threadIdx.x; j < i; j += blockDim.x) b[j] -= ri[j] * xi;
        __syncthreads();
    }
    for (int64_t j = threadIdx.x; j < n; j += blockDim.x) col[j] = b[j];
}

}  // namespace caqr
