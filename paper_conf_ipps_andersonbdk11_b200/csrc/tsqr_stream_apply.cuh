// tsqr_stream_apply.cuh -- Q^T C and Q C over the chains of a skinny plan
// (n <= 16, fp32, the streaming kernel's 256/128-row tiles), one WARP per chain.
//
// The replay of the factorization's leaf level ("apply_qt_h", and
// its transpose for Q, SORGQR P:L905-910) on the same chains of tiles: the
// chain's first tile is a leaf with V unit lower-trapezoidal, every later tile
// a structured step whose V is [I (the chain's R-slot rows); dense tile].  For
// k <= KC columns of C a warp keeps the chain's slot rows of C in registers
// (lane j holds slot row j), streams the tiles of V and C through registers
// (lane l holds rows l + 32 i) and applies each compact-WY step
//     W = V^T [C_slot; C_tile]  (one NC x KC warp all-reduce),
//     W <- T^T W (Q^T) or T W (Q),  C_slot -= W,  C_tile -= V_tile W,
// so every element of A and C crosses HBM once per apply -- the bound is HBM
// (read V, read + write C).  The tree levels run after (Q^T) or before (Q) as
// node_update launches.
#pragma once
#include "tsqr_stream.cuh"

namespace caqr {

constexpr int kStreamApplyWarps = 8;

template <int NC, int KC, int RPL>
__global__ void __launch_bounds__(32 * kStreamApplyWarps, 1)
stream_apply_chain_kernel(Geom g, const float* __restrict__ A, const float* __restrict__ Tws, float* C,
                          int64_t ldc, int k, int trans) {
    constexpr int NR = NC * KC;  // sums per step, reduced 32 at a time
    static_assert(NR % 32 == 0 && NR <= 256, "NC * KC: a multiple of 32, <= 256");
    __shared__ float s_red[kStreamApplyWarps][32 + 4];
    __shared__ float s_T[kStreamApplyWarps][NC][NC + 1];
    __shared__ float s_W[kStreamApplyWarps][NC][KC + 1];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t chain = (int64_t)blockIdx.x * kStreamApplyWarps + warp;
    if (chain >= g.P) return;  // warp-uniform
    const int wp = g.ncols;
    const int64_t t0 = chain * g.K;
    const int ntile = (int)min64(g.K, g.L - t0);
    const int64_t slot0 = g.row0 + t0 * g.b;                  // the chain's slot rows = its first tile's top
    const int hs = (int)min64(NC, g.mrows - t0 * g.b);        // rows of the slot (a short last chain)
    float cs[KC];  // lane j < NC: row j of the chain's slot rows of C
#pragma unroll
    for (int cc = 0; cc < KC; ++cc)
        cs[cc] = (!trans && lane < hs && cc < k) ? C[(int64_t)cc * ldc + slot0 + lane] : 0.f;
    for (int st = 0; st < ntile; ++st) {
        const int kt = trans ? st : ntile - 1 - st;
        const int64_t t = t0 + kt;
        const int64_t srow = g.row0 + t * g.b;
        const int h = (int)min64(g.b, g.mrows - t * g.b);
        float v[NC][RPL], c[KC][RPL];
#pragma unroll
        for (int i = 0; i < RPL; ++i) {
            const int r = lane + 32 * i;
            const bool in = r < h;
#pragma unroll
            for (int j = 0; j < NC; ++j) {
                const float raw = (in && j < wp) ? __ldcg(A + (g.col0 + j) * g.lda + srow + r) : 0.f;
                v[j][i] = kt == 0 ? (r > j ? raw : (r == j && j < wp ? 1.f : 0.f)) : raw;
            }
#pragma unroll
            for (int cc = 0; cc < KC; ++cc) c[cc][i] = (in && cc < k) ? __ldcg(C + cc * ldc + srow + r) : 0.f;
        }
        if (kt == 0 && !trans) {  // the leaf's top rows are the slot rows, current in cs
#pragma unroll
            for (int cc = 0; cc < KC; ++cc)
                if (lane < hs) c[cc][0] = cs[cc];
        }
        {   // T (wp x wp used) of this tile
            const float* tb = Tws + (t * g.npan) * (kPW * kPW);
            for (int e = lane; e < NC * NC; e += 32) {
                const int r = e % NC, cc = e / NC;
                s_T[warp][r][cc] = (r < wp && cc < wp) ? __ldcg(tb + cc * kPW + r) : 0.f;
            }
        }
        // W = V^T [C_slot; C_tile]: chain steps add the slot rows (V = I there);
        // 32 of the NC x KC sums per warp all-reduce, parked in shared memory
#pragma unroll
        for (int q = 0; q < NR / 32; ++q) {
            float part[32];
#pragma unroll
            for (int e = 0; e < 32; ++e) {
                const int j = (32 * q + e) / KC, cc = (32 * q + e) % KC;
                float a = (kt > 0 && lane == j) ? cs[cc] : 0.f;
#pragma unroll
                for (int i = 0; i < RPL; ++i) a = fmaf(v[j][i], c[cc][i], a);
                part[e] = a;
            }
            warp_allreduce<32>(part, &s_red[warp][0]);
            if (lane == 0)
#pragma unroll
                for (int e = 0; e < 32; ++e) s_W[warp][(32 * q + e) / KC][(32 * q + e) % KC] = part[e];
        }
        __syncwarp();
        // W2 = T^T W (Q^T) or T W (Q): lane j < NC computes row j
        float w2row[KC];
        if (lane < NC) {
#pragma unroll
            for (int cc = 0; cc < KC; ++cc) {
                float a = 0.f;
#pragma unroll
                for (int q = 0; q < NC; ++q)
                    a = fmaf(trans ? s_T[warp][q][lane] : s_T[warp][lane][q], s_W[warp][q][cc], a);
                w2row[cc] = a;
            }
        }
        __syncwarp();
        if (lane < NC)
#pragma unroll
            for (int cc = 0; cc < KC; ++cc) s_W[warp][lane][cc] = w2row[cc];
        __syncwarp();
        if (kt > 0 && lane < NC)
#pragma unroll
            for (int cc = 0; cc < KC; ++cc) cs[cc] -= w2row[cc];
#pragma unroll
        for (int cc = 0; cc < KC; ++cc)
#pragma unroll
            for (int j = 0; j < NC; ++j) {
                const float w = s_W[warp][j][cc];
#pragma unroll
                for (int i = 0; i < RPL; ++i) c[cc][i] = fmaf(-v[j][i], w, c[cc][i]);
            }
        if (kt == 0 && trans) {  // slot rows after the leaf: carried on in cs
#pragma unroll
            for (int cc = 0; cc < KC; ++cc)
                if (lane < hs) cs[cc] = c[cc][0];
        }
#pragma unroll
        for (int i = 0; i < RPL; ++i) {
            const int r = lane + 32 * i;
            if (r < h)
#pragma unroll
                for (int cc = 0; cc < KC; ++cc)
                    if (cc < k) C[cc * ldc + srow + r] = c[cc][i];
        }
        __syncwarp();  // s_T / s_W reused by the next step
    }
    if (trans) {  // the slot rows' final values (the leaf stored intermediate ones)
        __syncwarp();
#pragma unroll
        for (int cc = 0; cc < KC; ++cc)
            if (lane < hs && cc < k) C[(int64_t)cc * ldc + slot0 + lane] = cs[cc];
    }
}


// One tree level of Q^T C / Q C for a single-panel group of <= NC columns, one
// WARP per merge ("apply_qt_tree"): lane cc < k holds column cc of
// the C rows of both slots, V_2 (upper triangular, in R_b's slot) and T in
// shared memory;  W = C_a + V_2^T C_b,  W <- T^T W (Q^T) or T W (Q),
// C_a -= W,  C_b -= V_2 W.  k > 32 columns: the lanes loop over them.
template <int NC>
__global__ void __launch_bounds__(32 * kStreamApplyWarps)
stream_apply_tree_kernel(Geom g, const float* __restrict__ A, const float* __restrict__ Tws, float* C, int64_t ldc,
                         int64_t k, int level, int trans) {
    __shared__ float s_V[kStreamApplyWarps][NC][NC + 1];
    __shared__ float s_T[kStreamApplyWarps][NC][NC + 1];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t hl = int64_t(1) << level;
    const int64_t nm = (g.P - 1 >= hl) ? (g.P - 1 - hl) / (2 * hl) + 1 : 0;
    const int64_t node = (int64_t)blockIdx.x * kStreamApplyWarps + warp;
    if (node >= nm) return;  // warp-uniform
    const int wp = g.ncols;
    const int64_t a = node << (level + 1), b = a + hl;
    const int64_t ra = g.row0 + a * g.bm, rb = g.row0 + b * g.bm;
    const int nbr = (int)min64(min64(g.b, g.mrows - b * g.bm), wp);  // rows of R_b's slot
    const float* tb = Tws + ((g.L + b) * g.npan) * (kPW * kPW);
    for (int e = lane; e < NC * NC; e += 32) {
        const int i = e % NC, j = e / NC;
        s_V[warp][i][j] = (i <= j && i < nbr && j < wp) ? __ldcg(A + (g.col0 + j) * g.lda + rb + i) : 0.f;
        s_T[warp][i][j] = (i < wp && j < wp) ? __ldcg(tb + j * kPW + i) : 0.f;
    }
    __syncwarp();
    for (int64_t cc = lane; cc < k; cc += 32) {
        float ca[NC], cb[NC], w[NC];
        float* colp = C + cc * ldc;
#pragma unroll
        for (int j = 0; j < NC; ++j) {
            ca[j] = j < wp ? __ldcg(colp + ra + j) : 0.f;
            cb[j] = j < nbr ? __ldcg(colp + rb + j) : 0.f;
        }
#pragma unroll
        for (int j = 0; j < NC; ++j) {
            float acc = ca[j];
#pragma unroll
            for (int i = 0; i <= j; ++i) acc = fmaf(s_V[warp][i][j], cb[i], acc);
            w[j] = acc;
        }
        float w2[NC];
#pragma unroll
        for (int j = 0; j < NC; ++j) {
            float acc = 0.f;
#pragma unroll
            for (int q = 0; q < NC; ++q) acc = fmaf(trans ? s_T[warp][q][j] : s_T[warp][j][q], w[q], acc);
            w2[j] = acc;
        }
#pragma unroll
        for (int j = 0; j < NC; ++j)
            if (j < wp) colp[ra + j] = ca[j] - w2[j];
#pragma unroll
        for (int i = 0; i < NC; ++i) {
            float acc = cb[i];
#pragma unroll
            for (int j = i; j < NC; ++j) acc = fmaf(-s_V[warp][i][j], w2[j], acc);
            if (i < nbr) colp[rb + i] = acc;
        }
    }
}

}  // namespace caqr
