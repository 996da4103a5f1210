// tsqr_chain.cuh -- the chain phase of the whole-width TSQR (fp32), round 2.
//
// Every chain of K consecutive b-row tiles (a flat tree, "any tree shape",
// P:L339-341) is one task for one CTA of 32*NQ threads: the first tile is a
// leaf Householder QR ("factor"), every later tile the structured
// QR of [chain R; tile] (the tree step "factor_tree", with the
// chain's running R as the stacked upper triangle).  Per 32-column panel:
//
//  * factor: thread t owns column c = t / NQ of the panel and the contiguous
//    row segment q = t % NQ (SEG = b / NQ rows, in registers).  Reflector j
//    (xLARFG reading S1) is computed by column j's NQ threads (one shuffle
//    reduction of sigma), its v is broadcast through shared memory, and every
//    later column's threads form s = head + v^T x (one NQ-lane reduction) and
//    apply x -= tau s v: the matvec + rank-1 update of P:L704-711, one CTA
//    barrier per column.  The head row of reflector j is the chain's R row
//    32p + j (structured step: v = [e_j; v_tile]) or, in a leaf, the tile's own
//    row 32p + j (the leaf's 32 head rows of the panel live in shared memory).
//  * T (compact WY) is built DURING the factorization by the
//    threads whose columns are already done: at step j they form
//    G[c][j] = v_c^T v_j and, one step later, T[0:j,j] = -tau_j T G[0:j,j]
//    (xLARFT) -- off the reflector critical path.
//  * trailing update of the node's later columns (the horizontal update
//    P:L665-668 inside the node) in chunks of CW columns:
//    W = V^T C, W2 = T^T W, C -= V W2 on tensor cores (mma.sync m16n8k8 TF32,
//    3xTF32 split), the next panel's columns first so that they go straight
//    from shared memory into the factorization registers.
//
// The output is round 1's representation (Geom, node_rows): V in A, T blocks
// [L][npan][32][32] in the workspace, the chain R in the first tile's top n
// rows (its slot).  The binary tree over the P chain slots is the existing
// fused kernel in merge-only mode (do_leaves = 0).  Small CTAs (128 threads,
// ~60 KB shared memory) give 3 chains per SM instead of 2, and the per-column
// critical path carries no multi-value warp reductions.
#pragma once
#include "tsqr_fused.cuh"

namespace caqr {

template <int NQ, int SEG>
struct ChainCfg {
    static constexpr int NT = 32 * NQ;                 // threads
    static constexpr int NW = NT / 32;                 // warps
    static constexpr int B = NQ * SEG;                 // tile rows
    static constexpr int VP = B + 4;                   // column stride (floats): 16 bytes mod 128
    static constexpr int CW = 16;                      // trailing chunk width (columns)
    static constexpr int HS = 33;                      // stride of the 32 x 32 tiles
    static constexpr int WS = CW + 4;                  // stride of W / W2 (32 x CW)
    // shared memory (floats)
    static constexpr int OFF_V = 0;                    // Vs[32][VP]: the panel's V, tile rows
    static constexpr int OFF_C = OFF_V + 32 * VP;      // Cs[2][CW][VP]: C chunk, tile rows (double buffer)
    static constexpr int OFF_CS = OFF_C + 2 * CW * VP; // Csl[2][CW][32]: C chunk, slot rows 32p..
    static constexpr int OFF_H = OFF_CS + 2 * CW * 32; // Hh[32][HS] heads
    static constexpr int OFF_T = OFF_H + 32 * HS;      // Ts[32][HS]
    static constexpr int OFF_G = OFF_T + 32 * HS;      // Gs[32][HS]
    static constexpr int OFF_W = OFF_G + 32 * HS;      // Ws[32][WS]
    static constexpr int OFF_W2 = OFF_W + 32 * WS;     // W2s[32][WS]
    static constexpr int OFF_TAU = OFF_W2 + 32 * WS;   // taus[32]
    static constexpr int FLOATS = OFF_TAU + 32 + 4;
    static constexpr size_t BYTES = sizeof(float) * (size_t)FLOATS;
    static_assert(NQ == 4, "4 warps: one 16x8 output tile per warp in the small GEMMs");
    static_assert(SEG % 4 == 0 && B % 16 == 0, "SEG");
    static_assert((VP * 4) % 128 == 16, "VP");
};

// Group (NQ consecutive lanes) reduction.
template <int NQ>
__device__ __forceinline__ float qsum(float v, unsigned gm) {
#pragma unroll
    for (int o = 1; o < NQ; o <<= 1) v += __shfl_xor_sync(gm, v, o);
    return v;
}

// ---------------------------------------------------------------------------
// W(32 x CW) = V^T C (+ C_slot for a structured step) over the B tile rows,
// 3xTF32 mma.sync; warp w computes the 16 x 8 output tile (w & 1, w >> 1).
// Six independent accumulators (3 products x even / odd k-steps) keep the
// tensor pipe busy instead of one 72-deep dependent chain.
// ---------------------------------------------------------------------------
template <class Cfg>
__device__ __forceinline__ void chain_gemm_vtc(const float* Vs, const float* Cs, const float* Csl, bool slot,
                                               float* Ws) {
    constexpr int VP = Cfg::VP, B = Cfg::B, WS = Cfg::WS;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, t = lane & 3;
    const int mt = warp & 1, nt = warp >> 1;
    float acc[3][4];
#pragma unroll
    for (int a = 0; a < 3; ++a)
#pragma unroll
        for (int e = 0; e < 4; ++e) acc[a][e] = 0.f;
    const float* v0 = Vs + (size_t)(16 * mt + g) * VP;
    const float* v8 = v0 + 8 * (size_t)VP;
    const float* cc = Cs + (size_t)(8 * nt + g) * VP;
#pragma unroll 4
    for (int k = 0; k < B; k += 8) {
        uint32_t ah[4], al[4], bh[2], bl[2];
        split_tf32(v0[k + t], ah[0], al[0]);
        split_tf32(v8[k + t], ah[1], al[1]);
        split_tf32(v0[k + t + 4], ah[2], al[2]);
        split_tf32(v8[k + t + 4], ah[3], al[3]);
        split_tf32(cc[k + t], bh[0], bl[0]);
        split_tf32(cc[k + t + 4], bh[1], bl[1]);
        mma_tf32(acc[0], al, bh);
        mma_tf32(acc[1], ah, bl);
        mma_tf32(acc[2], ah, bh);
    }
    const int r0 = 16 * mt + g, c0 = 8 * nt + 2 * t;
    float w[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) w[e] = (acc[0][e] + acc[1][e]) + acc[2][e];
    if (slot) {  // structured head: V = [I; V_tile] -> W += C_slot (Csl[col][row])
        w[0] += Csl[c0 * 32 + r0];
        w[1] += Csl[(c0 + 1) * 32 + r0];
        w[2] += Csl[c0 * 32 + r0 + 8];
        w[3] += Csl[(c0 + 1) * 32 + r0 + 8];
    }
    Ws[r0 * WS + c0] = w[0];
    Ws[r0 * WS + c0 + 1] = w[1];
    Ws[(r0 + 8) * WS + c0] = w[2];
    Ws[(r0 + 8) * WS + c0 + 1] = w[3];
}

// G(32 x 32) = V^T V over the B tile rows (3xTF32 mma.sync): warp w computes
// the 16 x 8 tiles (w & 1, w >> 1) and (w & 1, 2 + (w >> 1)).  Only the strict
// upper part is used (T's recurrence); a structured step's head parts e_j are
// orthogonal, so G is the tile part alone.
template <class Cfg>
__device__ __forceinline__ void chain_gemm_gram(const float* Vs, float* Gs) {
    constexpr int VP = Cfg::VP, B = Cfg::B, HS = Cfg::HS;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, t = lane & 3;
    const int mt = warp & 1;
    float acc[2][3][4];
#pragma unroll
    for (int a = 0; a < 2; ++a)
#pragma unroll
        for (int b = 0; b < 3; ++b)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[a][b][e] = 0.f;
    const float* v0 = Vs + (size_t)(16 * mt + g) * VP;
    const float* v8 = v0 + 8 * (size_t)VP;
#pragma unroll 2
    for (int k = 0; k < B; k += 8) {
        uint32_t ah[4], al[4];
        split_tf32(v0[k + t], ah[0], al[0]);
        split_tf32(v8[k + t], ah[1], al[1]);
        split_tf32(v0[k + t + 4], ah[2], al[2]);
        split_tf32(v8[k + t + 4], ah[3], al[3]);
#pragma unroll
        for (int u = 0; u < 2; ++u) {
            const int nt = (warp >> 1) + 2 * u;
            const float* cc = Vs + (size_t)(8 * nt + g) * VP;
            uint32_t bh[2], bl[2];
            split_tf32(cc[k + t], bh[0], bl[0]);
            split_tf32(cc[k + t + 4], bh[1], bl[1]);
            mma_tf32(acc[u][0], al, bh);
            mma_tf32(acc[u][1], ah, bl);
            mma_tf32(acc[u][2], ah, bh);
        }
    }
#pragma unroll
    for (int u = 0; u < 2; ++u) {
        const int nt = (warp >> 1) + 2 * u;
        const int r0 = 16 * mt + g, c0 = 8 * nt + 2 * t;
        float w[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) w[e] = (acc[u][0][e] + acc[u][1][e]) + acc[u][2][e];
        Gs[r0 * HS + c0] = w[0];
        Gs[r0 * HS + c0 + 1] = w[1];
        Gs[(r0 + 8) * HS + c0] = w[2];
        Gs[(r0 + 8) * HS + c0 + 1] = w[3];
    }
}

// T (upper, Ts[r][c]) from G and tau (xLARFT forward / columnwise:
// T[j][j] = tau_j, T[0:j,j] = -tau_j T[0:j,0:j] G[0:j,j]); one warp, lane i
// keeps row i of T in registers; the G column is read by broadcast.  Also
// writes the workspace's column-major T block.
__device__ __forceinline__ void chain_build_t(const float* Gs, const float* taus, int wp, float* Ts, float* tb,
                                              int HS) {
    const int lane = threadIdx.x & 31;
    float row[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) {
        float a0 = 0.f, a1 = 0.f, a2 = 0.f, a3 = 0.f;
#pragma unroll
        for (int k = 0; k + 3 < j; k += 4) {
            a0 = fmaf(row[k + 0], Gs[(k + 0) * HS + j], a0);
            a1 = fmaf(row[k + 1], Gs[(k + 1) * HS + j], a1);
            a2 = fmaf(row[k + 2], Gs[(k + 2) * HS + j], a2);
            a3 = fmaf(row[k + 3], Gs[(k + 3) * HS + j], a3);
        }
#pragma unroll
        for (int k = j & ~3; k < j; ++k) a0 = fmaf(row[k], Gs[k * HS + j], a0);
        const float tau = j < wp ? taus[j] : 0.f;
        row[j] = (j == lane) ? tau : (j > lane ? -tau * ((a0 + a1) + (a2 + a3)) : 0.f);
    }
#pragma unroll
    for (int j = 0; j < 32; ++j) Ts[lane * HS + j] = row[j];
#pragma unroll
    for (int j = 0; j < 32; ++j) __stcg(tb + j * 32 + lane, row[j]);  // column-major, coalesced across lanes
}

// W2(32 x CW) = T^T W (T upper triangular), 3xTF32 mma.sync, one 16 x 8 tile per warp.
template <class Cfg>
__device__ __forceinline__ void chain_gemm_tw(const float* Ts, const float* Ws, float* W2s) {
    constexpr int HS = Cfg::HS, WS = Cfg::WS;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, t = lane & 3;
    const int mt = warp & 1, nt = warp >> 1;
    float acc[4] = {0.f, 0.f, 0.f, 0.f};
    const int i0 = 16 * mt + g;
#pragma unroll
    for (int k0 = 0; k0 < 32; k0 += 8) {
        if (k0 >= 16 * (mt + 1)) break;  // T^T is lower triangular: A[i][k] = T[k][i] = 0 for k > i
        uint32_t ah[4], al[4], bh[2], bl[2];
        split_tf32(Ts[(k0 + t) * HS + i0], ah[0], al[0]);
        split_tf32(Ts[(k0 + t) * HS + i0 + 8], ah[1], al[1]);
        split_tf32(Ts[(k0 + t + 4) * HS + i0], ah[2], al[2]);
        split_tf32(Ts[(k0 + t + 4) * HS + i0 + 8], ah[3], al[3]);
        split_tf32(Ws[(k0 + t) * WS + 8 * nt + g], bh[0], bl[0]);
        split_tf32(Ws[(k0 + t + 4) * WS + 8 * nt + g], bh[1], bl[1]);
        mma_3xtf32(acc, ah, al, bh, bl);
    }
    const int c0 = 8 * nt + 2 * t;
    W2s[i0 * WS + c0] = acc[0];
    W2s[i0 * WS + c0 + 1] = acc[1];
    W2s[(i0 + 8) * WS + c0] = acc[2];
    W2s[(i0 + 8) * WS + c0 + 1] = acc[3];
}

// Cs(B x CW) -= V(B x 32) W2(32 x CW) (3xTF32 mma.sync); warp w owns row
// tiles w, w + NW, ... of 16 rows and both 8-column tiles.
template <class Cfg>
__device__ __forceinline__ void chain_gemm_update(const float* Vs, float* Cs, const float* W2s) {
    constexpr int VP = Cfg::VP, B = Cfg::B, WS = Cfg::WS;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, t = lane & 3;
    uint32_t bh[4][2][2], bl[4][2][2];  // -W2 fragments: k-step kk, column tile nt
#pragma unroll
    for (int kk = 0; kk < 4; ++kk)
#pragma unroll
        for (int nt = 0; nt < 2; ++nt) {
            split_tf32(-W2s[(8 * kk + t) * WS + 8 * nt + g], bh[kk][nt][0], bl[kk][nt][0]);
            split_tf32(-W2s[(8 * kk + t + 4) * WS + 8 * nt + g], bh[kk][nt][1], bl[kk][nt][1]);
        }
    for (int mt = warp; mt < B / 16; mt += Cfg::NW) {
        const int m0 = 16 * mt;
        float d[2][4];
#pragma unroll
        for (int nt = 0; nt < 2; ++nt) {
            const float* c0 = Cs + (size_t)(8 * nt + 2 * t) * VP;
            d[nt][0] = c0[m0 + g];
            d[nt][1] = c0[VP + m0 + g];
            d[nt][2] = c0[m0 + g + 8];
            d[nt][3] = c0[VP + m0 + g + 8];
        }
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
            const float* va = Vs + (size_t)(8 * kk + t) * VP;
            const float* vb = va + 4 * (size_t)VP;
            uint32_t ah[4], al[4];
            split_tf32(va[m0 + g], ah[0], al[0]);
            split_tf32(va[m0 + g + 8], ah[1], al[1]);
            split_tf32(vb[m0 + g], ah[2], al[2]);
            split_tf32(vb[m0 + g + 8], ah[3], al[3]);
#pragma unroll
            for (int nt = 0; nt < 2; ++nt) mma_3xtf32(d[nt], ah, al, bh[kk][nt], bl[kk][nt]);
        }
#pragma unroll
        for (int nt = 0; nt < 2; ++nt) {
            float* c0 = Cs + (size_t)(8 * nt + 2 * t) * VP;
            c0[m0 + g] = d[nt][0];
            c0[VP + m0 + g] = d[nt][1];
            c0[m0 + g + 8] = d[nt][2];
            c0[VP + m0 + g + 8] = d[nt][3];
        }
    }
}

// cp.async one C chunk (columns cb0 .. cb0+ncb) into (Cs, Csl): tile rows
// [0, h) (a leaf: only rows >= 32p are needed; the others are zero-filled),
// and for a structured step the slot rows 32p .. 32p+wp.  Commits one group.
// Per-thread part of a chunk's row quads: column cc = tid / 8 (CW = 16 columns x
// 8 threads), quads u = tid % 8 + 8 k: tile-row quads u < B / 4, then the 8
// slot-row quads.
template <class Cfg>
struct ChunkMap {
    static constexpr int NQ4 = Cfg::B / 4;
    static constexpr int NU = (NQ4 + 8) / 8;  // quads per thread
    static_assert(Cfg::CW * 8 == Cfg::NT && (NQ4 + 8) % 8 == 0, "chunk map");
};

// cp.async one C chunk (columns cb0 .. cb0+ncb) into (Cs, Csl): tile rows
// [0, h) (a leaf: only rows >= 32p are needed; the others are zero-filled),
// and for a structured step the slot rows 32p .. 32p+wp.  Commits one group.
template <class Cfg>
__device__ __forceinline__ void chain_stage(float* Cs, float* Csl, const float* A, int64_t lda, int64_t cb0, int ncb,
                                            int64_t s, int h, int64_t slotp, int wp, bool leaf, int hr0) {
    using M = ChunkMap<Cfg>;
    const int cc = threadIdx.x >> 3, u0 = threadIdx.x & 7;
    const float* colp = A + (cb0 + min(cc, ncb - 1)) * lda;
    const bool colok = cc < ncb;
#pragma unroll
    for (int k = 0; k < M::NU; ++k) {
        const int u = u0 + 8 * k;
        float* dst;
        const float* src;
        int valid;
        if (u < M::NQ4) {
            const int r = 4 * u;
            dst = Cs + (size_t)cc * Cfg::VP + r;
            src = colp + s + r;
            valid = (colok && !(leaf && r + 4 <= hr0)) ? max(0, min(4, h - r)) : 0;
        } else {
            const int r = 4 * (u - M::NQ4);
            dst = Csl + cc * 32 + r;
            src = colp + slotp + r;
            valid = (!leaf && colok) ? max(0, min(4, wp - r)) : 0;
        }
        if (valid == 4 && (reinterpret_cast<uintptr_t>(src) & 15) == 0) {
            const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src) : "memory");
        } else {
#pragma unroll
            for (int e = 0; e < 4; ++e) dst[e] = e < valid ? __ldcg(src + e) : 0.f;
        }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

// Write a chunk back: tile rows < h (a leaf: rows >= 32p), slot rows < wp.
template <class Cfg>
__device__ __forceinline__ void chain_store(const float* Cs, const float* Csl, float* A, int64_t lda, int64_t cb0,
                                            int ncb, int64_t s, int h, int64_t slotp, int wp, bool leaf, int hr0) {
    using M = ChunkMap<Cfg>;
    const int cc = threadIdx.x >> 3, u0 = threadIdx.x & 7;
    if (cc >= ncb) return;
    float* colp = A + (cb0 + cc) * lda;
#pragma unroll
    for (int k = 0; k < M::NU; ++k) {
        const int u = u0 + 8 * k;
        const float* srcs;
        float* dst;
        int valid;
        if (u < M::NQ4) {
            const int r = 4 * u;
            srcs = Cs + (size_t)cc * Cfg::VP + r;
            dst = colp + s + r;
            valid = !(leaf && r + 4 <= hr0) ? max(0, min(4, h - r)) : 0;
        } else {
            const int r = 4 * (u - M::NQ4);
            srcs = Csl + cc * 32 + r;
            dst = colp + slotp + r;
            valid = !leaf ? max(0, min(4, wp - r)) : 0;
        }
        if (valid == 4 && (reinterpret_cast<uintptr_t>(dst) & 15) == 0) {
            __stcg(reinterpret_cast<float4*>(dst), *reinterpret_cast<const float4*>(srcs));
        } else {
            for (int e = 0; e < valid; ++e) dst[e] = srcs[e];
        }
    }
}

// ---------------------------------------------------------------------------
// The chain kernel.  Grid: persistent CTAs taking chains from sync[0].
// ---------------------------------------------------------------------------
template <int NQ, int SEG, int MINB>
__global__ void __launch_bounds__(32 * NQ, MINB)
tsqr_chain_kernel(Geom g, float* __restrict__ A, float* __restrict__ Tws, int* __restrict__ sync,
                  unsigned long long* prof) {
    using Cfg = ChainCfg<NQ, SEG>;
    constexpr int VP = Cfg::VP, HS = Cfg::HS, WS = Cfg::WS, CW = Cfg::CW;
    extern __shared__ __align__(16) unsigned char chain_smem_raw[];
    float* sm = reinterpret_cast<float*>(chain_smem_raw);
    float* Vs = sm + Cfg::OFF_V;
    float* Hh = sm + Cfg::OFF_H;
    float* Ts = sm + Cfg::OFF_T;
    float* Gs = sm + Cfg::OFF_G;
    float* Ws = sm + Cfg::OFF_W;
    float* W2s = sm + Cfg::OFF_W2;
    float* taus = sm + Cfg::OFF_TAU;
    __shared__ int s_task;
    // optional phase profile (diagnostics, CAQR_PROFILE=1): thread 0's clock
    __shared__ unsigned long long pacc[7];  // [6] = last stamp
    if (threadIdx.x < 7) pacc[threadIdx.x] = threadIdx.x == 6 ? (unsigned long long)clock64() : 0ull;
#define CHAIN_PROF(k)                                 \
    do {                                              \
        if (prof && threadIdx.x == 0) {               \
            const unsigned long long t1_ = clock64(); \
            pacc[k] += t1_ - pacc[6];                 \
            pacc[6] = t1_;                            \
        }                                             \
    } while (0)

    const int tid = threadIdx.x;
    const int c = tid / NQ, q = tid % NQ;
    const int lane = tid & 31;
    const unsigned gm = (NQ >= 32 ? 0xffffffffu : ((1u << NQ) - 1u)) << (lane & ~(NQ - 1));
    const int64_t lda = g.lda;
    float x[SEG];

    for (;;) {
        __syncthreads();
        if (tid == 0) s_task = atomicAdd(sync, 1);
        __syncthreads();
        const int64_t node = s_task;
        if (node >= g.P) break;
        const int64_t slot = g.row0 + node * g.bm;  // the chain's R slot (first tile's top rows)
        const int ntile = (int)min(g.K, g.L - node * g.K);
        for (int kt = 0; kt < ntile; ++kt) {
            const int64_t t = node * g.K + kt;
            const int64_t s = g.row0 + t * g.b;  // first row of the tile
            const int h = (int)min(g.b, g.mrows - t * g.b);
            const bool leaf = kt == 0;
            for (int p = 0; p < g.npan; ++p) {
                const int wp = min(kPW, g.ncols - 32 * p);
                const int64_t c0 = g.col0 + 32 * p;
                const int hr0 = 32 * p;  // leaf: first head row (tile-relative)
                // ---------------- load the panel ------------------------------
                // x: column c, tile rows q*SEG + i (zero beyond h / beyond wp);
                // leaf: rows < 32p zero, rows [32p, 32p+32) moved to Hh.
                // p > 0: the panel's columns were left in x by the previous
                // panel's trailing update (its chunks 0 and 1).
                if (p == 0) {
                    const float* col = A + (c0 + min(c, wp - 1)) * lda + s;
                    const bool vec = ((reinterpret_cast<uintptr_t>(col) & 15) == 0);
#pragma unroll
                    for (int i = 0; i < SEG; i += 4) {
                        const int r = q * SEG + i;
                        float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
                        if (c < wp) {
                            if (vec && r + 4 <= h) {
                                v = __ldcg(reinterpret_cast<const float4*>(col + r));
                            } else {
                                if (r < h) v.x = __ldcg(col + r);
                                if (r + 1 < h) v.y = __ldcg(col + r + 1);
                                if (r + 2 < h) v.z = __ldcg(col + r + 2);
                                if (r + 3 < h) v.w = __ldcg(col + r + 3);
                            }
                        }
                        x[i] = v.x;
                        x[i + 1] = v.y;
                        x[i + 2] = v.z;
                        x[i + 3] = v.w;
                    }
                }
                if (leaf) {
                    // move rows [32p, 32p+32) to Hh, zero rows < 32p + 32 in x
#pragma unroll
                    for (int i = 0; i < SEG; ++i) {
                        const int r = q * SEG + i;
                        if (r < hr0 + 32) {
                            if (r >= hr0) Hh[(r - hr0) * HS + c] = x[i];
                            x[i] = 0.f;
                        }
                    }
                } else {
                    // heads: the chain R's rows 32p.. (upper triangle of the panel block)
                    for (int e = tid; e < 32 * 32; e += Cfg::NT) {
                        const int i = e & 31, j = e >> 5;
                        Hh[i * HS + j] = (j < wp && i <= j) ? __ldcg(A + (c0 + j) * lda + slot + hr0 + i) : 0.f;
                    }
                }
                __syncthreads();

                CHAIN_PROF(0);
                // ---------------- factor ----------------------------------------
                // pivot of column jj by its NQ threads (called with c == jj)
                auto pivot = [&](int jj) {
                    float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
#pragma unroll
                    for (int i = 0; i < SEG; i += 4) {
                        s0 = fmaf(x[i], x[i], s0);
                        s1 = fmaf(x[i + 1], x[i + 1], s1);
                        s2 = fmaf(x[i + 2], x[i + 2], s2);
                        s3 = fmaf(x[i + 3], x[i + 3], s3);
                    }
                    float sg = (s0 + s1) + (s2 + s3);
                    if (leaf) {  // this thread's head rows k > jj (k = q mod NQ)
                        for (int k = q; k < 32; k += NQ)
                            if (k > jj) {
                                const float hv = Hh[k * HS + jj];
                                sg = fmaf(hv, hv, sg);
                            }
                    }
                    sg = qsum<NQ>(sg, gm);
                    __syncwarp(gm);  // (leaf) the group's head-row updates are visible
                    const float al = Hh[jj * HS + jj];
                    float tau = 0.f, beta = al, scale = 1.f;
                    if (sg != 0.f) {
                        float rmu, mu;
                        rsqrt_refined(fmaf(al, al, sg), rmu, mu);
                        beta = -copysignf(mu, al);
                        tau = fmaf(fabsf(al), rmu, 1.f);
                        scale = copysignf(rcp_refined(fabsf(al) + mu), al);
                    }
#pragma unroll
                    for (int i = 0; i < SEG; ++i) x[i] *= scale;
                    float* vc = Vs + (size_t)jj * VP + q * SEG;
#pragma unroll
                    for (int i = 0; i < SEG; i += 4)
                        *reinterpret_cast<float4*>(vc + i) = make_float4(x[i], x[i + 1], x[i + 2], x[i + 3]);
                    if (leaf)
                        for (int k = q; k < 32; k += NQ)
                            if (k > jj) Hh[k * HS + jj] *= scale;
                    __syncwarp(gm);
                    if (q == 0) {
                        Hh[jj * HS + jj] = beta;
                        taus[jj] = tau;
                    }
                };
                if (c == 0) pivot(0);
                __syncthreads();
                for (int j = 0; j < wp; ++j) {
                    if (c > j && c < wp) {
                        const float tau = taus[j];
                        float v[SEG];
                        const float* vj = Vs + (size_t)j * VP + q * SEG;
#pragma unroll
                        for (int i = 0; i < SEG; i += 4) {
                            const float4 f = *reinterpret_cast<const float4*>(vj + i);
                            v[i] = f.x;
                            v[i + 1] = f.y;
                            v[i + 2] = f.z;
                            v[i + 3] = f.w;
                        }
                        float d0 = 0.f, d1 = 0.f, d2 = 0.f, d3 = 0.f;
#pragma unroll
                        for (int i = 0; i < SEG; i += 4) {
                            d0 = fmaf(v[i], x[i], d0);
                            d1 = fmaf(v[i + 1], x[i + 1], d1);
                            d2 = fmaf(v[i + 2], x[i + 2], d2);
                            d3 = fmaf(v[i + 3], x[i + 3], d3);
                        }
                        float d = (d0 + d1) + (d2 + d3);
                        if (leaf) {
                            // head-block rows k >= j (v_j[k] = 1 at k == j)
                            for (int k = q; k < 32; k += NQ)
                                if (k >= j) {
                                    const float vk = k == j ? 1.f : Hh[k * HS + j];
                                    d = fmaf(vk, Hh[k * HS + c], d);
                                }
                        } else if (q == 0) {
                            d += Hh[j * HS + c];  // structured head: v_j = e_j on the slot rows
                        }
                        d = qsum<NQ>(d, gm);
                        {
                            const float st = tau * d;
                            if (leaf) {
                                for (int k = q; k < 32; k += NQ)
                                    if (k >= j) {
                                        const float vk = k == j ? 1.f : Hh[k * HS + j];
                                        Hh[k * HS + c] = fmaf(-st, vk, Hh[k * HS + c]);
                                    }
                            } else if (q == 0) {
                                Hh[j * HS + c] -= st;
                            }
#pragma unroll
                            for (int i = 0; i < SEG; ++i) x[i] = fmaf(-st, v[i], x[i]);
                            if (c == j + 1) pivot(j + 1);
                        }
                    }
                    __syncthreads();
                }
                CHAIN_PROF(1);
                // V columns >= wp are zero; a leaf's head-block rows: 1 on the
                // diagonal, v below, 0 above
                for (int jj = wp + (tid / 32); jj < 32; jj += Cfg::NW)
                    for (int r = lane; r < Cfg::B; r += 32) Vs[(size_t)jj * VP + r] = 0.f;
                if (leaf) {
                    for (int e = tid; e < 32 * 32; e += Cfg::NT) {
                        const int k = e & 31, jj = e >> 5;
                        if (jj < wp && hr0 + k < Cfg::B)
                            Vs[(size_t)jj * VP + hr0 + k] = k > jj ? Hh[k * HS + jj] : (k == jj ? 1.f : 0.f);
                    }
                }
                // ---------------- write V / R -----------------------------------
                if (c < wp) {
                    float* col = A + (c0 + c) * lda + s;
                    const bool vec = ((reinterpret_cast<uintptr_t>(col) & 15) == 0);
#pragma unroll
                    for (int i = 0; i < SEG; i += 4) {
                        const int r = q * SEG + i;
                        if (leaf && r + 4 <= hr0 + 32) continue;  // rows owned by R / the head block
                        if (vec && r + 4 <= h && !(leaf && r < hr0 + 32)) {
                            __stcg(reinterpret_cast<float4*>(col + r), make_float4(x[i], x[i + 1], x[i + 2], x[i + 3]));
                        } else {
#pragma unroll
                            for (int e = 0; e < 4; ++e)
                                if (r + e < h && !(leaf && r + e < hr0 + 32)) col[r + e] = x[i + e];
                        }
                    }
                }
                if (leaf) {
                    // head block: R on/above the diagonal, v below
                    for (int e = tid; e < 32 * 32; e += Cfg::NT) {
                        const int i = e & 31, jj = e >> 5;
                        if (jj < wp && hr0 + i < h) A[(c0 + jj) * lda + s + hr0 + i] = Hh[i * HS + jj];
                    }
                } else {
                    for (int e = tid; e < 32 * 32; e += Cfg::NT) {
                        const int i = e & 31, jj = e >> 5;
                        if (jj < wp && i <= jj) A[(c0 + jj) * lda + slot + hr0 + i] = Hh[i * HS + jj];
                    }
                }
                __syncthreads();
                chain_gemm_gram<Cfg>(Vs, Gs);  // G = V^T V (tile part)
                __syncthreads();
                if (tid < 32) chain_build_t(Gs, taus, wp, Ts, Tws + (t * g.npan + p) * (kPW * kPW), HS);

                CHAIN_PROF(2);
                // ---------------- trailing update --------------------------------
                const int64_t tfirst = c0 + 32, tend = g.col0 + g.ncols;
                const int nchunk = tend > tfirst ? (int)((tend - tfirst + CW - 1) / CW) : 0;
                const int64_t slotp = slot + hr0;
                // chunk order: the next panel's two chunks (0, 1) last, so that
                // they can go from shared memory straight into the registers
                auto cid = [&](int ib) { return nchunk >= 3 ? (ib + 2) % nchunk : ib; };
                auto chunk_cols = [&](int k, int64_t* cb) {
                    *cb = tfirst + (int64_t)CW * k;
                    return (int)min((int64_t)CW, tend - *cb);
                };
                if (nchunk > 0) {
                    int64_t cb;
                    const int n0c = chunk_cols(cid(0), &cb);
                    chain_stage<Cfg>(sm + Cfg::OFF_C, sm + Cfg::OFF_CS, A, lda, cb, n0c, s, h, slotp, wp, leaf, hr0);
                }
                for (int ib = 0; ib < nchunk; ++ib) {
                    int64_t cb0;
                    const int ncb = chunk_cols(cid(ib), &cb0);
                    float* Cs = sm + Cfg::OFF_C + (ib & 1) * CW * VP;
                    float* Csl = sm + Cfg::OFF_CS + (ib & 1) * CW * 32;
                    if (ib + 1 < nchunk) {  // prefetch the next chunk into the other buffer
                        int64_t cb1;
                        const int n1c = chunk_cols(cid(ib + 1), &cb1);
                        chain_stage<Cfg>(sm + Cfg::OFF_C + ((ib + 1) & 1) * CW * VP,
                                         sm + Cfg::OFF_CS + ((ib + 1) & 1) * CW * 32, A, lda, cb1, n1c, s, h, slotp, wp,
                                         leaf, hr0);
                        asm volatile("cp.async.wait_group 1;" ::: "memory");
                    } else {
                        asm volatile("cp.async.wait_group 0;" ::: "memory");
                    }
                    __syncthreads();
                    CHAIN_PROF(3);
                    chain_gemm_vtc<Cfg>(Vs, Cs, Csl, !leaf, Ws);
                    __syncthreads();
                    chain_gemm_tw<Cfg>(Ts, Ws, W2s);
                    __syncthreads();
                    if (!leaf)  // slot rows: C_slot -= W2 (V's head part is the identity)
                        for (int e = tid; e < CW * 32; e += Cfg::NT) {
                            const int cc = e >> 5, i = e & 31;
                            Csl[cc * 32 + i] -= W2s[i * WS + cc];
                        }
                    chain_gemm_update<Cfg>(Vs, Cs, W2s);
                    __syncthreads();
                    CHAIN_PROF(4);
                    chain_store<Cfg>(Cs, Csl, A, lda, cb0, ncb, s, h, slotp, wp, leaf, hr0);
                    if (ib + 1 < nchunk) __syncthreads();
                }
                if (nchunk > 0) {
                    // the next panel's columns (chunks 0 and 1, the last two
                    // processed) from shared memory into the registers
                    const int k = c / CW;
                    const int buf = nchunk >= 2 ? ((nchunk - 2 + k) & 1) : 0;
                    const bool ok = c < min(32, (int)(tend - tfirst));
                    const float* cs = sm + Cfg::OFF_C + buf * CW * VP + (size_t)(c % CW) * VP + q * SEG;
#pragma unroll
                    for (int i = 0; i < SEG; i += 4) {
                        const float4 f = ok ? *reinterpret_cast<const float4*>(cs + i) : make_float4(0.f, 0.f, 0.f, 0.f);
                        x[i] = f.x;
                        x[i + 1] = f.y;
                        x[i + 2] = f.z;
                        x[i + 3] = f.w;
                    }
                }
                __syncthreads();
                CHAIN_PROF(3);
            }
        }
        CHAIN_PROF(5);
    }
    if (prof && threadIdx.x == 0)
        for (int k = 0; k < 6; ++k) atomicAdd(prof + k, pacc[k]);
#undef CHAIN_PROF
}

template <int NQ, int SEG>
inline size_t chain_smem_bytes() {
    return ChainCfg<NQ, SEG>::BYTES;
}

}  // namespace caqr
