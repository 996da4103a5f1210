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
#include <type_traits>
#include <cuda_fp16.h>
#include "tsqr_fused.cuh"
#include "umma.cuh"

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

// W2(32 x 16) = T^T W (T upper triangular), 3xTF32 mma.sync, one 16 x 8 tile per
// warp (4 warps); strides of T and of W / W2 given.
template <int HS, int WS>
__device__ __forceinline__ void chain_gemm_tw_s(const float* Ts, const float* Ws, float* W2s) {
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
template <class Cfg>
__device__ __forceinline__ void chain_gemm_tw(const float* Ts, const float* Ws, float* W2s) {
    chain_gemm_tw_s<Cfg::HS, Cfg::WS>(Ts, Ws, W2s);
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
// tcgen05 (5th-generation tensor core) trailing update, fp16x2 operands.
//
// The three contractions of a node's blocked update -- G = V^T V (for T),
// W = V^T C and dC = V W2 -- run as tcgen05.mma kind::f16 with fp32 accumulators
// in tensor memory.  fp32 operands are split x ~ hi + lo (hi = fp16(x), lo =
// fp16(x - hi)), each with a power-of-two scale: V by 2^15 (|v| <= 1 for a
// Householder vector with unit head), every column of C and of W2 by 2^e with
// max|column| * 2^e in [2^14, 2^15).  The 11-bit fp16 significand equals
// TF32's, so hi + lo carries 22 bits: |x - hi - lo| <= 2^-22 max|column|, the
// three products hi*hi + hi*lo + lo*hi (exact in fp32, fp32 accumulation)
// give a normwise error ~2^-21 -- the 3xTF32 bound -- at the
// storage size of fp32.  One shared buffer holds V as the K-major operand V^T
// (G, W) and as the MN-major operand V (dC).
// ---------------------------------------------------------------------------
template <int NQ, int SEG>
struct ChainCfgTC {
    static constexpr int NT = 32 * NQ;
    static constexpr int NW = NT / 32;
    static constexpr int B = NQ * SEG;
    static constexpr int VP = B + 4;
    static constexpr int CW = 16;
    static constexpr int HS = 33;
    static constexpr int WS2 = 17;                     // stride of the 64-row TMEM dumps
    // floats
    static constexpr int OFF_V = 0;                    // fp32 Vs[32][VP] / fp16 V hi|lo (64 x B)
    static constexpr int OFF_C = OFF_V + 32 * VP;      // fp32 C chunk [2][CW][VP]
    static constexpr int OFF_H = OFF_C + CW * VP;      // Hh[32][HS], then G dump [64][HS] (C buffer 1)
    static constexpr int OFF_G = OFF_H;
    static constexpr int OFF_CH = OFF_C + 2 * CW * VP; // fp16 C hi|lo (CW x B each), then W dump [64][WS2]
    static constexpr int OFF_CS = OFF_CH + CW * B;     // Csl[2][CW][32]
    static constexpr int OFF_W2H = OFF_CS + 2 * CW * 32;  // fp16 W2 hi|lo (CW x 32 each)
    static constexpr int OFF_T = OFF_W2H + CW * 32;    // Ts[32][HS]
    static constexpr int OFF_TAU = OFF_T + 32 * HS;    // taus[32]
    static constexpr int OFF_SC = OFF_TAU + 32;        // C column scales [CW], W2 column scales [CW]
    static constexpr int OFF_MB = OFF_SC + 2 * CW;     // mbarrier (8 bytes)
    static constexpr int FLOATS = OFF_MB + 4;
    static constexpr size_t BYTES = sizeof(float) * (size_t)FLOATS;
    static constexpr uint32_t SBO_V = (B / 8) * 128;   // V: byte(i, r) = (i%8)16 + (r%8)2 + (i/8)SBO_V + (r/8)128
    static constexpr uint32_t SBO_C = (B / 8) * 128;   // C: byte(n, r) likewise
    static constexpr uint32_t TM_G = 0, TM_W = 32, TM_D1 = 48, TM_D2 = 64;  // TMEM columns
    static_assert(NQ == 4 && CW * 8 == NT, "layout");
    static_assert(B % 64 == 0, "row blocks of 128 (+64)");
    static_assert(OFF_MB % 2 == 0, "mbarrier alignment");
    static_assert(64 * HS <= CW * VP && 64 * WS2 <= CW * B, "dump areas");
};

__device__ __forceinline__ float pow2f(int e) { return __uint_as_float((uint32_t)(min(max(e, -126), 127) + 127) << 23); }
// Scale exponent for a column whose max |value| is m: m * 2^e in [2^14, 2^15).
__device__ __forceinline__ int col_exp(float m) {
    return m > 0.f ? 14 - ((int)((__float_as_uint(m) >> 23) & 0xff) - 127) : 0;
}
__device__ __forceinline__ void split_f16(float x, __half& h, __half& l) {
    h = __float2half_rn(x);
    l = __float2half_rn(x - __half2float(h));
}
// pack 4 halves into 8 bytes
__device__ __forceinline__ uint2 pack4(__half a, __half b, __half c, __half d) {
    return make_uint2((uint32_t)__half_as_ushort(a) | ((uint32_t)__half_as_ushort(b) << 16),
                      (uint32_t)__half_as_ushort(c) | ((uint32_t)__half_as_ushort(d) << 16));
}

// ---------------------------------------------------------------------------
// The chain kernel.  Grid: persistent CTAs taking chains from sync[0].
// ---------------------------------------------------------------------------
template <int NQ, int SEG, int MINB, bool TC>
__global__ void __launch_bounds__(32 * NQ, MINB)
tsqr_chain_kernel(Geom g, float* __restrict__ A, float* __restrict__ Tws, int* __restrict__ sync,
                  unsigned long long* prof) {
    using Cfg = typename std::conditional<TC, ChainCfgTC<NQ, SEG>, ChainCfg<NQ, SEG>>::type;
    constexpr int VP = Cfg::VP, HS = Cfg::HS, CW = Cfg::CW;
    extern __shared__ __align__(128) unsigned char chain_smem_raw[];
    float* sm = reinterpret_cast<float*>(chain_smem_raw);
    float* Vs = sm + Cfg::OFF_V;
    float* Hh = sm + Cfg::OFF_H;
    float* Ts = sm + Cfg::OFF_T;
    float* Gs = sm + Cfg::OFF_G;
    float* taus = sm + Cfg::OFF_TAU;
    __shared__ int s_task;
    __shared__ uint32_t s_tmem;
    uint32_t mph = 0;  // mbarrier phase (TC)
    if constexpr (TC) {
        if (threadIdx.x < 32) umma::tmem_alloc<128>(&s_tmem);
        if (threadIdx.x == 0) umma::mbar_init(reinterpret_cast<uint64_t*>(sm + Cfg::OFF_MB), 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        umma::fence_before_sync();
        __syncthreads();
        umma::fence_after_sync();
    }
    // optional phase profile (diagnostics, CAQR_PROFILE=1): thread 0's clock
    __shared__ unsigned long long pacc[11];  // [10] = last stamp
    if (threadIdx.x < 11) pacc[threadIdx.x] = threadIdx.x == 10 ? (unsigned long long)clock64() : 0ull;
#define CHAIN_PROF(k)                                 \
    do {                                              \
        if (prof && threadIdx.x == 0) {               \
            const unsigned long long t1_ = clock64(); \
            pacc[k] += t1_ - pacc[10];                \
            pacc[10] = t1_;                           \
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
                if constexpr (!TC)
                for (int jj = wp + (tid / 32); jj < 32; jj += Cfg::NW)
                    for (int r = lane; r < Cfg::B; r += 32) Vs[(size_t)jj * VP + r] = 0.f;
                if (!TC && leaf) {
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
                if constexpr (TC) {
                    using umma::smem_u32;
                    uint64_t* mbar = reinterpret_cast<uint64_t*>(sm + Cfg::OFF_MB);
                    const uint32_t tmem = s_tmem;
                    unsigned char* Vh = reinterpret_cast<unsigned char*>(sm + Cfg::OFF_V);   // fp16 V hi | lo
                    unsigned char* Ch = reinterpret_cast<unsigned char*>(sm + Cfg::OFF_CH);  // fp16 C hi | lo
                    unsigned char* W2h = reinterpret_cast<unsigned char*>(sm + Cfg::OFF_W2H);
                    float* cscale = sm + Cfg::OFF_SC;
                    float* wscale = cscale + CW;
                    const int warp = tid >> 5;
                    auto wait_mma = [&]() {
                        umma::mbar_wait(mbar, mph);
                        mph ^= 1u;
                        umma::fence_after_sync();
                    };
                    // ---- V -> fp16 hi | lo (scaled by 2^15), K-major V^T layout ----
                    __syncthreads();  // every consumer is done with the fp32 Vs; Hh complete
                    {
#pragma unroll
                        for (int i = 0; i < SEG; i += 4) {
                            const int r = q * SEG + i;
                            float v4[4];
#pragma unroll
                            for (int e = 0; e < 4; ++e) {
                                float v = x[i + e];
                                if (leaf) {
                                    const int k = r + e - hr0;  // head-block row
                                    if (k >= 0 && k < 32) v = k > c ? Hh[k * HS + c] : (k == c ? 1.f : 0.f);
                                }
                                v4[e] = c < wp ? v * 32768.f : 0.f;
                            }
                            __half h0, l0, h1, l1, h2, l2, h3, l3;
                            split_f16(v4[0], h0, l0);
                            split_f16(v4[1], h1, l1);
                            split_f16(v4[2], h2, l2);
                            split_f16(v4[3], h3, l3);
                            const uint32_t off = (c % 8) * 16 + (r % 8) * 2 + (c / 8) * Cfg::SBO_V + (r / 8) * 128;
                            *reinterpret_cast<uint2*>(Vh + off) = pack4(h0, h1, h2, h3);
                            *reinterpret_cast<uint2*>(Vh + off + 4 * Cfg::SBO_V) = pack4(l0, l1, l2, l3);
                        }
                    }
                    umma::fence_async_smem();
                    __syncthreads();
                    // ---- G = V^T V (M = 64: [hi; lo], N = 32, K = B) ----
                    if (tid == 0) {
                        umma::fence_after_sync();
                        const uint32_t id = umma::idesc_f16(64, 32, false, false);
                        for (int kk = 0; kk < Cfg::B / 16; ++kk)
                            for (int hl = 0; hl < 2; ++hl) {
                                const uint64_t ad = umma::sdesc(smem_u32(Vh) + kk * 256, 128, Cfg::SBO_V);
                                const uint64_t bd =
                                    umma::sdesc(smem_u32(Vh) + hl * 4 * Cfg::SBO_V + kk * 256, 128, Cfg::SBO_V);
                                umma::mma_f16(tmem + Cfg::TM_G, ad, bd, id, kk > 0 || hl > 0);
                            }
                        umma::commit(mbar);
                    }
                    if (nchunk > 0) {  // first chunk's staging overlaps G (Hh / G dump live in C buffer 1)
                        int64_t cb;
                        const int n0c = chunk_cols(cid(0), &cb);
                        chain_stage<Cfg>(sm + Cfg::OFF_C, sm + Cfg::OFF_CS, A, lda, cb, n0c, s, h, slotp, wp, leaf,
                                         hr0);
                    }
                    wait_mma();
                    {  // TMEM (M = 64 layout: warp w, lanes < 16 = rows 16w + l) -> G dump [64][HS]
                        float v[16];
                        const int row = 16 * warp + lane;
                        umma::tmem_ld16(tmem + ((uint32_t)(32 * warp) << 16) + Cfg::TM_G, v);
                        if (lane < 16)
#pragma unroll
                            for (int j = 0; j < 16; ++j) Gs[row * HS + j] = v[j];
                        umma::tmem_ld16(tmem + ((uint32_t)(32 * warp) << 16) + Cfg::TM_G + 16, v);
                        if (lane < 16)
#pragma unroll
                            for (int j = 0; j < 16; ++j) Gs[row * HS + 16 + j] = v[j];
                    }
                    __syncthreads();
                    for (int e = tid; e < 32 * 32; e += Cfg::NT) {  // G = (hi rows + lo rows) 2^-30
                        const int i = e >> 5, j = e & 31;
                        Gs[i * HS + j] = (Gs[i * HS + j] + Gs[(i + 32) * HS + j]) * 0x1p-30f;
                    }
                    __syncthreads();
                    if (tid < 32) chain_build_t(Gs, taus, wp, Ts, Tws + (t * g.npan + p) * (kPW * kPW), HS);
                    CHAIN_PROF(2);
                    // ---- trailing chunks ----
                    for (int ib = 0; ib < nchunk; ++ib) {
                        int64_t cb0;
                        const int ncb = chunk_cols(cid(ib), &cb0);
                        float* Cs = sm + Cfg::OFF_C + (ib & 1) * CW * VP;
                        float* Csl = sm + Cfg::OFF_CS + (ib & 1) * CW * 32;
                        asm volatile("cp.async.wait_group 0;" ::: "memory");
                        __syncthreads();  // chunk ib staged; previous chunk's epilogue done; T ready
                        if (ib + 1 < nchunk) {  // prefetch the next chunk into the other buffer
                            int64_t cb1;
                            const int n1c = chunk_cols(cid(ib + 1), &cb1);
                            chain_stage<Cfg>(sm + Cfg::OFF_C + ((ib + 1) & 1) * CW * VP,
                                             sm + Cfg::OFF_CS + ((ib + 1) & 1) * CW * 32, A, lda, cb1, n1c, s, h, slotp,
                                             wp, leaf, hr0);
                        }
                        CHAIN_PROF(3);
                        // C -> fp16 hi | lo with a power-of-two scale per column (K-major B of W = V^T C)
                        {
                            const int cc = tid >> 3, u0 = tid & 7;
                            constexpr int NQ4 = Cfg::B / 4;
                            float vals[(NQ4 + 7) / 8][4];
                            float m = 0.f;
#pragma unroll
                            for (int k2 = 0; k2 < (NQ4 + 7) / 8; ++k2) {
                                const int u = u0 + 8 * k2;
                                float4 f = make_float4(0.f, 0.f, 0.f, 0.f);
                                if (u < NQ4) f = *reinterpret_cast<const float4*>(Cs + (size_t)cc * VP + 4 * u);
                                vals[k2][0] = f.x;
                                vals[k2][1] = f.y;
                                vals[k2][2] = f.z;
                                vals[k2][3] = f.w;
                                m = fmaxf(m, fmaxf(fmaxf(fabsf(f.x), fabsf(f.y)), fmaxf(fabsf(f.z), fabsf(f.w))));
                            }
                            m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 1));
                            m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 2));
                            m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 4));
                            const int ex = col_exp(m);
                            const float sc = pow2f(ex);
                            if (u0 == 0) cscale[cc] = pow2f(-ex - 15);  // unscale of W: 2^-(15+e)
#pragma unroll
                            for (int k2 = 0; k2 < (NQ4 + 7) / 8; ++k2) {
                                const int u = u0 + 8 * k2;
                                if (u < NQ4) {
                                    const int r = 4 * u;
                                    __half h0, l0, h1, l1, h2, l2, h3, l3;
                                    split_f16(vals[k2][0] * sc, h0, l0);
                                    split_f16(vals[k2][1] * sc, h1, l1);
                                    split_f16(vals[k2][2] * sc, h2, l2);
                                    split_f16(vals[k2][3] * sc, h3, l3);
                                    const uint32_t off =
                                        (cc % 8) * 16 + (r % 8) * 2 + (cc / 8) * Cfg::SBO_C + (r / 8) * 128;
                                    *reinterpret_cast<uint2*>(Ch + off) = pack4(h0, h1, h2, h3);
                                    *reinterpret_cast<uint2*>(Ch + CW * Cfg::B * 2 + off) = pack4(l0, l1, l2, l3);
                                }
                            }
                        }
                        umma::fence_async_smem();
                        __syncthreads();
                        // ---- W = V^T C (M = 64 [hi; lo] x N = CW, K = B) ----
                        if (tid == 0) {
                            umma::fence_after_sync();
                            const uint32_t id = umma::idesc_f16(64, CW, false, false);
                            for (int kk = 0; kk < Cfg::B / 16; ++kk)
                                for (int hl = 0; hl < 2; ++hl) {
                                    const uint64_t ad = umma::sdesc(smem_u32(Vh) + kk * 256, 128, Cfg::SBO_V);
                                    const uint64_t bd = umma::sdesc(smem_u32(Ch) + hl * CW * Cfg::B * 2 + kk * 256,
                                                                    128, Cfg::SBO_C);
                                    umma::mma_f16(tmem + Cfg::TM_W, ad, bd, id, kk > 0 || hl > 0);
                                }
                            umma::commit(mbar);
                        }
                        wait_mma();
                        CHAIN_PROF(6);
                        float* Wd = sm + Cfg::OFF_CH;  // W dump [64][WS2] over the (consumed) fp16 C
                        {
                            float v[16];
                            umma::tmem_ld16(tmem + ((uint32_t)(32 * warp) << 16) + Cfg::TM_W, v);
                            __syncwarp();
                            if (lane < 16)
#pragma unroll
                                for (int j = 0; j < 16; ++j) Wd[(16 * warp + lane) * Cfg::WS2 + j] = v[j];
                        }
                        __syncthreads();
                        // W (rows 0..31) = (hi rows + lo rows) / (2^15 scale) (+ C_slot)
                        for (int e = tid; e < 32 * CW; e += Cfg::NT) {
                            const int i = e / CW, n = e % CW;
                            float w = (Wd[i * Cfg::WS2 + n] + Wd[(i + 32) * Cfg::WS2 + n]) * cscale[n];
                            if (!leaf) w += Csl[n * 32 + i];
                            Wd[i * Cfg::WS2 + n] = w;
                        }
                        __syncthreads();
                        chain_gemm_tw_s<Cfg::HS, Cfg::WS2>(Ts, Wd, Wd + 32 * Cfg::WS2);  // W2 (rows 32..63 of the dump)
                        __syncthreads();
                        // W2 -> C_slot update; fp16 hi | lo with a per-column scale (K-major B of dC = V W2)
                        {
                            const int n = tid >> 3, i0 = 4 * (tid & 7);
                            float w2[4];
                            float m = 0.f;
#pragma unroll
                            for (int u = 0; u < 4; ++u) {
                                w2[u] = Wd[(32 + i0 + u) * Cfg::WS2 + n];
                                m = fmaxf(m, fabsf(w2[u]));
                                if (!leaf) Csl[n * 32 + i0 + u] -= w2[u];
                            }
                            m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 1));
                            m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 2));
                            m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 4));
                            const int ex = col_exp(m);
                            const float sc = pow2f(ex);
                            if ((tid & 7) == 0) wscale[n] = pow2f(-ex - 15);  // unscale of dC: 2^-(15+e)
                            __half h0, l0, h1, l1, h2, l2, h3, l3;
                            split_f16(w2[0] * sc, h0, l0);
                            split_f16(w2[1] * sc, h1, l1);
                            split_f16(w2[2] * sc, h2, l2);
                            split_f16(w2[3] * sc, h3, l3);
                            const uint32_t off = (n % 8) * 16 + (i0 % 8) * 2 + (n / 8) * 512 + (i0 / 8) * 128;
                            *reinterpret_cast<uint2*>(W2h + off) = pack4(h0, h1, h2, h3);
                            *reinterpret_cast<uint2*>(W2h + CW * 32 * 2 + off) = pack4(l0, l1, l2, l3);
                        }
                        umma::fence_async_smem();
                        __syncthreads();
                        CHAIN_PROF(7);
                        // ---- dC = V W2 (A = V MN-major, row blocks of 128 (+ 64); 3 products) ----
                        if (tid == 0) {
                            umma::fence_after_sync();
                            constexpr int NB = (Cfg::B + 127) / 128;
                            for (int mb = 0; mb < NB; ++mb) {
                                const int mrows = min(128, Cfg::B - 128 * mb);
                                const uint32_t id = umma::idesc_f16(mrows, CW, true, false);
                                const uint32_t dcol = mb == 0 ? Cfg::TM_D1 : Cfg::TM_D2;
                                bool acc = false;
#pragma unroll
                                for (int pr = 0; pr < 3; ++pr) {
                                    const int ah = pr == 2 ? 1 : 0, bh = pr == 1 ? 1 : 0;  // (hi,hi) (hi,lo) (lo,hi)
                                    for (int kk = 0; kk < 2; ++kk) {
                                        const uint64_t ad = umma::sdesc(smem_u32(Vh) + mb * 16 * 128 + ah * 4 * Cfg::SBO_V +
                                                                            kk * 2 * Cfg::SBO_V,
                                                                        Cfg::SBO_V, 128);
                                        const uint64_t bd =
                                            umma::sdesc(smem_u32(W2h) + bh * CW * 32 * 2 + kk * 256, 128, 512);
                                        umma::mma_f16(tmem + dcol, ad, bd, id, acc);
                                        acc = true;
                                    }
                                }
                            }
                            umma::commit(mbar);
                        }
                        wait_mma();
                        CHAIN_PROF(4);
                        // ---- epilogue: C -= dC (rows: TMEM lanes), store tile rows + slot rows ----
                        {
                            auto rows_out = [&](int row, const float (&v)[16]) {
                                const bool rok = row < h && !(leaf && row < hr0);
                                float* gp = A + cb0 * lda + s + row;  // column cb0, this row; += lda per column
#pragma unroll
                                for (int n = 0; n < CW; ++n) {
                                    const float cn = fmaf(-v[n], wscale[n], Cs[(size_t)n * VP + row]);
                                    Cs[(size_t)n * VP + row] = cn;
                                    if (rok && n < ncb) __stcg(gp, cn);
                                    gp += lda;
                                }
                            };
                            float v[16];
                            umma::tmem_ld16(tmem + ((uint32_t)(32 * warp) << 16) + Cfg::TM_D1, v);
                            rows_out(32 * warp + lane, v);
                            if constexpr (Cfg::B > 128) {
                                umma::tmem_ld16(tmem + ((uint32_t)(32 * warp) << 16) + Cfg::TM_D2, v);
                                if constexpr (Cfg::B - 128 >= 128) {
                                    rows_out(128 + 32 * warp + lane, v);
                                } else {
                                    if (lane < 16) rows_out(128 + 16 * warp + lane, v);
                                }
                            }
                            if (!leaf)
                                for (int e = tid; e < CW * 32; e += Cfg::NT) {
                                    const int n = e >> 5, i = e & 31;
                                    if (n < ncb && i < wp) A[(cb0 + n) * lda + slotp + i] = Csl[n * 32 + i];
                                }
                        }
                        umma::fence_before_sync();
                        __syncthreads();
                        CHAIN_PROF(8);
                    }
                } else {
                __syncthreads();
                    chain_gemm_gram<Cfg>(Vs, Gs);  // G = V^T V (tile part)
                    __syncthreads();
                    if (tid < 32) chain_build_t(Gs, taus, wp, Ts, Tws + (t * g.npan + p) * (kPW * kPW), HS);
    
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
                        chain_gemm_vtc<Cfg>(Vs, Cs, Csl, !leaf, sm + Cfg::OFF_W);
                        __syncthreads();
                        chain_gemm_tw<Cfg>(Ts, sm + Cfg::OFF_W, sm + Cfg::OFF_W2);
                        __syncthreads();
                        if (!leaf)  // slot rows: C_slot -= W2 (V's head part is the identity)
                            for (int e = tid; e < CW * 32; e += Cfg::NT) {
                                const int cc = e >> 5, i = e & 31;
                                Csl[cc * 32 + i] -= sm[Cfg::OFF_W2 + i * Cfg::WS + cc];
                            }
                        chain_gemm_update<Cfg>(Vs, Cs, sm + Cfg::OFF_W2);
                        __syncthreads();
                        CHAIN_PROF(4);
                        chain_store<Cfg>(Cs, Csl, A, lda, cb0, ncb, s, h, slotp, wp, leaf, hr0);
                        if (ib + 1 < nchunk) __syncthreads();
                    }
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
        for (int k = 0; k < 10; ++k) atomicAdd(prof + k, pacc[k]);
    if constexpr (TC) {  // every MMA has completed (each chunk waited on its commit)
        umma::fence_before_sync();
        __syncthreads();
        if (threadIdx.x < 32) umma::tmem_free<128>(s_tmem);
    }
#undef CHAIN_PROF
}

template <int NQ, int SEG>
inline size_t chain_smem_bytes() {
    return ChainCfg<NQ, SEG>::BYTES;
}

}  // namespace caqr
