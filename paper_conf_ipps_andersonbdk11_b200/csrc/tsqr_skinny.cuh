// tsqr_skinny.cuh -- TSQR of a skinny panel group (n <= 16, fp32) with one
// WARP per task.
//
// For the s-step Krylov shape ("millions of rows by less than ten
// columns") the whole problem is a stream of A through HBM; a 256-thread CTA
// per chain of 8-column panels leaves the machine idle.  Here every task --
// a chain of tiles ([chain R; tile] steps, "any tree shape") or a
// merge of two n x n R factors -- is one warp: the gathered rows
// live in registers (lane l holds rows l + 32 i), each Householder reflector
// is a warp reduction, and ~2,000 chains keep enough loads in
// flight to run at HBM speed.  Same plan and representation as the block
// kernels (node_rows), so apply_qt / form_q are shared.
#pragma once
#include "tsqr_fused.cuh"

namespace caqr {

constexpr int kSkinnyWarps = 4;  // warps per CTA

// One node (one panel: the group has a single <= NC-column panel) by one warp.
template <int NC, int NR>
__device__ __forceinline__ void skinny_node(const Geom& g, float* A, float* Tws, int level, int64_t node, int kt,
                                            float* scr) {
    const int lane = threadIdx.x & 31;
    const int wp = g.ncols;
    const NodeRows nr = node_rows(g, level, node, 0, wp, kt);
    const int RG = nr.n0 + nr.n1;
    if (RG == 0) return;
    const int64_t c0 = g.col0;
    float x[NR][NC];
    // all loads first (memory-level parallelism), through L2 (cross-SM data)
#pragma unroll
    for (int i = 0; i < NR; ++i) {
        const int r = lane + 32 * i;
        const int64_t row = r < RG ? gathered_row(nr, r) : 0;
#pragma unroll
        for (int c = 0; c < NC; ++c)
            x[i][c] = (r < RG && c < wp && panel_entry_stored(nr, r, c, 0))
                          ? __ldcg(A + (c0 + c) * g.lda + row)
                          : 0.f;
    }
    float tau[NC];
#pragma unroll
    for (int j = 0; j < NC; ++j) {
        tau[j] = 0.f;
        if (j >= wp) continue;
        float sg = 0.f;
#pragma unroll
        for (int i = 0; i < NR; ++i) {
            const int r = lane + 32 * i;
            sg = (r > j) ? fmaf(x[i][j], x[i][j], sg) : sg;
        }
        const float al = __shfl_sync(0xffffffffu, x[0][j], j);
        sg = warp_sum(sg);
        float t = 0.f, beta = al, scale = 1.f;
        if (j < RG && sg > 0.f) {
            const float ss = fmaf(al, al, sg);
            const float aa = fabsf(al);
            float rmu, mu;
            rsqrt_refined(ss, rmu, mu);
            beta = -copysignf(mu, al);
            t = fmaf(aa, rmu, 1.f);
            scale = copysignf(rcp_refined(aa + mu), al);
        }
        tau[j] = t;
        float v[NR];
#pragma unroll
        for (int i = 0; i < NR; ++i) {
            const int r = lane + 32 * i;
            if (r > j) x[i][j] *= scale;
            if (r == j) x[i][j] = beta;
            v[i] = r > j ? x[i][j] : (r == j ? 1.f : 0.f);
        }
        if (t != 0.f && j + 1 < wp) {
            float d[NC];
#pragma unroll
            for (int k = 0; k < NC; ++k) {
                d[k] = 0.f;
                if (k > j)
#pragma unroll
                    for (int i = 0; i < NR; ++i) d[k] = fmaf(v[i], x[i][k], d[k]);
            }
            warp_reduce_many<NC>(d, scr);
#pragma unroll
            for (int k = 0; k < NC; ++k)
                if (k > j) {
                    const float st = t * d[k];
#pragma unroll
                    for (int i = 0; i < NR; ++i) x[i][k] = fmaf(-st, v[i], x[i][k]);
                }
        }
    }
    // compact-WY T: G = V^T V (strict upper part), then the xLARFT recurrence
    constexpr int NG = NC * (NC - 1) / 2;
    float gv[NG];
    {
        int e = 0;
#pragma unroll
        for (int a = 0; a < NC; ++a)
#pragma unroll
            for (int b = a + 1; b < NC; ++b, ++e) {
                float s = 0.f;
#pragma unroll
                for (int i = 0; i < NR; ++i) {
                    const int r = lane + 32 * i;
                    const float va = r > a ? x[i][a] : (r == a ? 1.f : 0.f);
                    const float vb = r > b ? x[i][b] : (r == b ? 1.f : 0.f);
                    s = fmaf(va, vb, s);
                }
                gv[e] = s;
            }
    }
    // reduce in chunks of <= 32 values through the warp scratch
#pragma unroll
    for (int base = 0; base < NG; base += 32) {
        constexpr int CH = NG < 32 ? NG : 32;
        float tmp[CH];
#pragma unroll
        for (int k = 0; k < CH; ++k) tmp[k] = (base + k < NG) ? gv[base + k] : 0.f;
        warp_reduce_many<CH>(tmp, scr);
#pragma unroll
        for (int k = 0; k < CH; ++k)
            if (base + k < NG) gv[base + k] = tmp[k];
    }
    // lane i < wp computes row i of T (registers), writes the wp x wp block
    {
        float row[NC];
#pragma unroll
        for (int j = 0; j < NC; ++j) {
            float acc = 0.f;
#pragma unroll
            for (int k = 0; k < j; ++k) {
                // g_kj with k < j sits at index k*NC - k(k+1)/2 + (j - k - 1)
                const int e = k * NC - k * (k + 1) / 2 + (j - k - 1);
                acc = fmaf(row[k], gv[e], acc);
            }
            row[j] = (j == lane) ? tau[j] : (j > lane ? -tau[j] * acc : 0.f);
        }
        float* tb = Tws + nr.tblk * (kPW * kPW);
        if (lane < wp)
#pragma unroll
            for (int j = 0; j < NC; ++j)
                if (j < wp) tb[j * kPW + lane] = row[j];  // column-major 32x32 slot, wp x wp used
    }
    // write back R / V (structure masks keep the neighbours' data intact)
#pragma unroll
    for (int i = 0; i < NR; ++i) {
        const int r = lane + 32 * i;
        if (r < RG) {
            const int64_t row = gathered_row(nr, r);
#pragma unroll
            for (int c = 0; c < NC; ++c)
                if (c < wp && panel_entry_stored(nr, r, c, 0)) A[(c0 + c) * g.lda + row] = x[i][c];
        }
    }
}

template <int NC, int NR>
__global__ void __launch_bounds__(32 * kSkinnyWarps, 4)
tsqr_skinny_kernel(Geom g, float* A, float* __restrict__ Tws, int* __restrict__ sync, int nlevels, int do_leaves) {
    constexpr int NP = NC <= 8 ? 8 : 16;
    __shared__ __align__(16) float scr_all[kSkinnyWarps][32 * (32 + 4) + 32];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    float* scr = scr_all[warp];
    (void)NP;
    int* ticket = sync;
    int* flags = sync + 32;
    const int64_t leaf_tasks = do_leaves ? g.P : 0;
    int64_t total = leaf_tasks;
    for (int l = 0; l < nlevels; ++l) {
        const int64_t h = int64_t(1) << l;
        total += (g.P - 1 >= h) ? (g.P - 1 - h) / (2 * h) + 1 : 0;
    }
    for (;;) {
        int tk = 0;
        if (lane == 0) tk = atomicAdd(ticket, 1);
        const int64_t task = __shfl_sync(0xffffffffu, tk, 0);
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
        int64_t slot_a = node;
        if (level >= 0) {
            slot_a = node << (level + 1);
            const int64_t slot_b = slot_a + (int64_t(1) << level);
            if (lane == 0) {
                const int va = expected_version(slot_a, level, g.P, do_leaves);
                const int vb = expected_version(slot_b, level, g.P, do_leaves);
                while (ld_acquire(flags + slot_a * g.npan) < va) __nanosleep(32);
                while (ld_acquire(flags + slot_b * g.npan) < vb) __nanosleep(32);
            }
            __syncwarp();
        }
        const int64_t ntile = level < 0 ? min(g.K, g.L - node * g.K) : 1;
        for (int kt = 0; kt < ntile; ++kt) {
            skinny_node<NC, NR>(g, A, Tws, level, node, kt, scr);
            __syncwarp();  // this warp's global writes are read back by its next tile
        }
        __threadfence();
        __syncwarp();
        if (lane == 0) st_release(flags + slot_a * g.npan, level < 0 ? 1 : level + 2);
    }
}

}  // namespace caqr
