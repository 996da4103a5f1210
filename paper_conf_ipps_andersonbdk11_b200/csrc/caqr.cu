#include <cstdio>
// caqr.cu -- host planner + C ABI of libcaqr.so (declared in include/caqr.h).
//
// The host side is the paper's "CPU coordinates the GPU's actions and updates
// pointers" (Sec. IV.B): it walks the plan -- panel groups, leaf
// panels, tree levels (Fig. 4) -- and enqueues kernels on the
// caller's stream.  No host synchronisation, no device allocation.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

#include "../../include/caqr.h"
#include "tsqr_fused.cuh"
#include "tsqr_chain.cuh"
#include "tsqr_kernels.cuh"
#include "tsqr_skinny.cuh"
#include "rpca.cuh"
#include "tsqr_stream_apply.cuh"
#include "tsqr_stream.cuh"

namespace caqr {

static thread_local int g_last_cuda_error = 0;

// ---- launch tracing (diagnostics: per-launch CUDA events on the launching
// stream + host-computed algorithmic flops/bytes; see caqr_trace_begin) -------
enum KernelId { K_PANEL_FACTOR = 0, K_PANEL_UPDATE = 1, K_EXTRACT_R = 2, K_SET_IDENTITY = 3,
                K_TSQR_FUSED = 4, K_TSQR_SKINNY = 5, K_SVD_SMALL = 6, K_SVT_CORE = 7, K_EMBED_TOP = 8,
                K_RPCA_UPDATE = 9, K_RPCA_INIT = 10, K_ABSMAX = 11, K_CHAIN_UPDATE = 12, K_STREAM_APPLY = 13,
                K_TRSM = 14, K_TSQR_CHAIN = 15, K_APPLY_ALL = 16, K_NUM = 17 };
static const char* const kKernelNames[K_NUM] = {"panel_factor", "panel_update", "extract_r", "set_identity",
                                                "tsqr_fused",   "tsqr_skinny",  "svd_small", "svt_core",
                                                "embed_top",    "rpca_update",  "rpca_init", "absmax",
                                                "node_update",  "stream_apply", "trsm_upper",
                                                "tsqr_chain",   "node_update_all"};
struct Trace {
    std::mutex mu;
    bool on = false;
    int cap = 0, n = 0;
    cudaEvent_t* ev = nullptr;
    int* kid = nullptr;
    double* flops = nullptr;
    double* bytes = nullptr;
};
static Trace g_trace;
struct TraceScope {  // records a start event now and a stop event at destruction
    int slot = -1;
    cudaStream_t s;
    TraceScope(int k, double fl, double by, cudaStream_t st) : s(st) {
        if (!g_trace.on) return;
        std::lock_guard<std::mutex> lk(g_trace.mu);
        if (!g_trace.on || g_trace.n >= g_trace.cap) return;
        slot = g_trace.n++;
        g_trace.kid[slot] = k;
        g_trace.flops[slot] = fl;
        g_trace.bytes[slot] = by;
        cudaEventRecord(g_trace.ev[2 * slot], s);
    }
    ~TraceScope() {
        if (slot >= 0) cudaEventRecord(g_trace.ev[2 * slot + 1], s);
    }
};

constexpr int64_t kMaxGroup = 256;    // widest single TSQR panel group
constexpr int64_t kMaxLeaf = 256;     // tallest tile the kernels stage in shared memory
constexpr int64_t kFusedLeaf = 224;   // default tile height: [32 R rows; tile] fits 256 rows
constexpr int64_t kChainTarget = 296; // chains per group (2 per B200 SM; device-independent constant)
constexpr int64_t kStreamChains = 1184;  // skinny chains: 8 warps x 148 B200 SMs
// CAQR_STREAM16=1: n <= 8 panels on 128-row tiles with 16 warps per SM
// (2368 chains) instead of 256-row tiles with 8 warps per SM.
static inline bool stream16_policy() {
    const char* e = getenv("CAQR_STREAM16");
    return e && e[0] == '1';
}
// n <= 8 panels on 256-row tiles: 16 warps per SM with one tile buffer each
// (default) or 8 warps with two (CAQR_STREAM_W16B=0).
static inline bool stream_w16b_policy() {
    const char* e = getenv("CAQR_STREAM_W16B");
    return !(e && e[0] == '0');
}

struct Plan {
    int64_t m = 0, n = 0;
    int dtype = 0;
    int64_t b = 0;   // leaf height
    int64_t nb = 0;  // panel-group width
    int64_t ngroups = 0;
    int64_t chain_target = 296;  // chains per group (tree leaves)
    bool skinny = false;         // warp-per-task skinny kernel (fp32, n <= 16)
    bool chain = false;          // chain kernel + merge-only fused tree (fp32, 16 < n <= 256)
};

static inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Chain kernel policy (CAQR_CHAIN=1: the chain kernel does the chains, the
// fused kernel the tree; default: the fused kernel does both) and its tile height: 128 / 192 / 256 rows (>= n: the chain R lives in
// the first tile's top n rows).  Read per call so tests can compare paths.
static inline bool chain_policy() {
    const char* e = getenv("CAQR_CHAIN");
    return e && e[0] == '1';
}
static inline int64_t chain_tile_rows(int64_t n) { return n <= 128 ? 128 : (n <= 192 ? 192 : 256); }
constexpr int64_t kChainTarget2 = 444;  // chains: 3 per B200 SM (device-independent constant)
static inline int64_t round_up(int64_t a, int64_t b) { return ceil_div(a, b) * b; }

// Returns 0, or the info code of the offending argument position `opt_pos`.
static int make_plan(int64_t m, int64_t n, int dtype, const caqr_opts* o, int opt_pos, Plan* pl) {
    pl->m = m;
    pl->n = n;
    pl->dtype = dtype;
    // default group width: the whole matrix for n <= 224 (one TSQR); 128 for
    // n in (224, 256] -- a 256-wide group's top tree merges need 2*32 + 224 =
    // 288 > 256 gathered rows, which only the per-level split path takes (SURVEY
    // 8(f) f3: 8192 x 256 was 6 ms that way, vs two 128-wide CAQR groups);
    // 128-wide CAQR groups beyond (round 2: caqr_tune's search put (b, nb) =
    // (256, 128) first or within a few % on every wide shape measured --
    // 8192^2 68.8 vs 75.6 ms for nb = 64, 4096^2 f64 29.0 vs 32.5 ms,
    // profiles/round2_measurements.txt)
    int64_t nb = (o && o->panel_cols > 0) ? o->panel_cols : (n <= 224 ? n : 128);
    if (nb > kMaxGroup) return -opt_pos;
    nb = std::max<int64_t>(1, std::min(nb, std::max<int64_t>(n, 1)));
    // skinny fp32 panels (n <= 16, one group): one warp per chain, 256-row (n <= 8)
    // or 128-row (n <= 16) tiles, ~1,100 chains (tsqr_stream.cuh).  With the
    // arrival-counter tree it wins from m = 4096 up (measured 4096 x 16: 0.099 vs
    // 0.139 ms for the block kernel; 65536 x 8: 0.078 vs 0.169; 200000 x 8: 0.095
    // vs 0.207), so every m >= 1024 takes it.
    static const int64_t skinny_min_m = [] {  // diagnostics: CAQR_SKINNY_MIN_M overrides the threshold
        const char* e = getenv("CAQR_SKINNY_MIN_M");
        return e ? (int64_t)atoll(e) : int64_t(1024);
    }();
    pl->skinny = dtype == CAQR_F32 && n <= 16 && nb >= n && m >= skinny_min_m;
    // streaming kernel: one chain per warp, 8 warps per SM (148 SMs)
    const bool s16 = pl->skinny && n <= 8 && stream16_policy();
    const bool w16 = pl->skinny && n <= 8 && (s16 || stream_w16b_policy());
    pl->chain_target = pl->skinny ? (w16 ? 2 * kStreamChains : kStreamChains) : kChainTarget;
    if (const char* e = getenv("CAQR_CHAIN_TARGET"))  // diagnostics: chains per group (tile sweep)
        pl->chain_target = std::max<int64_t>(1, atoll(e));
    // fp32 whole-width groups (16 < n <= 256): the chain kernel (tsqr_chain.cuh),
    // tiles of 128 / 192 / 256 rows (>= n), ~3 chains per SM
    pl->chain = dtype == CAQR_F32 && !pl->skinny && nb == n && n > 16 && n <= 256 && chain_policy() &&
                !(o && o->leaf_rows > 0 && o->leaf_rows != chain_tile_rows(n));
    if (pl->chain && !getenv("CAQR_CHAIN_TARGET")) pl->chain_target = kChainTarget2;
    int64_t b = (o && o->leaf_rows > 0) ? o->leaf_rows
                                        : pl->chain ? chain_tile_rows(n)
                                        : (pl->skinny ? (n <= 8 && !s16 ? 256 : 128)
                                                      : (nb <= kFusedLeaf && (n <= 224 || ceil_div(m, kMaxLeaf) >
                                                                                              pl->chain_target)
                                                             ? kFusedLeaf
                                                             : kMaxLeaf));
    // (256-row tiles only when every chain is one tile: a chain step of a
    // 256-row tile gathers 288 rows, beyond the fused kernel, so tall groups
    // of a 224 < n <= 256 matrix would fall back to the split path --
    // measured 1M x 256: 31.6 ms with b = 256 vs 1M x 192: 5.3 ms)
    if (b % 32 != 0 || b > kMaxLeaf) return -opt_pos;
    b = std::max(b, round_up(nb, 32));
    if (b > kMaxLeaf) return -opt_pos;
    pl->nb = nb;
    pl->b = b;
    pl->ngroups = n == 0 ? 0 : ceil_div(n, nb);
    return 0;
}

static Geom group_geom(const Plan& pl, int64_t g, int64_t lda) {
    Geom G;
    G.lda = lda;
    G.col0 = g * pl.nb;
    G.row0 = G.col0;
    G.mrows = pl.m - G.row0;
    G.ncols = (int32_t)std::min(pl.nb, pl.n - G.col0);
    G.npan = (int32_t)ceil_div(G.ncols, kPW);
    G.b = pl.b;
    G.L = std::max<int64_t>(1, ceil_div(G.mrows, pl.b));
    G.K = ceil_div(G.L, pl.chain_target);
    G.P = ceil_div(G.L, G.K);
    G.bm = G.K * G.b;
    return G;
}

static inline int tree_levels(int64_t L) {
    int lv = 0;
    while ((int64_t(1) << lv) < L) ++lv;
    return lv;
}
static inline int64_t merges_at(int64_t L, int level) {
    const int64_t h = int64_t(1) << level;
    return (L - 1 >= h) ? (L - 1 - h) / (2 * h) + 1 : 0;
}
// Workspace of one panel group: T blocks [L + P][npan][32][32] (tile T's, then
// merge T's indexed by the merge's right member's slot), then the fused kernel's
// ticket + per-(slot, panel) ready flags.
static inline size_t group_t_bytes(const Geom& G, size_t es) {
    // one 32 x 32 T per (tile, panel), then one per (merge, panel) indexed by
    // the merge's right member (a chain slot, < P)
    return (size_t)(G.L + G.P) * G.npan * kPW * kPW * es;
}
static inline size_t group_sync_bytes(const Geom& G) {
    int64_t ints = 32 + G.L * G.npan;
    // skinny groups: room for the streaming kernel's cross-CTA exchange area
    // (one n x n R per CTA at sync + 64) and arrival counters (tsqr_stream.cuh)
    if (G.npan == 1 && ((G.ncols <= 8 && (G.b == 256 || G.b == 128)) || (G.ncols <= 16 && G.b == 128))) {
        const int64_t nct = ceil_div(G.P, 8);  // CTAs of 8 (or 16) warps
        const int64_t rx = G.ncols <= 8 ? stream_rx_ints<float, 8>(nct) : stream_rx_ints<float, 16>(nct);
        ints = std::max<int64_t>(ints, 64 + rx + 16 * nct);
    }
    return (size_t)round_up(ints * (int64_t)sizeof(int), 256);
}
static inline size_t group_ws_bytes(const Geom& G, size_t es) {
    return group_t_bytes(G, es) + group_sync_bytes(G);
}

static size_t plan_ws_bytes(const Plan& pl) {
    size_t bytes = 0;
    const size_t es = pl.dtype == CAQR_F64 ? 8 : 4;
    for (int64_t g = 0; g < pl.ngroups; ++g) bytes += group_ws_bytes(group_geom(pl, g, pl.m), es);
    return bytes;
}

// Can the persistent fused kernel take this group?  Every task's gathered rows
// must fit its 256-row register layout: leaves (b rows) and merges (2 wp + 32 p).
static bool fused_ok(const Geom& G) {
    if (G.b > kFusedMaxRows) return false;
    if (G.K > 1 && 32 + G.b > kFusedMaxRows) return false;  // [chain R; tile] nodes
    for (int p = 0; p < G.npan; ++p) {
        const int wp = std::min<int>(kPW, G.ncols - 32 * p);
        if (2 * wp + 32 * p > kFusedMaxRows) return false;
    }
    return true;
}
static int num_sms() {
    static int cache[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 64 && cache[dev]) return cache[dev];
    int n = 148;
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (dev < 64) cache[dev] = n;
    return n;
}

// ---- launch helpers ---------------------------------------------------------

// Host replica of node_rows()'s gathered-row count (trace bookkeeping only).
static int64_t node_rg(const Geom& G, int level, int64_t node, int p, int wp, int kt) {
    if (level < 0) {
        const int64_t t = node * G.K + kt;
        if (t >= G.L) return 0;
        const int64_t h = std::min(G.b, G.mrows - t * G.b);
        return kt == 0 ? std::max<int64_t>(0, h - 32 * p) : wp + h;
    }
    const int64_t a = node << (level + 1), bb = a + (int64_t(1) << level);
    const int64_t hb = std::min(G.b, G.mrows - bb * G.bm);
    return wp + std::min<int64_t>(32 * p + wp, hb);
}
// Algorithmic work of one launch: Householder QR of each node's gathered
// RG x wp panel (LAPACK count) / the two GEMMs of the blocked update
// (4 RG wp ccount); bytes = the panel / C block read and written once (+ V).
static void trace_counts(const Geom& G, int level, int p, int kt, int64_t nodes, bool update,
                         int64_t ccount, size_t es, double* fl, double* by) {
    *fl = 0;
    *by = 0;
    if (!g_trace.on) return;
    const int wp = std::min<int>(kPW, G.ncols - 32 * p);
    for (int64_t nd = 0; nd < nodes; ++nd) {
        const double rg = (double)node_rg(G, level, nd, p, wp, kt);
        const double k = std::min<double>(rg, wp);
        if (!update) {
            *fl += 2.0 * rg * wp * k - 2.0 / 3.0 * k * k * k;
            *by += 2.0 * rg * wp * es;
        } else {
            *fl += 4.0 * rg * wp * ccount;
            *by += (2.0 * rg * ccount + rg * wp) * es;
        }
    }
}
// Opt a kernel into > 48 KB of dynamic shared memory, once per (kernel, device).
static cudaError_t allow_smem_ptr(const void* kernel, size_t bytes) {
    if (bytes <= 48 * 1024) return cudaSuccess;
    static std::mutex mu;
    static const void* keys[256];
    static int devs[256];
    static int nkeys = 0;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lk(mu);
    for (int i = 0; i < nkeys; ++i)
        if (keys[i] == kernel && devs[i] == dev) return cudaSuccess;
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, kernel);
    if (e != cudaSuccess) return e;
    const int maxdyn = optin - (int)fa.sharedSizeBytes;
    if (maxdyn < (int)bytes) return cudaErrorInvalidValue;
    e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, maxdyn);
    if (e == cudaSuccess && nkeys < 256) {
        keys[nkeys] = kernel;
        devs[nkeys] = dev;
        ++nkeys;
    }
    return e;
}
template <typename K>
static cudaError_t allow_smem(K kernel, size_t bytes) {
    return allow_smem_ptr(reinterpret_cast<const void*>(kernel), bytes);
}
// Resident CTAs per SM of (kernel, threads, dynamic smem) on the current
// device, cached (the runtime query costs tens of microseconds of host time
// per call -- as much as a small factorisation's device time).
static cudaError_t occupancy_ptr(int* occ, const void* kernel, int threads, size_t smem) {
    struct Key {
        const void* k;
        int dev, threads;
        size_t smem;
        int occ;
    };
    static std::mutex mu;
    static Key keys[256];
    static int nkeys = 0;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lk(mu);
    for (int i = 0; i < nkeys; ++i)
        if (keys[i].k == kernel && keys[i].dev == dev && keys[i].threads == threads && keys[i].smem == smem) {
            *occ = keys[i].occ;
            return cudaSuccess;
        }
    const cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kernel, threads, smem);
    if (e == cudaSuccess && nkeys < 256) keys[nkeys++] = Key{kernel, dev, threads, smem, *occ};
    return e;
}
template <typename K>
static cudaError_t occupancy(int* occ, K kernel, int threads, size_t smem) {
    return occupancy_ptr(occ, reinterpret_cast<const void*>(kernel), threads, smem);
}

template <typename T>
static int launch_factor(const Geom& G, T* A, T* Tws, int level, int p, int kt, int64_t nodes,
                         cudaStream_t s) {
    if (nodes <= 0) return 0;
    const int wp = std::min<int>(kPW, G.ncols - 32 * p);
    const int rgmax = level < 0 ? (kt == 0 ? (int)std::min<int64_t>(G.b, G.mrows) : wp + (int)G.b)
                                : 2 * wp + 32 * p;
    const size_t smem = panel_factor_smem<T>(wp, rgmax);
    cudaError_t e = allow_smem(panel_factor_kernel<T>, smem);
    double fl, by;
    trace_counts(G, level, p, kt, nodes, false, 0, sizeof(T), &fl, &by);
    TraceScope ts(K_PANEL_FACTOR, fl, by, s);
    if (e == cudaSuccess) {
        panel_factor_kernel<T><<<dim3((unsigned)nodes), kThreads, smem, s>>>(G, A, Tws, level, p, kt);
        e = cudaGetLastError();
    }
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}

template <typename T>
static int launch_update(const Geom& G, const T* A, const T* Tws, int level, int p, int kt,
                         int64_t nodes, T* C, int64_t ldc, int64_t cfirst, int64_t ccount, int trans,
                         cudaStream_t s, bool mma = false) {
    if (nodes <= 0 || ccount <= 0) return 0;
    const int wp = std::min<int>(kPW, G.ncols - 32 * p);
    const int rgmax = level < 0 ? (kt == 0 ? (int)std::min<int64_t>(G.b, G.mrows) : wp + (int)G.b)
                                : 2 * wp + 32 * p;
    const size_t smem = panel_update_smem<T>(rgmax);
    const bool use_mma = mma && sizeof(T) == 4;
    cudaError_t e = cudaSuccess;
    if constexpr (sizeof(T) == 4)
        e = use_mma ? allow_smem(panel_update_kernel<T, true>, smem) : allow_smem(panel_update_kernel<T, false>, smem);
    else
        e = allow_smem(panel_update_kernel<T, false>, smem);
    double fl, by;
    trace_counts(G, level, p, kt, nodes, true, ccount, sizeof(T), &fl, &by);
    TraceScope ts(K_PANEL_UPDATE, fl, by, s);
    if (e == cudaSuccess) {
        // several 32-column blocks per CTA (V and T staged once) while keeping
        // >= ~4 CTAs per SM of work
        const int64_t nblk = ceil_div(ccount, 32);
        const int64_t cpb = std::max<int64_t>(1, std::min<int64_t>(8, nodes * nblk / (4 * num_sms())));
        dim3 grid((unsigned)nodes, (unsigned)ceil_div(nblk, cpb));
        if (use_mma) {
            if constexpr (sizeof(T) == 4)
                panel_update_kernel<T, true><<<grid, kThreads, smem, s>>>(G, A, Tws, level, p, kt, C, ldc,
                                                                          cfirst, ccount, trans, (int)cpb);
        } else {
            panel_update_kernel<T, false><<<grid, kThreads, smem, s>>>(G, A, Tws, level, p, kt, C, ldc,
                                                                       cfirst, ccount, trans, (int)cpb);
        }
        e = cudaGetLastError();
    }
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}

// Q^T C / Q C node by node: one launch for every chain's tiles and panels
// (level < 0) or for one whole tree level (node_update_kernel), instead of one
// launch per (tile or level, panel).  CAQR_CHAIN_APPLY=0 restores the
// per-(tile or level, panel) launches.
static inline bool chain_apply_policy() {
    const char* e = getenv("CAQR_CHAIN_APPLY");
    return !(e && e[0] == '0');
}

// CAQR_APPLY_ALL=0: one launch per tree level (+ one for the chains) instead
// of node_update_all_kernel's single launch per group.
static inline bool apply_all_policy() {
    const char* e = getenv("CAQR_APPLY_ALL");
    return !(e && e[0] == '0');
}

// Q^T C / Q C of a group -- chains (do_leaves) and every tree level -- in one
// persistent launch (node_update_all_kernel); the tasks of each phase are
// node_update_kernel's grid.  *done = false when the group does not qualify.
template <typename T>
static int launch_node_update_all(const Geom& G, const T* A, const T* Tws, bool do_leaves, T* C, int64_t ldc,
                                  int64_t cfirst, int64_t ccount, int trans, cudaStream_t s, bool* done) {
    *done = false;
    if (!apply_all_policy()) return 0;
    *done = true;
    if (ccount <= 0) return 0;
    const int nl = tree_levels(G.P);
    std::vector<int> order;
    if (trans) {
        if (do_leaves) order.push_back(-1);
        for (int lv = 0; lv < nl; ++lv) order.push_back(lv);
    } else {
        for (int lv = nl - 1; lv >= 0; --lv) order.push_back(lv);
        if (do_leaves) order.push_back(-1);
    }
    ApplyPhases ph{};
    const int64_t nblk = ceil_div(ccount, 32);
    int rgmax = 0;
    double fl = 0, by = 0;
    for (int level : order) {
        const int64_t nodes = level < 0 ? G.P : merges_at(G.P, level);
        if (nodes <= 0) continue;
        if (ph.n >= kMaxApplyPhases) {
            *done = false;
            return 0;
        }
        const int64_t groups = std::max<int64_t>(1, std::min<int64_t>(nblk, (2 * num_sms()) / nodes));
        const int64_t cpb = ceil_div(nblk, groups);
        const int64_t gy = ceil_div(nblk, cpb);
        if ((int64_t)ph.start[ph.n] + nodes * gy > INT32_MAX / 2) {
            *done = false;
            return 0;
        }
        ph.level[ph.n] = level;
        ph.nodes[ph.n] = (int)nodes;
        ph.cpb[ph.n] = (int)cpb;
        ph.start[ph.n + 1] = ph.start[ph.n] + (int)(nodes * gy);
        ++ph.n;
        rgmax = std::max(rgmax, level < 0 ? (int)(G.K > 1 ? G.b + kPW : std::min<int64_t>(G.b, G.mrows))
                                          : (int)(kPW + std::min<int64_t>(G.ncols, G.b)));
        if (g_trace.on)
            for (int kt = 0; kt < (level < 0 ? G.K : 1); ++kt)
                for (int p = 0; p < G.npan; ++p) {
                    double f1, b1;
                    trace_counts(G, level, p, kt, nodes, true, ccount, sizeof(T), &f1, &b1);
                    fl += f1;
                    by += b1;
                }
    }
    const int total = ph.start[ph.n];
    if (total == 0) return 0;
    const size_t smem = panel_update_smem<T>(rgmax);
    cudaError_t e = allow_smem(node_update_all_kernel<T>, smem);
    int occ = 0;  // a cooperative grid: every CTA resident
    if (e == cudaSuccess)
        e = occupancy(&occ, node_update_all_kernel<T>, kThreads, smem);
    if (e == cudaSuccess && occ < 1) {
        *done = false;
        return 0;
    }
    if (e == cudaSuccess) {
        TraceScope ts(K_APPLY_ALL, fl, by, s);
        const unsigned grid = (unsigned)std::min<int64_t>(total, (int64_t)occ * num_sms());
        Geom g = G;
        const T* a = A;
        const T* tw = Tws;
        T* c = C;
        int64_t ld = ldc, cf = cfirst, cc = ccount;
        int tr = trans;
        void* args[] = {&g, &a, &tw, &c, &ld, &cf, &cc, &tr, &ph};
        e = cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(node_update_all_kernel<T>), dim3(grid),
                                        dim3(kThreads), args, smem, s);
        if (e == cudaSuccess) e = cudaGetLastError();
    }
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}

template <typename T>
static int launch_node_update(const Geom& G, const T* A, const T* Tws, int level, T* C, int64_t ldc,
                              int64_t cfirst, int64_t ccount, int trans, cudaStream_t s) {
    const int64_t nodes = level < 0 ? G.P : merges_at(G.P, level);
    if (nodes <= 0 || ccount <= 0) return 0;
    // tallest node: a [chain R; tile] step (<= 32 slot rows + b tile rows) or a
    // merge (<= 32 + ncols rows)
    const int rgmax = level < 0 ? (int)(G.K > 1 ? G.b + kPW : std::min<int64_t>(G.b, G.mrows))
                                : (int)(kPW + std::min<int64_t>(G.ncols, G.b));
    const size_t smem = panel_update_smem<T>(rgmax);
    cudaError_t e = allow_smem(node_update_kernel<T, false>, smem);
    double fl = 0, by = 0;
    if (g_trace.on) {
        for (int kt = 0; kt < (level < 0 ? G.K : 1); ++kt)
            for (int p = 0; p < G.npan; ++p) {
                double f1, b1;
                trace_counts(G, level, p, kt, nodes, true, ccount, sizeof(T), &f1, &b1);
                fl += f1;
                by += b1;
            }
    }
    TraceScope ts(level < 0 ? K_CHAIN_UPDATE : K_PANEL_UPDATE, fl, by, s);
    if (e == cudaSuccess) {
        // one CTA per (node, group of 32-column blocks): each node's V / T staged
        // once per CTA, with >= 2 CTAs per SM when there are enough blocks
        const int64_t nblk = ceil_div(ccount, 32);
        const int64_t groups = std::max<int64_t>(1, std::min<int64_t>(nblk, (2 * num_sms()) / nodes));
        const int64_t cpb = ceil_div(nblk, groups);
        dim3 grid((unsigned)nodes, (unsigned)ceil_div(nblk, cpb));
        node_update_kernel<T, false><<<grid, kThreads, smem, s>>>(G, A, Tws, level, C, ldc, cfirst, ccount, trans,
                                                                  (int)cpb);
        e = cudaGetLastError();
    }
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}

// Leaf level of Q^T C / Q C for skinny fp32 plans (one panel of <= 16 columns
// on 256-row tiles for n <= 8, 128-row tiles for n <= 16): one warp per chain
// (tsqr_stream_apply.cuh), C in groups of KC columns.  *done = false when the
// plan does not qualify (node_update_kernel then runs).  CAQR_STREAM_APPLY=0
// disables it.
template <typename T>
static int launch_stream_apply(const Geom& G, const T* A, const T* Tws, T* C, int64_t ldc, int64_t cfirst,
                               int64_t ccount, int trans, cudaStream_t s, bool* done) {
    *done = false;
    if constexpr (sizeof(T) == 4) {
        const char* env = getenv("CAQR_STREAM_APPLY");
        if (env && env[0] == '0') return 0;
        const bool nc8 = G.npan == 1 && G.ncols <= 8 && G.b == 256;
        const bool nc16 = G.npan == 1 && G.ncols <= 16 && G.b == 128;
        if (!nc8 && !nc16) return 0;
        const int KC = nc8 ? 8 : 16;
        const unsigned grid = (unsigned)ceil_div(G.P, kStreamApplyWarps);
        cudaError_t e = cudaSuccess;
        for (int64_t c0 = 0; c0 < ccount && e == cudaSuccess; c0 += KC) {
            const int kk = (int)std::min<int64_t>(KC, ccount - c0);
            T* Cg = C + (cfirst + c0) * ldc;
            double fl = 0, by = 0;
            if (g_trace.on) {
                fl = 4.0 * (double)G.mrows * G.ncols * kk;
                by = (double)G.mrows * (G.ncols + 2.0 * kk) * sizeof(T);
            }
            TraceScope ts(K_STREAM_APPLY, fl, by, s);
            if (nc8)
                stream_apply_chain_kernel<8, 8, 8><<<grid, 32 * kStreamApplyWarps, 0, s>>>(G, A, Tws, Cg, ldc, kk,
                                                                                        trans);
            else
                stream_apply_chain_kernel<16, 16, 4><<<grid, 32 * kStreamApplyWarps, 0, s>>>(G, A, Tws, Cg, ldc,
                                                                                          kk, trans);
            e = cudaGetLastError();
        }
        if (e != cudaSuccess) {
            g_last_cuda_error = (int)e;
            return CAQR_ERR_CUDA;
        }
        *done = true;
    }
    return 0;
}

// One tree level of Q^T C / Q C for a single-panel group of <= 16 fp32
// columns: one warp per merge (stream_apply_tree_kernel).  *done = false when
// the group does not qualify.
template <typename T>
static int launch_stream_apply_tree(const Geom& G, const T* A, const T* Tws, int level, T* C, int64_t ldc,
                                    int64_t cfirst, int64_t ccount, int trans, cudaStream_t s, bool* done) {
    *done = false;
    if constexpr (sizeof(T) == 4) {
        const char* env = getenv("CAQR_STREAM_APPLY");
        if (env && env[0] == '0') return 0;
        if (G.npan != 1 || G.ncols > 16) return 0;
        const int64_t nodes = merges_at(G.P, level);
        *done = true;
        if (nodes <= 0 || ccount <= 0) return 0;
        const unsigned grid = (unsigned)ceil_div(nodes, kStreamApplyWarps);
        TraceScope ts(K_STREAM_APPLY, 0.0, 0.0, s);
        T* Cg = C + cfirst * ldc;
        if (G.ncols <= 8)
            stream_apply_tree_kernel<8><<<grid, 32 * kStreamApplyWarps, 0, s>>>(G, A, Tws, Cg, ldc, ccount, level,
                                                                              trans);
        else
            stream_apply_tree_kernel<16><<<grid, 32 * kStreamApplyWarps, 0, s>>>(G, A, Tws, Cg, ldc, ccount, level,
                                                                               trans);
        const cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) {
            g_last_cuda_error = (int)e;
            return CAQR_ERR_CUDA;
        }
    }
    return 0;
}

// Phase profile of the fused kernel (diagnostics, CAQR_PROFILE=1).
static unsigned long long* g_prof = nullptr;
static unsigned long long* prof_buffer() {
    static int on = -1;
    if (on < 0) {
        const char* e = getenv("CAQR_PROFILE");
        on = (e && e[0] == '1') ? 1 : 0;
    }
    if (!on) return nullptr;
    if (!g_prof && cudaMalloc(&g_prof, 16 * sizeof(unsigned long long)) == cudaSuccess)
        cudaMemset(g_prof, 0, 16 * sizeof(unsigned long long));
    return g_prof;
}

template <typename T>
static int launch_fused(const Geom& G, T* A, T* Tws, int* sync, bool do_leaves, cudaStream_t s) {
    const int nl = tree_levels(G.P);
    int64_t total = do_leaves ? G.P : 0;
    for (int lv = 0; lv < nl; ++lv) total += merges_at(G.P, lv);
    if (total <= 0) return 0;
    cudaError_t e = cudaMemsetAsync(sync, 0, group_sync_bytes(G), s);
    double fl = 0, by = 0;
    if (g_trace.on) {
        const double mr = (double)G.mrows, nc = (double)G.ncols;
        fl = do_leaves ? 2.0 * mr * nc * nc - 2.0 / 3.0 * nc * nc * nc
                       : (double)(G.P - 1) * 2.0 / 3.0 * nc * nc * nc;
        by = 2.0 * mr * nc * sizeof(T);
    }
    bool done = false;
    if (!done) {
        const size_t smem = fused_smem_bytes<T>();
        if (e == cudaSuccess) e = allow_smem(tsqr_fused_kernel<T>, smem);
        int occ = 1;
        if (e == cudaSuccess)
            e = occupancy(&occ, tsqr_fused_kernel<T>, kThreads, smem);
        if (e == cudaSuccess) {
            const int64_t grid = std::min<int64_t>(total, (int64_t)std::max(occ, 1) * num_sms());
            TraceScope ts(K_TSQR_FUSED, fl, by, s);
            tsqr_fused_kernel<T><<<(unsigned)grid, kThreads, smem, s>>>(G, A, Tws, sync, nl, do_leaves ? 1 : 0,
                                                                        prof_buffer());
            e = cudaGetLastError();
        }
    }
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}

// CAQR_FUSED=0 forces the split (one launch per level and panel) path; read
// on every call so tests can compare both paths in one process.
// CAQR_EARLY=0 disables the early-start overlap of the CAQR panel loop.
static inline bool early_start_policy() {
    const char* e = getenv("CAQR_EARLY");
    return !(e && e[0] == '0');
}
// One non-blocking side stream and two timing-free events per device, created
// on first use (the only resources the library ever creates).
static bool side_stream(cudaStream_t* s2, cudaEvent_t* ev_ready, cudaEvent_t* ev_done) {
    static std::mutex mu;
    static cudaStream_t streams[64] = {};
    static cudaEvent_t evs[64][2] = {};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev >= 64) return false;
    std::lock_guard<std::mutex> lk(mu);
    if (!streams[dev]) {
        if (cudaStreamCreateWithFlags(&streams[dev], cudaStreamNonBlocking) != cudaSuccess) return false;
        if (cudaEventCreateWithFlags(&evs[dev][0], cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&evs[dev][1], cudaEventDisableTiming) != cudaSuccess)
            return false;
    }
    *s2 = streams[dev];
    *ev_ready = evs[dev][0];
    *ev_done = evs[dev][1];
    return true;
}

// CAQR trailing update: FFMA (exact fp32 products) by default; CAQR_MMA=1 selects
// 3xTF32 mma.sync -- measured slower (8192^2: 81.8 vs 76.1 ms) and 17-28x less
// accurate (residual 4.7e-5 vs 2.8e-6: the ~2^-21 product error compounds over
// the 128 panel groups).
static inline bool mma_policy() {
    const char* e = getenv("CAQR_MMA");
    return e && e[0] == '1';
}

// CAQR_SKINNY=0: no skinny kernel; =2: the older warp-per-task kernel with
// flag-waiting merges instead of the streaming kernel.
static inline int skinny_policy() {
    const char* e = getenv("CAQR_SKINNY");
    return (e && e[0] == '0') ? 0 : (e && e[0] == '2') ? 2 : 1;
}

static inline int fused_policy() {
    const char* e = getenv("CAQR_FUSED");
    return (e && e[0] == '0') ? 0 : 1;
}

// TSQR of one panel group (Fig. 4 minus the trailing update): every leaf's
// panels (factor + intra-group trailing update), then every tree level.
// Skinny groups (fp32, n <= 16): the warp-per-task kernel; true if launched.
template <typename T>
static int launch_skinny(const Geom& G, T* A, T* Tws, int* sync, bool do_leaves, cudaStream_t s, bool* done) {
    *done = false;
    if constexpr (sizeof(T) == 4) {
        const int nr_need = (int)ceil_div(G.ncols + G.b, 32);
        const bool fit8 = G.ncols <= 8 && nr_need <= 9, fit16 = G.ncols <= 16 && nr_need <= 5;
        if (!fit8 && !fit16) return 0;
        const int nl = tree_levels(G.P);
        int64_t total = do_leaves ? G.P : 0;
        for (int lv = 0; lv < nl; ++lv) total += merges_at(G.P, lv);
        if (total <= 0) {
            *done = true;
            return 0;
        }
        cudaError_t e = cudaMemsetAsync(sync, 0, group_sync_bytes(G), s);
        if (e == cudaSuccess) {
            const int64_t warps = std::min<int64_t>(total, (int64_t)num_sms() * 16);
            const unsigned grid = (unsigned)ceil_div(warps, kSkinnyWarps);
            double fl = 0, by = 0;
            if (g_trace.on) {
                const double mr = (double)G.mrows, nc = (double)G.ncols;
                fl = 2.0 * mr * nc * nc - 2.0 / 3.0 * nc * nc * nc;
                by = 2.0 * mr * nc * sizeof(T);
            }
            TraceScope ts(K_TSQR_SKINNY, fl, by, s);
            if (fit8)
                tsqr_skinny_kernel<8, 9><<<grid, 32 * kSkinnyWarps, 0, s>>>(G, A, Tws, sync, nl, do_leaves ? 1 : 0);
            else
                tsqr_skinny_kernel<16, 5><<<grid, 32 * kSkinnyWarps, 0, s>>>(G, A, Tws, sync, nl, do_leaves ? 1 : 0);
            e = cudaGetLastError();
        }
        if (e != cudaSuccess) {
            g_last_cuda_error = (int)e;
            return CAQR_ERR_CUDA;
        }
        *done = true;
    }
    return 0;
}

// Streaming skinny TSQR (tsqr_stream.cuh): n <= 16, tiles of 256 (n <= 8) or
// 128 rows, one chain per warp, 8 warps per CTA; true in *done if launched.
template <typename T, int NC, int RPL, int NW = 8, int NBUF = 2>
static cudaError_t launch_stream_nc(const Geom& G, T* A, T* Tws, int* sync, bool vec, cudaStream_t s) {
    const unsigned grid = (unsigned)ceil_div(G.P, NW);
    const size_t smem = stream_smem_bytes<T, NC, RPL, NW, NBUF>(grid);
    const int nl = tree_levels(G.P);
    cudaError_t e;
    unsigned long long* prof = prof_buffer();
    const char* dbe = getenv("CAQR_STREAM_DBG");
    const int dbg = dbe ? atoi(dbe) : 0;
    if (prof) cudaMemsetAsync(prof, 0xff, sizeof(unsigned long long), s);  // [0] is a running min
    if (vec) {
        e = allow_smem(tsqr_stream_kernel<T, NC, RPL, NW, NBUF, true>, smem);
        if (e == cudaSuccess)
            tsqr_stream_kernel<T, NC, RPL, NW, NBUF, true><<<grid, 32 * NW, smem, s>>>(G, A, Tws, sync, nl, prof, dbg);
    } else {
        e = allow_smem(tsqr_stream_kernel<T, NC, RPL, NW, NBUF, false>, smem);
        if (e == cudaSuccess)
            tsqr_stream_kernel<T, NC, RPL, NW, NBUF, false><<<grid, 32 * NW, smem, s>>>(G, A, Tws, sync, nl, prof, dbg);
    }
    return e == cudaSuccess ? cudaGetLastError() : e;
}

template <typename T>
static int launch_stream(const Geom& G, T* A, T* Tws, int* sync, cudaStream_t s, bool* done) {
    *done = false;
    if constexpr (sizeof(T) == 4) {
        const bool nc8 = G.ncols <= 8 && G.b == 256, nc16 = G.ncols <= 16 && G.b == 128;
        if (!nc8 && !nc16) return 0;
        const bool w16 = G.ncols <= 8 && G.b == 128;  // 16 warps x 128-row tiles (CAQR_STREAM16)
        // 16 warps x 256-row tiles, one buffer each, once there are more
        // tiles than 8 warps per SM would take (fewer: 8 warps, less tree)
        const bool w16b = nc8 && G.L > kStreamChains && stream_w16b_policy();
        // the CTAs' R's travel through the workspace's flag area
        const int64_t nct = ceil_div(G.P, (w16 || w16b) ? 16 : 8);
        // (plus one arrival counter per (cross-CTA level, CTA))
        const int64_t rx = (nc8 || w16) ? stream_rx_ints<T, 8>(nct) : stream_rx_ints<T, 16>(nct);
        if ((64 + rx + (int64_t)tree_levels(G.P) * nct) * (int64_t)sizeof(int) > (int64_t)group_sync_bytes(G)) return 0;
        if ((w16b  ? stream_smem_bytes<T, 8, 8, 16, 1>(nct)
             : nc8 ? stream_smem_bytes<T, 8, 8, 8>(nct)
             : w16 ? stream_smem_bytes<T, 8, 4, 16>(nct) : stream_smem_bytes<T, 16, 4, 8>(nct)) > 220 * 1024)
            return 0;
        // 16-byte cp.async needs every tile column start 16-byte aligned
        const bool vec = (reinterpret_cast<uintptr_t>(A) % 16 == 0) && (G.lda % 4 == 0) && (G.row0 % 4 == 0);
        cudaError_t e = cudaMemsetAsync(sync, 0, group_sync_bytes(G), s);
        if (e == cudaSuccess) {
            double fl = 0, by = 0;
            if (g_trace.on) {
                const double mr = (double)G.mrows, nc = (double)G.ncols;
                fl = 2.0 * mr * nc * nc - 2.0 / 3.0 * nc * nc * nc;
                by = 2.0 * mr * nc * sizeof(T);
            }
            TraceScope ts(K_TSQR_SKINNY, fl, by, s);
            e = w16b  ? launch_stream_nc<T, 8, 8, 16, 1>(G, A, Tws, sync, vec, s)
                : nc8 ? launch_stream_nc<T, 8, 8>(G, A, Tws, sync, vec, s)
                : w16 ? launch_stream_nc<T, 8, 4, 16>(G, A, Tws, sync, vec, s)
                      : launch_stream_nc<T, 16, 4>(G, A, Tws, sync, vec, s);
        }
        if (e != cudaSuccess) {
            g_last_cuda_error = (int)e;
            return CAQR_ERR_CUDA;
        }
        *done = true;
    }
    return 0;
}

// Chain phase of a whole-width fp32 group (tsqr_chain.cuh): one persistent
// launch over the P chains; the tree over their slots follows (merge-only
// fused kernel).
static inline bool chain_tc_policy() {  // CAQR_CHAIN_TC=0: mma.sync trailing update in the chain kernel
    const char* e = getenv("CAQR_CHAIN_TC");
    return !(e && e[0] == '0');
}
template <int NQ, int SEG, int MINB, bool TC>
static cudaError_t launch_chain_cfg(const Geom& G, float* A, float* Tws, int* sync, cudaStream_t s) {
    const size_t smem = TC ? ChainCfgTC<NQ, SEG>::BYTES : ChainCfg<NQ, SEG>::BYTES;
    auto kern = tsqr_chain_kernel<NQ, SEG, MINB, TC>;
    cudaError_t e = allow_smem(kern, smem);
    int occ = 1;
    if (e == cudaSuccess) e = occupancy(&occ, kern, 32 * NQ, smem);
    if (e != cudaSuccess) return e;
    if (TC) {
        // The occupancy API counts a tcgen05 kernel as one CTA per SM; the
        // CTAs co-reside as long as their TMEM allocations (128 columns each)
        // and registers / shared memory fit.
        cudaFuncAttributes fa;
        if (cudaFuncGetAttributes(&fa, kern) == cudaSuccess) {
            const int by_smem = (int)((228 * 1024) / (smem + fa.sharedSizeBytes + 1024));
            const int by_regs = 65536 / (((fa.numRegs * 32 + 255) / 256) * 256 * NQ);
            occ = std::max(1, std::min(4, std::min(by_smem, by_regs)));
        }
    }
    if (const char* e = getenv("CAQR_CHAIN_OCC")) occ = atoi(e);  // diagnostics
    const int64_t grid = std::min<int64_t>(G.P, (int64_t)std::max(occ, 1) * num_sms());
    if (getenv("CAQR_CHAIN_DBG")) {
        cudaFuncAttributes fa;
        cudaFuncGetAttributes(&fa, kern);
        int o2 = 0, o3 = 0, o4 = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o2, kern, 32 * NQ, 0);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o3, kern, 32 * NQ, 40000);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o4, kern, 32 * NQ, 60000);
        fprintf(stderr,
                "chain kernel TC=%d NQ=%d SEG=%d smem=%zu occ=%d grid=%lld P=%lld K=%lld regs=%d static=%zu "
                "maxdyn=%d occ(0)=%d occ(40k)=%d occ(60k)=%d\n",
                (int)TC, NQ, SEG, smem, occ, (long long)grid, (long long)G.P, (long long)G.K, fa.numRegs,
                fa.sharedSizeBytes, fa.maxDynamicSharedSizeBytes, o2, o3, o4);
    }
    unsigned long long* prof = prof_buffer();
    kern<<<(unsigned)grid, 32 * NQ, smem, s>>>(G, A, Tws, sync, prof);
    return cudaGetLastError();
}
template <int NQ, int SEG, int MINB>
static cudaError_t launch_chain_cfg(const Geom& G, float* A, float* Tws, int* sync, cudaStream_t s) {
    return chain_tc_policy() ? launch_chain_cfg<NQ, SEG, MINB, true>(G, A, Tws, sync, s)
                             : launch_chain_cfg<NQ, SEG, MINB, false>(G, A, Tws, sync, s);
}

template <typename T>
static int launch_chain(const Geom& G, T* A, T* Tws, int* sync, cudaStream_t s, bool* done) {
    *done = false;
    if constexpr (sizeof(T) == 4) {
        if (G.ncols <= 16 || G.ncols > G.b || !(G.b == 128 || G.b == 192 || G.b == 256)) return 0;
        cudaError_t e = cudaMemsetAsync(sync, 0, group_sync_bytes(G), s);
        if (e == cudaSuccess) {
            double fl = 0, by = 0;
            if (g_trace.on) {
                const double mr = (double)G.mrows, nc = (double)G.ncols;
                fl = 2.0 * mr * nc * nc - 2.0 / 3.0 * nc * nc * nc;
                by = 2.0 * mr * nc * sizeof(T);
            }
            TraceScope ts(K_TSQR_CHAIN, fl, by, s);
            e = G.b == 128   ? launch_chain_cfg<4, 32, 3>(G, A, Tws, sync, s)
                : G.b == 192 ? launch_chain_cfg<4, 48, 3>(G, A, Tws, sync, s)
                             : launch_chain_cfg<4, 64, 2>(G, A, Tws, sync, s);
        }
        if (e != cudaSuccess) {
            g_last_cuda_error = (int)e;
            return CAQR_ERR_CUDA;
        }
        *done = true;
    }
    return 0;
}

template <typename T>
static int factor_group(const Geom& G, T* A, T* Tws, int* sync, bool do_leaves, cudaStream_t s,
                        bool chain = false) {
    if (chain && do_leaves && fused_ok(G)) {
        bool done = false;
        int rc = launch_chain<T>(G, A, Tws, sync, s, &done);
        if (rc) return rc;
        if (done) return launch_fused<T>(G, A, Tws, sync, false, s);  // tree over the chain slots
    }
    if (fused_policy() && do_leaves && G.npan == 1 && G.ncols <= 16 && skinny_policy() == 1) {
        bool done = false;
        const int rc = launch_stream<T>(G, A, Tws, sync, s, &done);
        if (rc || done) return rc;
    }
    if (fused_policy() && G.npan == 1 && G.ncols <= 16 && skinny_policy()) {
        bool done = false;
        const int rc = launch_skinny<T>(G, A, Tws, sync, do_leaves, s, &done);
        if (rc || done) return rc;
    }
    if (fused_policy() && fused_ok(G)) return launch_fused<T>(G, A, Tws, sync, do_leaves, s);
    int rc = 0;
    if (do_leaves) {
        for (int kt = 0; kt < G.K && !rc; ++kt)
            for (int p = 0; p < G.npan && !rc; ++p) {
                rc = launch_factor<T>(G, A, Tws, -1, p, kt, G.P, s);
                if (!rc && p + 1 < G.npan)
                    rc = launch_update<T>(G, A, Tws, -1, p, kt, G.P, A, G.lda, G.col0 + 32 * (p + 1),
                                          G.ncols - 32 * (p + 1), 1, s);
            }
    }
    const int nl = tree_levels(G.P);
    for (int lv = 0; lv < nl && !rc; ++lv) {
        const int64_t nm = merges_at(G.P, lv);
        for (int p = 0; p < G.npan && !rc; ++p) {
            rc = launch_factor<T>(G, A, Tws, lv, p, 0, nm, s);
            if (!rc && p + 1 < G.npan)
                rc = launch_update<T>(G, A, Tws, lv, p, 0, nm, A, G.lda, G.col0 + 32 * (p + 1),
                                      G.ncols - 32 * (p + 1), 1, s);
        }
    }
    return rc;
}

// C[rows of the group, cfirst:cfirst+ccount] <- Q_g^T C (trans) or Q_g C.
// Q_g^T = (tree top)^T ... (tree level 0)^T (leaves)^T, each node's panels in
// order 0..npan-1; Q_g is the reverse.
template <typename T>
static int apply_group(const Geom& G, const T* A, const T* Tws, bool do_leaves, T* C,
                       int64_t ldc, int64_t cfirst, int64_t ccount, int trans, cudaStream_t s,
                       bool mma = false, bool one_launch = true) {
    int rc = 0;
    const int nl = tree_levels(G.P);
    if (!mma && chain_apply_policy()) {  // one launch per tree level (+ one for the chains)
        // groups the warp-per-chain skinny apply does not take: one launch
        const bool skinny = sizeof(T) == 4 && G.npan == 1 &&
                            ((G.ncols <= 8 && G.b == 256) || (G.ncols <= 16 && G.b == 128));
        if (one_launch && (!skinny || (getenv("CAQR_STREAM_APPLY") && getenv("CAQR_STREAM_APPLY")[0] == '0'))) {
            bool done = false;
            const char* dbg = getenv("CAQR_APPLY_ALL");
            if (dbg && dbg[0] == '2') {  // diagnostics: chains by node_update_kernel, tree in one launch
                if (trans && do_leaves) rc = launch_node_update<T>(G, A, Tws, -1, C, ldc, cfirst, ccount, 1, s);
                if (!rc) rc = launch_node_update_all<T>(G, A, Tws, false, C, ldc, cfirst, ccount, trans, s, &done);
                if (!rc && !trans && do_leaves) rc = launch_node_update<T>(G, A, Tws, -1, C, ldc, cfirst, ccount, 0, s);
                return rc;
            }
            rc = launch_node_update_all<T>(G, A, Tws, do_leaves, C, ldc, cfirst, ccount, trans, s, &done);
            if (rc || done) return rc;
        }
        auto leaves = [&](int tr) {
            bool done = false;
            int r = launch_stream_apply<T>(G, A, Tws, C, ldc, cfirst, ccount, tr, s, &done);
            if (!r && !done) r = launch_node_update<T>(G, A, Tws, -1, C, ldc, cfirst, ccount, tr, s);
            return r;
        };
        auto level = [&](int lv, int tr) {
            bool done = false;
            int r = launch_stream_apply_tree<T>(G, A, Tws, lv, C, ldc, cfirst, ccount, tr, s, &done);
            if (!r && !done) r = launch_node_update<T>(G, A, Tws, lv, C, ldc, cfirst, ccount, tr, s);
            return r;
        };
        if (trans) {
            if (do_leaves) rc = leaves(1);
            for (int lv = 0; lv < nl && !rc; ++lv) rc = level(lv, 1);
        } else {
            for (int lv = nl - 1; lv >= 0 && !rc; --lv) rc = level(lv, 0);
            if (do_leaves && !rc) rc = leaves(0);
        }
        return rc;
    }
    if (trans) {
        if (do_leaves)
            for (int kt = 0; kt < G.K && !rc; ++kt)
                for (int p = 0; p < G.npan && !rc; ++p)
                    rc = launch_update<T>(G, A, Tws, -1, p, kt, G.P, C, ldc, cfirst, ccount, 1, s, mma);
        for (int lv = 0; lv < nl && !rc; ++lv)
            for (int p = 0; p < G.npan && !rc; ++p)
                rc = launch_update<T>(G, A, Tws, lv, p, 0, merges_at(G.P, lv), C, ldc, cfirst, ccount,
                                      1, s, mma);
    } else {
        for (int lv = nl - 1; lv >= 0 && !rc; --lv)
            for (int p = G.npan - 1; p >= 0 && !rc; --p)
                rc = launch_update<T>(G, A, Tws, lv, p, 0, merges_at(G.P, lv), C, ldc, cfirst, ccount,
                                      0, s, mma);
        if (do_leaves)
            for (int kt = (int)G.K - 1; kt >= 0 && !rc; --kt)
                for (int p = G.npan - 1; p >= 0 && !rc; --p)
                    rc = launch_update<T>(G, A, Tws, -1, p, kt, G.P, C, ldc, cfirst, ccount, 0, s, mma);
    }
    return rc;
}

template <typename T>
static int launch_extract_r(int64_t n, const T* A, int64_t lda, T* R, int64_t ldr, cudaStream_t s) {
    if (n <= 0) return 0;
    dim3 grid((unsigned)std::min<int64_t>(ceil_div(n, 256), 64), (unsigned)n);
    TraceScope ts(K_EXTRACT_R, 0.0, 2.0 * n * n * sizeof(T), s);
    extract_r_kernel<T><<<grid, 256, 0, s>>>(n, A, lda, R, ldr);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}

// ---- the ABI bodies ---------------------------------------------------------
template <typename T>
static int factor_impl(int64_t m, int64_t n, T* A, int64_t lda, T* R, int64_t ldr, void* ws,
                       size_t ws_bytes, const caqr_opts* opts, cudaStream_t s, int dtype) {
    // dimensions first; LAPACK-style quick return before any pointer is used
    if (m < 0) return -1;
    if (n < 0 || n > m) return -2;
    if (lda < std::max<int64_t>(1, m)) return -4;
    if (ldr < std::max<int64_t>(1, n)) return -6;
    Plan pl;
    int rc = make_plan(m, n, dtype, opts, 9, &pl);
    if (rc) return rc;
    if (m == 0 || n == 0) return 0;
    if (!A) return -3;
    if (!R) return -5;
    if (!ws) return -7;
    if (ws_bytes < plan_ws_bytes(pl)) return -8;
    // Group offsets in the workspace.
    auto group_ptrs = [&](int64_t g, T** tws, int** sync) {
        char* wsb = static_cast<char*>(ws);
        for (int64_t q = 0; q < g; ++q) wsb += group_ws_bytes(group_geom(pl, q, lda), sizeof(T));
        *tws = reinterpret_cast<T*>(wsb);
        *sync = reinterpret_cast<int*>(wsb + group_t_bytes(group_geom(pl, g, lda), sizeof(T)));
    };
    // CAQR with early start ("the trailing matrix update can begin
    // before the entire panel is factored"): after group g's TSQR, its Q^T is
    // applied first to the next group's columns; the next TSQR then runs on a
    // side stream while the rest of the trailing matrix is updated on `s`.
    cudaStream_t s2 = nullptr;
    cudaEvent_t ev_ready = nullptr, ev_done = nullptr;
    const bool overlap = pl.ngroups > 1 && early_start_policy() && side_stream(&s2, &ev_ready, &ev_done);
    // The side stream and its two events are per device and shared by every
    // call: hold a per-device lock while this call records / waits on them, so
    // that a concurrent call on another host thread cannot re-record ev_ready
    // between this call's record and its wait (host issue is serialised; the
    // GPU work stays asynchronous).
    static std::mutex overlap_mu[64];
    int dev_id = 0;
    cudaGetDevice(&dev_id);
    std::unique_lock<std::mutex> overlap_lock(overlap_mu[dev_id & 63], std::defer_lock);
    if (overlap) overlap_lock.lock();
    for (int64_t g = 0; g < pl.ngroups && !rc; ++g) {
        const Geom G = group_geom(pl, g, lda);
        T* Tws;
        int* sync;
        group_ptrs(g, &Tws, &sync);
        if (!overlap || g == 0) {
            rc = factor_group<T>(G, A, Tws, sync, true, s, pl.chain);
        } else if (cudaStreamWaitEvent(s, ev_done, 0) != cudaSuccess) {  // TSQR_g ran on s2
            rc = CAQR_ERR_CUDA;
        }
        const int64_t trail0 = G.col0 + G.ncols;
        if (rc || trail0 >= n) continue;
        // CAQR trailing update; fp32: tensor cores (3xTF32)
        const int64_t next_cols = overlap ? std::min<int64_t>(pl.nb, n - trail0) : n - trail0;
        rc = apply_group<T>(G, A, Tws, true, A, lda, trail0, next_cols, 1, s, mma_policy());
        if (!rc && overlap && g + 1 < pl.ngroups) {
            const Geom Gn = group_geom(pl, g + 1, lda);
            T* Twn;
            int* syncn;
            group_ptrs(g + 1, &Twn, &syncn);
            if (cudaEventRecord(ev_ready, s) != cudaSuccess || cudaStreamWaitEvent(s2, ev_ready, 0) != cudaSuccess)
                rc = CAQR_ERR_CUDA;
            if (!rc) rc = factor_group<T>(Gn, A, Twn, syncn, true, s2);
            if (!rc && cudaEventRecord(ev_done, s2) != cudaSuccess) rc = CAQR_ERR_CUDA;
        }
        if (!rc && next_cols < n - trail0)
            // (per-level launches: a cooperative grid would hold every SM and
            // shut out the next TSQR running beside it on s2; C5 76 -> 95 ms)
            rc = apply_group<T>(G, A, Tws, true, A, lda, trail0 + next_cols, n - trail0 - next_cols, 1, s,
                                mma_policy(), !overlap);
    }
    if (!rc) rc = launch_extract_r<T>(n, A, lda, R, ldr, s);
    return rc;
}

template <typename T>
static int apply_impl(int64_t m, int64_t n, const T* A, int64_t lda, const void* ws, int64_t k,
                      T* C, int64_t ldc, const caqr_opts* opts, cudaStream_t s, int dtype,
                      int trans) {
    if (m < 0) return -1;
    if (n < 0 || n > m) return -2;
    if (lda < std::max<int64_t>(1, m)) return -4;
    if (k < 0) return -6;
    if (ldc < std::max<int64_t>(1, m)) return -8;
    Plan pl;
    int rc = make_plan(m, n, dtype, opts, 9, &pl);
    if (rc) return rc;
    if (m == 0 || n == 0 || k == 0) return 0;
    if (!A) return -3;
    if (!C) return -7;
    if (!ws) return -5;
    const T* base = static_cast<const T*>(ws);
    // group offsets into the workspace
    const T* tws[1024];
    int64_t ng = pl.ngroups;
    if (ng > 1024) return CAQR_ERR_UNSUPPORTED;
    {
        const char* t = reinterpret_cast<const char*>(base);
        for (int64_t g = 0; g < ng; ++g) {
            tws[g] = reinterpret_cast<const T*>(t);
            t += group_ws_bytes(group_geom(pl, g, lda), sizeof(T));
        }
    }
    if (trans) {
        for (int64_t g = 0; g < ng && !rc; ++g)
            rc = apply_group<T>(group_geom(pl, g, lda), A, tws[g], true, C, ldc, 0, k, 1, s);
    } else {
        for (int64_t g = ng - 1; g >= 0 && !rc; --g)
            rc = apply_group<T>(group_geom(pl, g, lda), A, tws[g], true, C, ldc, 0, k, 0, s);
    }
    return rc;
}

template <typename T>
static int form_q_impl(int64_t m, int64_t n, const T* A, int64_t lda, const void* ws, T* Q,
                       int64_t ldq, const caqr_opts* opts, cudaStream_t s, int dtype) {
    if (m < 0) return -1;
    if (n < 0 || n > m) return -2;
    if (lda < std::max<int64_t>(1, m)) return -4;
    if (ldq < std::max<int64_t>(1, m)) return -7;
    if (m == 0 || n == 0) return 0;
    if (!A) return -3;
    if (!Q) return -6;
    if (!ws) return -5;
    dim3 grid((unsigned)std::min<int64_t>(ceil_div(m, 256), 1024), (unsigned)n);
    cudaError_t e;
    {
        TraceScope ts(K_SET_IDENTITY, 0.0, (double)m * n * sizeof(T), s);
        set_identity_kernel<T><<<grid, 256, 0, s>>>(m, n, Q, ldq);
        e = cudaGetLastError();
    }
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    const int rc = apply_impl<T>(m, n, A, lda, ws, n, Q, ldq, opts, s, dtype, 0);
    return rc == -6 ? -7 : rc;
}

// Combine geometry: P slots of n rows (the leaves are the given R factors).
static Geom combine_geom(int P, int64_t n, int64_t ld) {
    Geom G;
    G.lda = ld;
    G.row0 = 0;
    G.col0 = 0;
    G.mrows = (int64_t)P * n;
    G.ncols = (int32_t)n;
    G.npan = (int32_t)ceil_div(n, kPW);
    G.b = n;
    G.L = P;
    G.K = 1;
    G.P = P;
    G.bm = n;
    return G;
}

template <typename T>
static int combine_impl(int P, int64_t n, T* Rs, int64_t ld, T* R, int64_t ldr, void* ws,
                        size_t ws_bytes, cudaStream_t s, int dtype) {
    if (P < 1) return -1;
    if (n < 0 || n > kMaxGroup) return -2;
    if (!Rs) return -3;
    if (ld < std::max<int64_t>(1, (int64_t)P * n)) return -4;
    if (!R) return -5;
    if (ldr < std::max<int64_t>(1, n)) return -6;
    if (n == 0) return 0;
    if (!ws) return -7;
    if (ws_bytes < caqr_combine_workspace_bytes(P, n, dtype)) return -8;
    const Geom G = combine_geom(P, n, ld);
    int* sync = reinterpret_cast<int*>(static_cast<char*>(ws) + group_t_bytes(G, sizeof(T)));
    int rc = factor_group<T>(G, Rs, static_cast<T*>(ws), sync, false, s);
    if (!rc) rc = launch_extract_r<T>(n, Rs, ld, R, ldr, s);
    return rc;
}

template <typename T>
static int combine_apply_impl(int P, int64_t n, const T* Rs, int64_t ld, const void* ws, int trans,
                              int64_t k, T* C, int64_t ldc, cudaStream_t s) {
    if (P < 1) return -1;
    if (n < 0 || n > kMaxGroup) return -2;
    if (!Rs) return -3;
    if (ld < std::max<int64_t>(1, (int64_t)P * n)) return -4;
    if (k < 0) return -7;
    if (!C) return -8;
    if (ldc < std::max<int64_t>(1, (int64_t)P * n)) return -9;
    if (n == 0 || k == 0) return 0;
    if (!ws) return -5;
    const Geom G = combine_geom(P, n, ld);
    return apply_group<T>(G, Rs, static_cast<const T*>(ws), false, C, ldc, 0, k, trans ? 1 : 0, s);
}

}  // namespace caqr

using namespace caqr;


// ---- application layer: SVD via QR and robust PCA (rpca.cuh) ----
static inline unsigned elem_grid(int64_t total, int threads) {
    const int64_t want = (total + threads - 1) / threads;
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(want, (int64_t)num_sms() * 8));
}

template <typename T>
static int svd_small_impl(int64_t n, const T* R, int64_t ldr, T* U, int64_t ldu, T* sigma, T* V, int64_t ldv,
                          cudaStream_t s) {
    if (n < 0 || n > kSvdMaxN) return -1;
    if (ldr < std::max<int64_t>(1, n)) return -3;
    if (ldu < std::max<int64_t>(1, n)) return -5;
    if (ldv < std::max<int64_t>(1, n)) return -8;
    if (n == 0) return 0;
    if (!R) return -2;
    if (!U) return -4;
    if (!sigma) return -6;
    const size_t smem = jacobi_svd_smem<T>((int)n);  // (V == NULL: right vectors not formed)
    cudaError_t e = allow_smem(jacobi_svd_kernel<T>, smem);
    if (e == cudaSuccess) {
        TraceScope ts(K_SVD_SMALL, 0.0, 3.0 * n * n * sizeof(T), s);
        // a pair counts as orthogonal at |b_p.b_q| <= tol ||b_p|| ||b_q||: U's
        // orthogonality is tol-level, far below the output precision's epsilon
        const double tol = sizeof(T) == 4 ? 1e-8 : 1e-15;
        static const int max_sweeps = [] {
            const char* e = getenv("CAQR_SVD_SWEEPS");  // diagnostics: cap the Jacobi sweeps
            return e ? std::max(1, atoi(e)) : 30;
        }();
        const char* be = getenv("CAQR_SVD_BLOCK");  // 0: always the single-CTA kernel
        if (V == nullptr && n >= 32 && !(be && be[0] == '0')) {
            // U, sigma only: block Jacobi over an 8-CTA cluster (DSMEM block moves)
            jacobi_svd_block_kernel<T><<<kSvdCl, kSvdClT, 0, s>>>((int)n, R, ldr, U, ldu, sigma, tol, max_sweeps);
        } else {
            jacobi_svd_kernel<T><<<1, kSvdThreads, smem, s>>>((int)n, R, ldr, U, ldu, sigma, V, ldv, tol,
                                                              max_sweeps);
        }
        e = cudaGetLastError();
    }
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}

static int launch_status() {
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}


template <typename T>
static int trsm_impl(int64_t n, int64_t k, const T* R, int64_t ldr, T* B, int64_t ldb, cudaStream_t s) {
    if (n < 0) return -1;
    if (k < 0) return -2;
    if (ldr < std::max<int64_t>(1, n)) return -4;
    if (ldb < std::max<int64_t>(1, n)) return -6;
    if (n == 0 || k == 0) return 0;
    if (!R) return -3;
    if (!B) return -5;
    const size_t smem = sizeof(T) * (size_t)n;
    if (smem > 200 * 1024) return -1;
    cudaError_t e = allow_smem(trsm_upper_kernel<T>, smem);
    if (e == cudaSuccess) {
        TraceScope ts(K_TRSM, (double)n * n * k, (double)n * n * sizeof(T) / 2 + 2.0 * n * k * sizeof(T), s);
        for (int64_t c0 = 0; c0 < k && e == cudaSuccess; c0 += 65535) {
            const unsigned g = (unsigned)std::min<int64_t>(65535, k - c0);
            trsm_upper_kernel<T><<<g, 256, smem, s>>>(n, R, ldr, B + c0 * ldb, ldb);
            e = cudaGetLastError();
        }
    }
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}

// ---- [I_n; 0] -------------------------------------------------------------
template <typename T>
static int set_identity_impl(int64_t m, int64_t n, T* Q, int64_t ldq, cudaStream_t s) {
    if (m < 0) return -1;
    if (n < 0 || n > m) return -2;
    if (ldq < std::max<int64_t>(1, m)) return -4;
    if (m == 0 || n == 0) return 0;
    if (!Q) return -3;
    dim3 grid((unsigned)std::min<int64_t>(ceil_div(m, 256), 1024), (unsigned)n);
    TraceScope ts(K_SET_IDENTITY, 0.0, (double)m * n * sizeof(T), s);
    set_identity_kernel<T><<<grid, 256, 0, s>>>(m, n, Q, ldq);
    return launch_status();
}
// ---- Host-streamed factorisation (caqr_factor_host_*) ----------------------
// The row chunks of A are a one-GPU instance of the distributed TSQR the paper
// cites: chunk c is factored by the ordinary path as soon as its
// H2D copy (a copy engine, second stream) has landed, while later chunks are
// still in flight; the chunks' R factors are then combined by the structured
// tree of caqr_combine.  Chunk c = rows [m*c/S, m*(c+1)/S).
static inline int64_t host_chunk_row(int64_t m, int S, int c) { return (int64_t)(((__int128)m * c) / S); }
static inline size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

// Offsets of the chunk workspaces, the R stack and the combine workspace.
// Returns 0 on illegal arguments.
static size_t host_layout(int64_t m, int64_t n, int S, int dtype, const caqr_opts* opts, int c,
                          int64_t* row0, int64_t* rows, size_t* off) {
    if (m < 0 || n < 0 || n > m || S < 1 || S > 1024 || (dtype != CAQR_F32 && dtype != CAQR_F64)) return 0;
    if (S > 1 && (n > kMaxGroup || m / S < n)) return 0;
    const size_t es = dtype == CAQR_F64 ? 8 : 4;
    size_t o = 0;
    for (int q = 0; q < S; ++q) {
        const int64_t r0 = host_chunk_row(m, S, q), mc = host_chunk_row(m, S, q + 1) - r0;
        const size_t wb = caqr_workspace_bytes(mc, n, dtype, opts);
        if (wb == 0) return 0;
        if (q == c) {
            *row0 = r0;
            *rows = mc;
            *off = o;
        }
        o += align256(wb);
    }
    const size_t rstack = align256((size_t)S * n * n * es);
    if (c == S) { *row0 = 0; *rows = (int64_t)S * n; *off = o; }           // the R stack
    o += rstack;
    const size_t cw = S > 1 ? caqr_combine_workspace_bytes(S, n, dtype) : 256;
    if (cw == 0) return 0;
    if (c == S + 1) { *row0 = 0; *rows = 0; *off = o; }                    // the combine workspace
    return o + align256(cw);
}

// One copy stream and a pool of events per device for the H2D pipeline.
// (plus a second compute stream: consecutive chunks' TSQRs alternate between
// the caller's stream and it, so one chunk's latency-bound tree tail overlaps
// the next chunk's leaves).
static bool copy_stream(cudaStream_t* cs, cudaStream_t* s2, cudaEvent_t** evs) {
    static std::mutex mu;
    static cudaStream_t streams[64][2] = {};
    static cudaEvent_t pool[64][1027] = {};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev >= 64) return false;
    std::lock_guard<std::mutex> lk(mu);
    if (!streams[dev][0]) {
        if (cudaStreamCreateWithFlags(&streams[dev][0], cudaStreamNonBlocking) != cudaSuccess ||
            cudaStreamCreateWithFlags(&streams[dev][1], cudaStreamNonBlocking) != cudaSuccess)
            return false;
        for (int i = 0; i < 1027; ++i)
            if (cudaEventCreateWithFlags(&pool[dev][i], cudaEventDisableTiming) != cudaSuccess) return false;
    }
    *cs = streams[dev][0];
    *s2 = streams[dev][1];
    *evs = pool[dev];
    return true;
}

static inline bool host_dual_policy() {
    const char* e = getenv("CAQR_HOST_DUAL");
    return !(e && e[0] == '0');
}

template <typename T>
static int factor_host_impl(int64_t m, int64_t n, int S, const T* Ah, int64_t ldh, T* A, int64_t lda, T* R,
                            int64_t ldr, void* ws, size_t ws_bytes, const caqr_opts* opts, cudaStream_t s,
                            int dtype) {
    if (m < 0) return -1;
    if (n < 0 || n > m) return -2;
    if (S < 1 || S > 1024 || (S > 1 && (n > kMaxGroup || m / S < n))) return -3;
    if (ldh < std::max<int64_t>(1, m)) return -5;
    if (lda < std::max<int64_t>(1, m)) return -7;
    if (ldr < std::max<int64_t>(1, n)) return -9;
    int64_t r0, mc;
    size_t off;
    const size_t need = host_layout(m, n, S, dtype, opts, 0, &r0, &mc, &off);
    if (need == 0) return -12;
    if (m == 0 || n == 0) return 0;
    if (!Ah) return -4;
    if (!A) return -6;
    if (!R) return -8;
    if (!ws) return -10;
    if (ws_bytes < need) return -11;
    cudaStream_t cs, s2;
    cudaEvent_t* ev;
    if (!copy_stream(&cs, &s2, &ev)) return CAQR_ERR_CUDA;
    // The copy stream and its events are shared per process: calls from
    // several host threads issue one at a time (each wait binds to its own
    // call's event records).
    static std::mutex issue_mu;
    std::lock_guard<std::mutex> issue_lock(issue_mu);
    // The copies may overwrite A only after the work already queued on s.
    const bool dual = S > 1 && host_dual_policy();
    if (cudaEventRecord(ev[S], s) != cudaSuccess || cudaStreamWaitEvent(cs, ev[S], 0) != cudaSuccess ||
        (dual && cudaStreamWaitEvent(s2, ev[S], 0) != cudaSuccess))
        return CAQR_ERR_CUDA;
    // On an error return after this point, make `stream` wait for whatever the
    // copy stream and the second compute stream already hold (queued H2D
    // copies, odd chunks' TSQRs), so that a caller who synchronises `stream`
    // may free A_host / ws safely and a capture has no unjoined fork.
    auto join_fail = [&](int code) {
        g_last_cuda_error = (int)cudaGetLastError();
        cudaEventRecord(ev[S], cs);
        cudaStreamWaitEvent(s, ev[S], 0);
        if (dual) {
            cudaEventRecord(ev[S + 1], s2);
            cudaStreamWaitEvent(s, ev[S + 1], 0);
        }
        return code;
    };
    char* wsb = static_cast<char*>(ws);
    for (int c = 0; c < S; ++c) {
        host_layout(m, n, S, dtype, opts, c, &r0, &mc, &off);
        if (cudaMemcpy2DAsync(A + r0, lda * sizeof(T), Ah + r0, ldh * sizeof(T), mc * sizeof(T), n,
                              cudaMemcpyHostToDevice, cs) != cudaSuccess ||
            cudaEventRecord(ev[c], cs) != cudaSuccess)
            return join_fail(CAQR_ERR_CUDA);
    }
    int64_t rs0, rsn;
    size_t rs_off, cw_off;
    host_layout(m, n, S, dtype, opts, S, &rs0, &rsn, &rs_off);
    host_layout(m, n, S, dtype, opts, S + 1, &rs0, &rsn, &cw_off);
    T* Rs = reinterpret_cast<T*>(wsb + rs_off);
    const int64_t ld = (int64_t)S * n;
    int rc = 0;
    for (int c = 0; c < S && !rc; ++c) {
        host_layout(m, n, S, dtype, opts, c, &r0, &mc, &off);
        cudaStream_t sc = dual && (c & 1) ? s2 : s;
        if (cudaStreamWaitEvent(sc, ev[c], 0) != cudaSuccess) return join_fail(CAQR_ERR_CUDA);
        const size_t wb = caqr_workspace_bytes(mc, n, dtype, opts);
        if (S == 1) {
            rc = factor_impl<T>(mc, n, A + r0, lda, R, ldr, wsb + off, wb, opts, s, dtype);
            return rc ? join_fail(rc) : 0;
        }
        rc = factor_impl<T>(mc, n, A + r0, lda, Rs + (int64_t)c * n, ld, wsb + off, wb, opts, sc, dtype);
    }
    if (rc) return join_fail(rc);
    if (dual && (cudaEventRecord(ev[S + 1], s2) != cudaSuccess || cudaStreamWaitEvent(s, ev[S + 1], 0) != cudaSuccess))
        return join_fail(CAQR_ERR_CUDA);
    return combine_impl<T>(S, n, Rs, ld, R, ldr, wsb + cw_off, caqr_combine_workspace_bytes(S, n, dtype), s,
                           dtype);
}

// Plan search (caqr_tune): every candidate (leaf_rows, panel_cols) whose plan
// is valid and distinct, timed on a scratch copy of A.
template <typename T>
static int tune_impl(int64_t m, int64_t n, const T* A, int64_t lda, int reps, int dtype, caqr_opts* best,
                     float* best_ms, float* default_ms, int* ntried, cudaStream_t s) {
    if (m < 0) return -1;
    if (n < 0 || n > m) return -2;
    if (lda < std::max<int64_t>(1, m)) return -5;
    if (!best || !best_ms) return -7;
    if (!A && m > 0 && n > 0) return -4;
    *best = caqr_opts{};
    *best_ms = 0.f;
    if (default_ms) *default_ms = 0.f;
    if (ntried) *ntried = 0;
    if (m == 0 || n == 0) return 0;
    reps = std::max(1, std::min(reps, 50));
    // candidates: the default first (ties keep it), then the sweep axes of
    // P:L796-824 (tile height; panel-group width for wide matrices)
    const int64_t leafs[] = {0, 64, 96, 128, 160, 192, 224, 256};
    std::vector<int64_t> nbs = {0};
    for (int64_t nb : {32, 64, 96, 128, 160, 192, 224, 256})
        if (nb < n) nbs.push_back(nb);
    struct Cand {
        caqr_opts o;
        int64_t b, nb;
        bool chain, skinny;
        size_t ws;
    };
    std::vector<Cand> cands;
    for (int64_t nb : nbs)
        for (int64_t lf : leafs) {
            caqr_opts o{};
            o.leaf_rows = lf;
            o.panel_cols = nb;
            Plan pl;
            if (make_plan(m, n, dtype, &o, 9, &pl)) continue;
            bool dup = false;
            for (const Cand& c : cands)
                dup |= c.b == pl.b && c.nb == pl.nb && c.chain == pl.chain && c.skinny == pl.skinny;
            if (!dup) cands.push_back(Cand{o, pl.b, pl.nb, pl.chain, pl.skinny, std::max<size_t>(plan_ws_bytes(pl), 256)});
        }
    size_t wsmax = 256;
    for (const Cand& c : cands) wsmax = std::max(wsmax, c.ws);
    T *Ac = nullptr, *Rc = nullptr;
    void* ws = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(&Ac), sizeof(T) * (size_t)m * n);
    if (e == cudaSuccess) e = cudaMalloc(reinterpret_cast<void**>(&Rc), sizeof(T) * (size_t)n * n);
    if (e == cudaSuccess) e = cudaMalloc(&ws, wsmax);
    if (e == cudaSuccess) e = cudaEventCreate(&e0);
    if (e == cudaSuccess) e = cudaEventCreate(&e1);
    int rc = 0;
    float bestt = 0.f;
    int tried = 0;
    for (size_t ci = 0; ci < cands.size() && e == cudaSuccess && !rc; ++ci) {
        std::vector<float> ts;
        for (int r = 0; r <= reps && e == cudaSuccess && !rc; ++r) {  // r = 0: warm-up
            e = cudaMemcpy2DAsync(Ac, sizeof(T) * m, A, sizeof(T) * lda, sizeof(T) * m, n,
                                  cudaMemcpyDeviceToDevice, s);
            if (e == cudaSuccess) e = cudaEventRecord(e0, s);
            if (e == cudaSuccess)
                rc = factor_impl<T>(m, n, Ac, m, Rc, n, ws, cands[ci].ws, &cands[ci].o, s, dtype);
            if (!rc && e == cudaSuccess) e = cudaEventRecord(e1, s);
            if (!rc && e == cudaSuccess) e = cudaEventSynchronize(e1);
            float ms = 0.f;
            if (!rc && e == cudaSuccess) e = cudaEventElapsedTime(&ms, e0, e1);
            if (r > 0) ts.push_back(ms);
        }
        if (rc || e != cudaSuccess) break;
        std::sort(ts.begin(), ts.end());
        const float t = ts[ts.size() / 2];
        ++tried;
        if (ci == 0 && default_ms) *default_ms = t;
        if (ci == 0 || t < bestt) {
            bestt = t;
            *best = cands[ci].o;
        }
    }
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    if (Ac) cudaFree(Ac);
    if (Rc) cudaFree(Rc);
    if (ws) cudaFree(ws);
    if (ntried) *ntried = tried;
    *best_ms = bestt;
    if (rc) return rc;
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    return 0;
}

extern "C" {

int caqr_tune(int64_t m, int64_t n, int dtype, const void* A, int64_t lda, int reps, caqr_opts* best,
              float* best_ms, float* default_ms, int* ntried, caqr_stream_t stream) {
    if (dtype == CAQR_F32)
        return tune_impl<float>(m, n, static_cast<const float*>(A), lda, reps, dtype, best, best_ms, default_ms,
                                ntried, stream);
    if (dtype == CAQR_F64)
        return tune_impl<double>(m, n, static_cast<const double*>(A), lda, reps, dtype, best, best_ms, default_ms,
                                 ntried, stream);
    return -3;
}

size_t caqr_workspace_bytes(int64_t m, int64_t n, int dtype, const caqr_opts* opts) {
    if (m < 0 || n < 0 || n > m || (dtype != CAQR_F32 && dtype != CAQR_F64)) return 0;
    Plan pl;
    if (make_plan(m, n, dtype, opts, 4, &pl)) return 0;
    return std::max<size_t>(plan_ws_bytes(pl), 256);
}

int caqr_factor_f32(int64_t m, int64_t n, float* A, int64_t lda, float* R, int64_t ldr, void* ws,
                    size_t ws_bytes, const caqr_opts* opts, caqr_stream_t stream) {
    return factor_impl<float>(m, n, A, lda, R, ldr, ws, ws_bytes, opts, stream, CAQR_F32);
}
int caqr_factor_f64(int64_t m, int64_t n, double* A, int64_t lda, double* R, int64_t ldr,
                    void* ws, size_t ws_bytes, const caqr_opts* opts, caqr_stream_t stream) {
    return factor_impl<double>(m, n, A, lda, R, ldr, ws, ws_bytes, opts, stream, CAQR_F64);
}
int caqr_apply_qt_f32(int64_t m, int64_t n, const float* A, int64_t lda, const void* ws, int64_t k,
                      float* C, int64_t ldc, const caqr_opts* opts, caqr_stream_t stream) {
    return apply_impl<float>(m, n, A, lda, ws, k, C, ldc, opts, stream, CAQR_F32, 1);
}
int caqr_apply_qt_f64(int64_t m, int64_t n, const double* A, int64_t lda, const void* ws,
                      int64_t k, double* C, int64_t ldc, const caqr_opts* opts,
                      caqr_stream_t stream) {
    return apply_impl<double>(m, n, A, lda, ws, k, C, ldc, opts, stream, CAQR_F64, 1);
}
int caqr_apply_q_f32(int64_t m, int64_t n, const float* A, int64_t lda, const void* ws, int64_t k,
                     float* C, int64_t ldc, const caqr_opts* opts, caqr_stream_t stream) {
    return apply_impl<float>(m, n, A, lda, ws, k, C, ldc, opts, stream, CAQR_F32, 0);
}
int caqr_apply_q_f64(int64_t m, int64_t n, const double* A, int64_t lda, const void* ws, int64_t k,
                     double* C, int64_t ldc, const caqr_opts* opts, caqr_stream_t stream) {
    return apply_impl<double>(m, n, A, lda, ws, k, C, ldc, opts, stream, CAQR_F64, 0);
}
int caqr_form_q_f32(int64_t m, int64_t n, const float* A, int64_t lda, const void* ws, float* Q,
                    int64_t ldq, const caqr_opts* opts, caqr_stream_t stream) {
    return form_q_impl<float>(m, n, A, lda, ws, Q, ldq, opts, stream, CAQR_F32);
}
int caqr_form_q_f64(int64_t m, int64_t n, const double* A, int64_t lda, const void* ws, double* Q,
                    int64_t ldq, const caqr_opts* opts, caqr_stream_t stream) {
    return form_q_impl<double>(m, n, A, lda, ws, Q, ldq, opts, stream, CAQR_F64);
}

size_t caqr_combine_workspace_bytes(int P, int64_t n, int dtype) {
    if (P < 1 || n < 0 || n > kMaxGroup || (dtype != CAQR_F32 && dtype != CAQR_F64)) return 0;
    if (n == 0) return 256;
    const Geom G = combine_geom(P, n, (int64_t)P * n);
    // T blocks + room for P contiguous n x n blocks (the NCCL receive buffer of
    // caqr_dist_factor_*).
    const size_t es = dtype == CAQR_F64 ? 8 : 4;
    return group_ws_bytes(G, es) + (size_t)P * n * n * es;
}
int caqr_combine_f32(int P, int64_t n, float* Rs, int64_t ld, float* R, int64_t ldr, void* ws,
                     size_t ws_bytes, caqr_stream_t stream) {
    return combine_impl<float>(P, n, Rs, ld, R, ldr, ws, ws_bytes, stream, CAQR_F32);
}
int caqr_combine_f64(int P, int64_t n, double* Rs, int64_t ld, double* R, int64_t ldr, void* ws,
                     size_t ws_bytes, caqr_stream_t stream) {
    return combine_impl<double>(P, n, Rs, ld, R, ldr, ws, ws_bytes, stream, CAQR_F64);
}
int caqr_combine_apply_f32(int P, int64_t n, const float* Rs, int64_t ld, const void* ws, int trans,
                           int64_t k, float* C, int64_t ldc, caqr_stream_t stream) {
    return combine_apply_impl<float>(P, n, Rs, ld, ws, trans, k, C, ldc, stream);
}
int caqr_combine_apply_f64(int P, int64_t n, const double* Rs, int64_t ld, const void* ws,
                           int trans, int64_t k, double* C, int64_t ldc, caqr_stream_t stream) {
    return combine_apply_impl<double>(P, n, Rs, ld, ws, trans, k, C, ldc, stream);
}

const char* caqr_strerror(int info) {
    if (info == 0) return "success";
    if (info == CAQR_ERR_CUDA) return "CUDA launch failed (see caqr_last_cuda_error)";
    if (info == CAQR_ERR_NCCL) return "NCCL call failed";
    if (info == CAQR_ERR_UNSUPPORTED) return "unsupported size";
    if (info == CAQR_ERR_TIMEOUT) return "distributed call timed out (communicator aborted)";
    if (info < 0) return "illegal argument (-info = position)";
    return "unknown";
}
int caqr_last_cuda_error(void) { return g_last_cuda_error; }

int caqr_trace_begin(int capacity) {
    if (capacity < 1) return -1;
    std::lock_guard<std::mutex> lk(g_trace.mu);
    if (g_trace.on) return -2;
    if (g_trace.cap < capacity) {
        for (int i = 0; i < 2 * g_trace.cap; ++i) cudaEventDestroy(g_trace.ev[i]);
        delete[] g_trace.ev;
        delete[] g_trace.kid;
        delete[] g_trace.flops;
        delete[] g_trace.bytes;
        g_trace.ev = new cudaEvent_t[2 * capacity];
        g_trace.kid = new int[capacity];
        g_trace.flops = new double[capacity];
        g_trace.bytes = new double[capacity];
        for (int i = 0; i < 2 * capacity; ++i)
            if (cudaEventCreate(&g_trace.ev[i]) != cudaSuccess) {
                g_trace.cap = i / 2;
                return CAQR_ERR_CUDA;
            }
        g_trace.cap = capacity;
    }
    g_trace.n = 0;
    g_trace.on = true;
    return 0;
}

int caqr_trace_end(int* kernel_ids, float* ms, double* flops, double* bytes, int cap) {
    std::lock_guard<std::mutex> lk(g_trace.mu);
    g_trace.on = false;
    const int n = std::min(g_trace.n, cap);
    for (int i = 0; i < n; ++i) {
        float t = 0.f;
        if (cudaEventSynchronize(g_trace.ev[2 * i + 1]) != cudaSuccess ||
            cudaEventElapsedTime(&t, g_trace.ev[2 * i], g_trace.ev[2 * i + 1]) != cudaSuccess)
            t = -1.f;
        if (kernel_ids) kernel_ids[i] = g_trace.kid[i];
        if (ms) ms[i] = t;
        if (flops) flops[i] = g_trace.flops[i];
        if (bytes) bytes[i] = g_trace.bytes[i];
    }
    return g_trace.n;
}

int caqr_debug_profile_read(unsigned long long out[16]) {
    if (!g_prof) return -1;
    cudaDeviceSynchronize();
    cudaMemcpy(out, g_prof, 16 * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
    cudaMemset(g_prof, 0, 16 * sizeof(unsigned long long));
    return 0;
}

const char* caqr_kernel_name(int id) { return (id >= 0 && id < K_NUM) ? kKernelNames[id] : "?"; }

const char* caqr_build_info(void) {
    return "libcaqr: sm_100a TSQR/CAQR (panel_factor + panel_update kernels, FFMA/DFMA), "
           "built " __DATE__ " " __TIME__;
}

int caqr_plan_info(int64_t m, int64_t n, int dtype, const caqr_opts* opts, int64_t out[8]) {
    if (!out) return -5;
    if (m < 0) return -1;
    if (n < 0 || n > m) return -2;
    if (dtype != CAQR_F32 && dtype != CAQR_F64) return -3;
    Plan pl;
    int rc = make_plan(m, n, dtype, opts, 4, &pl);
    if (rc) return rc;
    std::memset(out, 0, 8 * sizeof(int64_t));
    out[0] = pl.b;
    out[1] = pl.nb;
    out[2] = pl.ngroups;
    if (pl.ngroups == 0) return 0;
    const Geom G = group_geom(pl, 0, m);
    out[3] = G.L;
    out[4] = tree_levels(G.P);
    out[5] = G.npan;
    out[7] = G.P;
    int64_t launches = 1;  // extract_r
    for (int64_t g = 0; g < pl.ngroups; ++g) {
        const Geom Gg = group_geom(pl, g, m);
        const int nl = tree_levels(Gg.P);
        if (pl.chain)
            launches += 2;  // chain kernel + the fused kernel's tree
        else if (fused_ok(Gg) || (pl.skinny && Gg.npan == 1))
            launches += 1;
        else
            launches += (int64_t)(nl + Gg.K) * (2 * Gg.npan - 1);
        const int64_t trail0 = Gg.col0 + Gg.ncols;
        if (trail0 < n) {  // trailing update (defaults: early start, FFMA apply)
            launches += 1;  // the next group's columns: one cooperative launch
            if (n - trail0 > pl.nb) launches += nl + 1;  // the rest beside the next TSQR: chains + levels
        }
    }
    out[6] = launches;
    return 0;
}


// ---- application layer (SVD via QR, robust PCA) ----------------------------
int caqr_svd_small_f32(int64_t n, const float* R, int64_t ldr, float* U, int64_t ldu, float* sigma, float* V,
                       int64_t ldv, caqr_stream_t stream) {
    return svd_small_impl<float>(n, R, ldr, U, ldu, sigma, V, ldv, (cudaStream_t)stream);
}
int caqr_svd_small_f64(int64_t n, const double* R, int64_t ldr, double* U, int64_t ldu, double* sigma, double* V,
                       int64_t ldv, caqr_stream_t stream) {
    return svd_small_impl<double>(n, R, ldr, U, ldu, sigma, V, ldv, (cudaStream_t)stream);
}

int caqr_svt_core_f32(int64_t n, const float* U, int64_t ldu, const float* sigma, const float* V, int64_t ldv,
                      float tau, float* W, int64_t ldw, caqr_stream_t stream) {
    if (n < 0 || n > kSvdMaxN) return -1;
    if (ldu < std::max<int64_t>(1, n)) return -3;
    if (ldv < std::max<int64_t>(1, n)) return -6;
    if (ldw < std::max<int64_t>(1, n)) return -9;
    if (n == 0) return 0;
    if (!U) return -2;
    if (!sigma) return -4;
    if (!V) return -5;
    if (!W) return -8;
    cudaStream_t s = (cudaStream_t)stream;
    TraceScope ts(K_SVT_CORE, 2.0 * n * n * n, 4.0 * 3 * n * n, s);
    svt_core_kernel<float><<<(unsigned)n, 128, 0, s>>>((int)n, U, ldu, sigma, V, ldv, tau, W, ldw);
    return launch_status();
}

int caqr_svt_core_r_f32(int64_t n, const float* U, int64_t ldu, const float* sigma, const float* R, int64_t ldr,
                        float tau, float* W, int64_t ldw, caqr_stream_t stream) {
    if (n < 0 || n > kSvdMaxN) return -1;
    if (ldu < std::max<int64_t>(1, n)) return -3;
    if (ldr < std::max<int64_t>(1, n)) return -6;
    if (ldw < std::max<int64_t>(1, n)) return -9;
    if (n == 0) return 0;
    if (!U) return -2;
    if (!sigma) return -4;
    if (!R) return -5;
    if (!W) return -8;
    cudaStream_t s = (cudaStream_t)stream;
    TraceScope ts(K_SVT_CORE, 4.0 * n * n * n, 4.0 * 3 * n * n, s);
    svt_core_r_kernel<float><<<(unsigned)n, 128, 0, s>>>((int)n, U, ldu, sigma, R, ldr, tau, W, ldw);
    return launch_status();
}

int caqr_embed_top_f32(int64_t m, int64_t n, const float* W, int64_t ldw, float* C, int64_t ldc,
                       caqr_stream_t stream) {
    if (m < 0) return -1;
    if (n < 0 || n > m) return -2;
    if (ldw < std::max<int64_t>(1, n)) return -4;
    if (ldc < std::max<int64_t>(1, m)) return -6;
    if (m == 0 || n == 0) return 0;
    if (!W) return -3;
    if (!C) return -5;
    cudaStream_t s = (cudaStream_t)stream;
    TraceScope ts(K_EMBED_TOP, 0.0, 4.0 * m * n, s);
    embed_top_kernel<float><<<elem_grid(m * n, 256), 256, 0, s>>>(m, n, W, ldw, C, ldc);
    return launch_status();
}

int caqr_rpca_update_f32(int64_t m, int64_t n, const float* M, int64_t ldm, const float* L, int64_t ldl, float* S,
                         int64_t lds, float* Y, int64_t ldy, float* X, int64_t ldx, float mu, float mu_next,
                         float lambda, double* resid, caqr_stream_t stream) {
    if (m < 0) return -1;
    if (n < 0) return -2;
    const int64_t lm = std::max<int64_t>(1, m);
    if (ldm < lm) return -4;
    if (ldl < lm) return -6;
    if (lds < lm) return -8;
    if (ldy < lm) return -10;
    if (ldx < lm) return -12;
    if (!(mu > 0.f)) return -13;
    if (!(mu_next > 0.f)) return -14;
    if (!(lambda >= 0.f)) return -15;
    if (!resid) return -16;
    if (m > 0 && n > 0) {
        if (!M) return -3;
        if (!L) return -5;
        if (!S) return -7;
        if (!Y) return -9;
        if (!X) return -11;
    }
    cudaStream_t s = (cudaStream_t)stream;
    {
        TraceScope ts(K_RPCA_UPDATE, 12.0 * m * n, 4.0 * 7 * m * n, s);
        rpca_update_kernel<float><<<kRpcaBlocks, 256, 0, s>>>(m, n, M, ldm, L, ldl, S, lds, Y, ldy, X, ldx, mu,
                                                              mu_next, lambda, resid);
    }
    sum_parts_kernel<<<1, 256, 0, s>>>(kRpcaBlocks, resid);
    return launch_status();
}

int caqr_rpca_init_f32(int64_t m, int64_t n, const float* M, int64_t ldm, float yscale, float* S, int64_t lds,
                       float* Y, int64_t ldy, float* X, int64_t ldx, float mu, caqr_stream_t stream) {
    if (m < 0) return -1;
    if (n < 0) return -2;
    const int64_t lm = std::max<int64_t>(1, m);
    if (ldm < lm) return -4;
    if (lds < lm) return -7;
    if (ldy < lm) return -9;
    if (ldx < lm) return -11;
    if (!(mu > 0.f)) return -12;
    if (m == 0 || n == 0) return 0;
    if (!M) return -3;
    if (!S) return -6;
    if (!Y) return -8;
    if (!X) return -10;
    cudaStream_t s = (cudaStream_t)stream;
    TraceScope ts(K_RPCA_INIT, 2.0 * m * n, 4.0 * 4 * m * n, s);
    rpca_init_kernel<float><<<elem_grid(m * n, 256), 256, 0, s>>>(m, n, M, ldm, yscale, S, lds, Y, ldy, X, ldx, mu);
    return launch_status();
}

int caqr_rpca_schedule_f32(const float* sigma, const float* amax, double lambda, double mu_factor,
                           double mu_max_factor, double rho, double* sched, caqr_stream_t stream) {
    if (!sigma) return -1;
    if (!amax) return -2;
    if (!(lambda > 0.0)) return -3;
    if (!(mu_factor > 0.0)) return -4;
    if (!(mu_max_factor >= 1.0)) return -5;
    if (!(rho >= 1.0)) return -6;
    if (!sched) return -7;
    rpca_schedule_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(sigma, amax, lambda, mu_factor, mu_max_factor, rho,
                                                             sched);
    return launch_status();
}

int caqr_rpca_init_sched_f32(int64_t m, int64_t n, const float* M, int64_t ldm, const double* sched, float* S,
                             int64_t lds, float* Y, int64_t ldy, float* X, int64_t ldx, caqr_stream_t stream) {
    if (m < 0) return -1;
    if (n < 0) return -2;
    const int64_t lm = std::max<int64_t>(1, m);
    if (ldm < lm) return -4;
    if (!sched) return -5;
    if (lds < lm) return -7;
    if (ldy < lm) return -9;
    if (ldx < lm) return -11;
    if (m == 0 || n == 0) return 0;
    if (!M) return -3;
    if (!S) return -6;
    if (!Y) return -8;
    if (!X) return -10;
    cudaStream_t s = (cudaStream_t)stream;
    TraceScope ts(K_RPCA_INIT, 2.0 * m * n, 4.0 * 4 * m * n, s);
    rpca_init_kernel<float><<<elem_grid(m * n, 256), 256, 0, s>>>(m, n, M, ldm, 0.f, S, lds, Y, ldy, X, ldx, 1.f,
                                                                  sched);
    return launch_status();
}

int caqr_svt_core_r_sched_f32(int64_t n, const float* U, int64_t ldu, const float* sigma, const float* R,
                              int64_t ldr, const double* sched, float* W, int64_t ldw, caqr_stream_t stream) {
    if (n < 0 || n > kSvdMaxN) return -1;
    if (ldu < std::max<int64_t>(1, n)) return -3;
    if (ldr < std::max<int64_t>(1, n)) return -6;
    if (!sched) return -7;
    if (ldw < std::max<int64_t>(1, n)) return -9;
    if (n == 0) return 0;
    if (!U) return -2;
    if (!sigma) return -4;
    if (!R) return -5;
    if (!W) return -8;
    cudaStream_t s = (cudaStream_t)stream;
    TraceScope ts(K_SVT_CORE, 4.0 * n * n * n, 4.0 * 3 * n * n, s);
    svt_core_r_kernel<float><<<(unsigned)n, 128, 0, s>>>((int)n, U, ldu, sigma, R, ldr, 0.f, W, ldw, sched);
    return launch_status();
}

int caqr_rpca_update_sched_f32(int64_t m, int64_t n, const float* M, int64_t ldm, const float* L, int64_t ldl,
                               float* S, int64_t lds, float* Y, int64_t ldy, float* X, int64_t ldx, double* sched,
                               double* resid, caqr_stream_t stream) {
    if (m < 0) return -1;
    if (n < 0) return -2;
    const int64_t lm = std::max<int64_t>(1, m);
    if (ldm < lm) return -4;
    if (ldl < lm) return -6;
    if (lds < lm) return -8;
    if (ldy < lm) return -10;
    if (ldx < lm) return -12;
    if (!sched) return -13;
    if (!resid) return -14;
    if (m > 0 && n > 0) {
        if (!M) return -3;
        if (!L) return -5;
        if (!S) return -7;
        if (!Y) return -9;
        if (!X) return -11;
    }
    cudaStream_t s = (cudaStream_t)stream;
    {
        TraceScope ts(K_RPCA_UPDATE, 12.0 * m * n, 4.0 * 7 * m * n, s);
        rpca_update_kernel<float><<<kRpcaBlocks, 256, 0, s>>>(m, n, M, ldm, L, ldl, S, lds, Y, ldy, X, ldx, 1.f, 1.f,
                                                              0.f, resid, sched);
    }
    sum_parts_kernel<<<1, 256, 0, s>>>(kRpcaBlocks, resid, sched);  // also mu <- min(rho mu, mu_max)
    return launch_status();
}

int caqr_absmax_f32(int64_t m, int64_t n, const float* M, int64_t ldm, float* out, caqr_stream_t stream) {
    if (m < 0) return -1;
    if (n < 0) return -2;
    if (ldm < std::max<int64_t>(1, m)) return -4;
    if (!out) return -5;
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e = cudaMemsetAsync(out, 0, sizeof(float), s);
    if (e != cudaSuccess) {
        g_last_cuda_error = (int)e;
        return CAQR_ERR_CUDA;
    }
    if (m == 0 || n == 0) return 0;
    if (!M) return -3;
    TraceScope ts(K_ABSMAX, 0.0, 4.0 * m * n, s);
    absmax_kernel<float><<<elem_grid(m * n, 256), 256, 0, s>>>(m, n, M, ldm, out);
    return launch_status();
}


// ---- least squares (xGELS through the CAQR factorization) -------------------
int caqr_trsm_upper_f32(int64_t n, int64_t k, const float* R, int64_t ldr, float* B, int64_t ldb,
                        caqr_stream_t stream) {
    return trsm_impl<float>(n, k, R, ldr, B, ldb, (cudaStream_t)stream);
}
int caqr_trsm_upper_f64(int64_t n, int64_t k, const double* R, int64_t ldr, double* B, int64_t ldb,
                        caqr_stream_t stream) {
    return trsm_impl<double>(n, k, R, ldr, B, ldb, (cudaStream_t)stream);
}
int caqr_lstsq_f32(int64_t m, int64_t n, const float* A, int64_t lda, const void* ws, int64_t k, float* B,
                   int64_t ldb, const caqr_opts* opts, caqr_stream_t stream) {
    int rc = apply_impl<float>(m, n, A, lda, ws, k, B, ldb, opts, (cudaStream_t)stream, CAQR_F32, 1);
    if (rc) return rc;
    return trsm_impl<float>(n, k, A, lda, B, ldb, (cudaStream_t)stream);  // R: A's top n x n upper triangle
}
int caqr_lstsq_f64(int64_t m, int64_t n, const double* A, int64_t lda, const void* ws, int64_t k, double* B,
                   int64_t ldb, const caqr_opts* opts, caqr_stream_t stream) {
    int rc = apply_impl<double>(m, n, A, lda, ws, k, B, ldb, opts, (cudaStream_t)stream, CAQR_F64, 1);
    if (rc) return rc;
    return trsm_impl<double>(n, k, A, lda, B, ldb, (cudaStream_t)stream);
}


int caqr_set_identity_f32(int64_t m, int64_t n, float* Q, int64_t ldq, caqr_stream_t stream) {
    return set_identity_impl<float>(m, n, Q, ldq, (cudaStream_t)stream);
}
int caqr_set_identity_f64(int64_t m, int64_t n, double* Q, int64_t ldq, caqr_stream_t stream) {
    return set_identity_impl<double>(m, n, Q, ldq, (cudaStream_t)stream);
}

size_t caqr_factor_host_workspace_bytes(int64_t m, int64_t n, int chunks, int dtype, const caqr_opts* opts) {
    int64_t r0, mc;
    size_t off;
    return host_layout(m, n, chunks, dtype, opts, 0, &r0, &mc, &off);
}
int caqr_factor_host_layout(int64_t m, int64_t n, int chunks, int dtype, const caqr_opts* opts, int c,
                            int64_t* out3) {
    if (!out3) return -7;
    if (c < 0 || c > chunks + 1) return -6;
    int64_t r0 = 0, mc = 0;
    size_t off = 0;
    if (host_layout(m, n, chunks, dtype, opts, c, &r0, &mc, &off) == 0) return -3;
    out3[0] = r0;
    out3[1] = mc;
    out3[2] = (int64_t)off;
    return 0;
}
int caqr_factor_host_f32(int64_t m, int64_t n, int chunks, const float* A_host, int64_t lda_host, float* A,
                         int64_t lda, float* R, int64_t ldr, void* ws, size_t ws_bytes, const caqr_opts* opts,
                         caqr_stream_t stream) {
    return factor_host_impl<float>(m, n, chunks, A_host, lda_host, A, lda, R, ldr, ws, ws_bytes, opts, stream,
                                   CAQR_F32);
}
int caqr_factor_host_f64(int64_t m, int64_t n, int chunks, const double* A_host, int64_t lda_host, double* A,
                         int64_t lda, double* R, int64_t ldr, void* ws, size_t ws_bytes, const caqr_opts* opts,
                         caqr_stream_t stream) {
    return factor_host_impl<double>(m, n, chunks, A_host, lda_host, A, lda, R, ldr, ws, ws_bytes, opts, stream,
                                    CAQR_F64);
}

}  // extern "C"
