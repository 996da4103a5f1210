/*
 * caqr.h -- C ABI of libcaqr.so: B200-native (sm_100a) TSQR / CAQR.
 *
 * Paper: M. Anderson, G. Ballard, J. Demmel, K. Keutzer, "Communication-Avoiding
 * QR Decomposition for GPUs", IPDPS 2011.  "P:Lnnn" below = line nnn of the
 * paper text, with its section.
 *
 * Operation (Sec. I): A = Q R with Q orthogonal (m x m) and R upper
 * triangular (n x n), for a real m x n matrix A with m >= n, in single precision
 * as the paper (Sec. IV) and in double precision.
 *
 * Method: TSQR panel factorisation (Sec. II.B, Fig. 2) -- the rows of
 * a panel are cut into leaves, each leaf is QR-factored by Householder
 * reflectors (kernel "factor"), the leaves' R factors are reduced
 * pairwise up a binary tree of structured stacked-triangle QRs (kernel
 * "factor_tree"; tree shape free) -- and, when n is
 * wider than one panel, CAQR (Sec. II.C, Fig. 3/4): the panel's
 * implicit Q^T is applied to the trailing columns leaf by leaf ("apply_qt_h",
 * P:L665-668) and node by node up the tree ("apply_qt_tree"), then
 * the grid is redrawn nb rows lower.  Reflectors are applied in
 * compact-WY form I - V T V^T (Sec. II.A) with T built from the
 * inner products of the vectors.
 *
 * Conventions for every entry point:
 *   - Matrices are column-major with a leading dimension ("originally
 *     stored in column major order").  ALL matrix and workspace pointers are
 *     DEVICE pointers (cudaMalloc'd or torch CUDA storage) on the current device,
 *     except A_host of caqr_factor_host_* (host memory, by name).
 *   - Calls only enqueue work on `stream` (0 = legacy default stream); they never
 *     synchronise the device, never allocate device memory, and can be captured
 *     into a CUDA graph (tests/test_gpu_parity.py test_cuda_graph_capture:
 *     factor, apply_qt, form_q, the CAQR loop with its early-start fork/join).
 *     They are reentrant (calls from several host threads: test_concurrent_
 *     caqr_calls_two_threads); the only process state is
 *     a lazily-filled per-device attribute cache and the lazily-created side
 *     stream (CAQR early start) and copy + second compute stream
 *     (caqr_factor_host_*) per device.
 *   - Return value: LAPACK "info".  0 = success; -i = argument i is illegal (the
 *     call does nothing); CAQR_ERR_CUDA (1) = a CUDA launch failed (see
 *     caqr_last_cuda_error); CAQR_ERR_NCCL (2) = an NCCL call failed.
 *     m = 0 or n = 0 is a quick return with 0 (dimensions and leading
 *     dimensions are checked first, pointers only when there is work, as
 *     LAPACK never dereferences them then).  NaN/Inf are not checked; they
 *     propagate as in LAPACK.
 *   - Householder convention (reading S1): LAPACK xLARFG
 *     (beta = -sign(alpha)||x||, v(head) = 1, tau = (beta-alpha)/beta).  R_jj may be
 *     negative; the library does not normalise signs.
 *   - Rows n..m-1 of Q^T C depend on the tree shape and leaf size (several
 *     correct answers, reading S17); rows 0..n-1 and every column norm
 *     do not.
 *   - `opts` selects the plan (leaf height, panel-group width).  NULL = the
 *     default plan for (m, n, dtype).  The SAME opts must be passed to
 *     caqr_workspace_bytes, caqr_factor_* and every later apply/form_q call on
 *     that factorisation.
 */
#ifndef CAQR_H
#define CAQR_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *caqr_stream_t; /* == cudaStream_t */

enum { CAQR_F32 = 0, CAQR_F64 = 1 };
enum { CAQR_OK = 0, CAQR_ERR_CUDA = 1, CAQR_ERR_NCCL = 2, CAQR_ERR_UNSUPPORTED = 3, CAQR_ERR_TIMEOUT = 4 };

/* Plan options; a field <= 0 means "default" (caqr_tune searches them).
 *   leaf_rows  b: rows per TSQR tile (P:L633 / P:L822-823 used 64 and 128 on
 *              Fermi; here a multiple of 32, b >= the panel-group width,
 *              b <= 256).  Default 224 for n <= 224, 256 for wider matrices;
 *              fp32 n <= 16 (streaming kernel): 256 for n <= 8, 128 for n <= 16.
 *              Consecutive tiles form chains (flat trees) of K = ceil(L/296)
 *              tiles (skinny: ~1184 / 2368 chains); the chains' R factors are
 *              reduced by a binary tree.
 *   panel_cols nb: CAQR panel-group width (one TSQR per group).
 *              Default: n if n <= 224 (one whole-width TSQR), else 128. */
typedef struct caqr_opts {
    int64_t leaf_rows;
    int64_t panel_cols;
    int64_t reserved[6];
} caqr_opts;

/* Bytes of device workspace the factorisation of an m x n matrix of `dtype`
 * needs (the T factors of every compact-WY block).  Returns 0 on illegal
 * arguments (m < 0, n < 0, n > m, bad dtype, bad opts). */
size_t caqr_workspace_bytes(int64_t m, int64_t n, int dtype, const caqr_opts *opts);

/* QR factorisation, SGEQRF semantics (Sec. V.C: "doesn't return Q
 * explicitly, instead it returns an intermediate representation that can later
 * be used to retrieve or apply Q").
 *   m, n       matrix size, m >= n >= 0                        (info -1, -2)
 *   A          device, m x n, lda >= max(1,m); overwritten      (info -3, -4)
 *              by the implicit-Q representation (Householder vectors of the
 *              leaves below the leaves' diagonals, tree vectors in the upper
 *              triangles of non-root leaf tops) and, in its top n x n upper
 *              triangle, by R.
 *   R          device, n x n, ldr >= max(1,n): receives R with  (info -5, -6)
 *              the strict lower triangle zeroed.
 *   ws         device workspace of ws_bytes >=                  (info -7, -8)
 *              caqr_workspace_bytes(m, n, dtype, opts); receives the T factors.
 *   opts       plan (may be NULL)                               (info -9)
 *   stream     CUDA stream.
 * A and ws together are the implicit Q; keep them unchanged for
 * caqr_apply_qt / caqr_apply_q / caqr_form_q. */
int caqr_factor_f32(int64_t m, int64_t n, float *A, int64_t lda, float *R, int64_t ldr,
                    void *ws, size_t ws_bytes, const caqr_opts *opts, caqr_stream_t stream);
int caqr_factor_f64(int64_t m, int64_t n, double *A, int64_t lda, double *R, int64_t ldr,
                    void *ws, size_t ws_bytes, const caqr_opts *opts, caqr_stream_t stream);

/* C <- Q^T C  (the trailing-matrix update of P:L603-610 applied to any C).
 *   m, n, A, lda, ws, opts : exactly as passed to caqr_factor_*   (info -1..-4, -5)
 *   k          columns of C, k >= 0                               (info -6)
 *   C          device, m x k, ldc >= max(1,m), updated in place   (info -7, -8)
 * Order: leaves, then the tree bottom-up (Fig. 4). */
int caqr_apply_qt_f32(int64_t m, int64_t n, const float *A, int64_t lda, const void *ws,
                      int64_t k, float *C, int64_t ldc, const caqr_opts *opts,
                      caqr_stream_t stream);
int caqr_apply_qt_f64(int64_t m, int64_t n, const double *A, int64_t lda, const void *ws,
                      int64_t k, double *C, int64_t ldc, const caqr_opts *opts,
                      caqr_stream_t stream);

/* C <- Q C (tree top-down, then leaves).  Arguments as caqr_apply_qt_*. */
int caqr_apply_q_f32(int64_t m, int64_t n, const float *A, int64_t lda, const void *ws,
                     int64_t k, float *C, int64_t ldc, const caqr_opts *opts,
                     caqr_stream_t stream);
int caqr_apply_q_f64(int64_t m, int64_t n, const double *A, int64_t lda, const void *ws,
                     int64_t k, double *C, int64_t ldc, const caqr_opts *opts,
                     caqr_stream_t stream);

/* Explicit thin Q (m x n) with A_original = Q R: SORGQR via CAQR (P:L905-910,
 * "retrieving Q explicitly (SORGQR) using CAQR is just as efficient as
 * factoring").  Q = (Q_leaves Q_tree) [I_n; 0].
 *   m, n, A, lda, ws, opts : as passed to caqr_factor_*     (info -1..-5)
 *   Q          device, m x n, ldq >= max(1,m); overwritten    (info -6, -7) */
int caqr_form_q_f32(int64_t m, int64_t n, const float *A, int64_t lda, const void *ws,
                    float *Q, int64_t ldq, const caqr_opts *opts, caqr_stream_t stream);
int caqr_form_q_f64(int64_t m, int64_t n, const double *A, int64_t lda, const void *ws,
                    double *Q, int64_t ldq, const caqr_opts *opts, caqr_stream_t stream);

/* ---- Combine: the extra tree level of a row-sharded (multi-GPU) TSQR --------
 * Not in the paper (single GPU); it is the distributed TSQR the
 * paper cites, one more tree level whose leaves are GPUs.
 * Rstack holds P n x n upper-triangular factors stacked vertically (a
 * (P*n) x n column-major matrix, ld >= P*n; entries below each diagonal are
 * ignored).  Factors the stack with the same structured binary tree as
 * caqr_factor (deterministic: bitwise-identical results on every rank that
 * passes the same stack), leaves the tree vectors in Rstack and the T factors
 * in ws, writes the combined R (strict lower zeroed) to R.
 *   P >= 1 (info -1), 0 <= n <= 256 (-2), Rstack/ld (-3, -4), R/ldr (-5, -6),
 *   ws/ws_bytes (-7, -8) with ws_bytes >= caqr_combine_workspace_bytes. */
size_t caqr_combine_workspace_bytes(int P, int64_t n, int dtype);
int caqr_combine_f32(int P, int64_t n, float *Rstack, int64_t ld, float *R, int64_t ldr,
                     void *ws, size_t ws_bytes, caqr_stream_t stream);
int caqr_combine_f64(int P, int64_t n, double *Rstack, int64_t ld, double *R, int64_t ldr,
                     void *ws, size_t ws_bytes, caqr_stream_t stream);
/* C (P*n x k, ld ldc) <- Qc^T C (trans = 1) or Qc C (trans = 0), Qc the
 * combine's orthogonal factor as left in Rstack/ws by caqr_combine_*. */
int caqr_combine_apply_f32(int P, int64_t n, const float *Rstack, int64_t ld, const void *ws,
                           int trans, int64_t k, float *C, int64_t ldc, caqr_stream_t stream);
int caqr_combine_apply_f64(int P, int64_t n, const double *Rstack, int64_t ld, const void *ws,
                           int trans, int64_t k, double *C, int64_t ldc, caqr_stream_t stream);

/* ---- Host-streamed factorisation (end-to-end from host memory) ------------
 * A = QR of a matrix that lives in HOST memory (pinned for overlap).  The rows
 * are split into `chunks` row blocks, chunk c = rows [m*c/chunks,
 * m*(c+1)/chunks); each block's H2D copy runs on a copy engine (a library copy
 * stream) while the previous blocks are factored by caqr_factor_* (odd chunks
 * on a second library stream joined back into `stream`, CAQR_HOST_DUAL=0: all
 * on `stream`);
 * the chunks' R factors are then reduced by caqr_combine_* — the extra tree
 * level of the distributed TSQR the paper cites, here with row
 * blocks of one GPU as its leaves.  Not in the paper (its runtimes exclude the
 * transfer); it hides the PCIe copy behind the factorisation.
 *   m, n        m >= n >= 0                                       (info -1, -2)
 *   chunks      1..1024; if > 1: n <= 256 and m/chunks >= n       (info -3)
 *   A_host      host, m x n column-major, lda_host >= max(1,m)    (info -4, -5)
 *   A           device, m x n, lda >= max(1,m): receives A, then   (info -6, -7)
 *               each chunk's implicit-Q representation (as caqr_factor_* on
 *               the chunk's rows)
 *   R           device, n x n, ldr >= n: the global R, strict      (info -8, -9)
 *               lower zeroed
 *   ws          device, ws_bytes >= caqr_factor_host_workspace_bytes (-10, -11)
 *   opts        plan of every chunk's factorisation (NULL = default) (-12)
 * Q = diag(Q_0..Q_{S-1}) * [rows n of each chunk -> Qc], Qc the combine's
 * orthogonal factor.  caqr_factor_host_layout(..., c, out3) gives, for
 * c < chunks, out3 = {first row, rows, byte offset of the chunk's workspace in
 * ws}; for c = chunks, {0, chunks*n, offset of the R stack ((chunks*n) x n,
 * ld chunks*n: the combine's tree vectors)}; for c = chunks+1, {0, 0, offset
 * of the combine workspace}: with them, caqr_apply_qt_* per chunk followed by
 * caqr_combine_apply_* on the chunks' top n rows applies Q^T (as for the
 * row-sharded multi-GPU factorization).  The caller keeps A_host unchanged
 * until the stream reaches the end of the call.  Calls from several host
 * threads are serialised while they issue (shared copy stream and events).
 * Layout query: 0, or -3 (bad
 * m, n, chunks, dtype, opts), -6 (c out of range), -7 (out3 NULL).
 * caqr_factor_host_workspace_bytes returns 0 on illegal arguments. */
size_t caqr_factor_host_workspace_bytes(int64_t m, int64_t n, int chunks, int dtype, const caqr_opts *opts);
int caqr_factor_host_layout(int64_t m, int64_t n, int chunks, int dtype, const caqr_opts *opts, int c,
                            int64_t *out3);
int caqr_factor_host_f32(int64_t m, int64_t n, int chunks, const float *A_host, int64_t lda_host, float *A,
                         int64_t lda, float *R, int64_t ldr, void *ws, size_t ws_bytes,
                         const caqr_opts *opts, caqr_stream_t stream);
int caqr_factor_host_f64(int64_t m, int64_t n, int chunks, const double *A_host, int64_t lda_host, double *A,
                         int64_t lda, double *R, int64_t ldr, void *ws, size_t ws_bytes,
                         const caqr_opts *opts, caqr_stream_t stream);

/* Q (m x n, ldq >= m) = [I_n; 0]: the start of an explicit Q (caqr_form_q does
 * it internally); used with caqr_combine_apply / caqr_apply_q to form the rows
 * of a row-sharded factorization's Q on each rank.
 * info: -1 m, -2 n (0 <= n <= m), -3 Q, -4 ldq. */
int caqr_set_identity_f32(int64_t m, int64_t n, float *Q, int64_t ldq, caqr_stream_t stream);
int caqr_set_identity_f64(int64_t m, int64_t n, double *Q, int64_t ldq, caqr_stream_t stream);

/* ---- Multi-GPU row-sharded TSQR over NCCL (one process per GPU) -----------
 * caqr_dist_create: nccl_unique_id = the 128-byte ncclUniqueId made by rank 0
 * and broadcast by the caller (e.g. through torch.distributed).  The handle owns
 * an NCCL communicator; the caller's current device is the rank's GPU.
 * Returns 0 or CAQR_ERR_NCCL / -1 (nranks < 1) / -2 (rank out of range) /
 * -3 (null pointers). */
typedef struct caqr_dist caqr_dist;
/* ncclGetUniqueId: writes the 128-byte id to out128 (host memory).  0 or
 * CAQR_ERR_NCCL, -1 if out128 is NULL.  Call on rank 0 only. */
int caqr_dist_unique_id(void *out128);
int caqr_dist_create(caqr_dist **handle, int nranks, int rank, const void *nccl_unique_id);
void caqr_dist_destroy(caqr_dist *handle);
/* Every rank: local TSQR of its m_local x n shard (m_local >= n: else -2),
 * ncclAllGather
 * of the local R factors over NVLink, then the same deterministic combine on
 * every rank -> the global R (identical bits on all ranks).
 *   A, lda, ws, ws_bytes: the local factorisation (caqr_workspace_bytes(m_local,
 *   n, dtype, opts));  gather: device, (nranks*n) x n, ld nranks*n, receives the
 *   stacked local R's and then the combine's tree vectors;  cws, cws_bytes:
 *   caqr_combine_workspace_bytes(nranks, n, dtype). */
int caqr_dist_factor_f32(caqr_dist *h, int64_t m_local, int64_t n, float *A, int64_t lda,
                         float *R, int64_t ldr, void *ws, size_t ws_bytes, float *gather,
                         void *cws, size_t cws_bytes, const caqr_opts *opts,
                         caqr_stream_t stream);
int caqr_dist_factor_f64(caqr_dist *h, int64_t m_local, int64_t n, double *A, int64_t lda,
                         double *R, int64_t ldr, void *ws, size_t ws_bytes, double *gather,
                         void *cws, size_t cws_bytes, const caqr_opts *opts,
                         caqr_stream_t stream);

/* The post-exchange half of caqr_dist_factor, NCCL-free (caqr_dist_factor
 * calls it after its all-gather; a caller with its own exchange -- or a test
 * emulating P ranks on one GPU -- calls it directly): restack P contiguous
 * column-major n x n upper-triangular blocks (rank order; `blocks`, device,
 * P*n*n elements) into the (P*n) x n stack `gather` (ld ldg >= P*n) and run
 * caqr_combine on it: R (n x n, ldr >= n) = the global R, `gather` keeps the
 * combine's tree vectors, cws its T factors (caqr_combine_apply uses both).
 * The distributed TSQR's extra tree level.
 *   info: -1 P < 1, -2 n outside [0, 256], -3 blocks, -4 gather, -5 ldg,
 *   -6 R, -7 ldr, -8 cws, -9 cws_bytes < caqr_combine_workspace_bytes(P, n,
 *   dtype); CAQR_ERR_CUDA. */
int caqr_dist_combine_blocks_f32(int P, int64_t n, const float *blocks, float *gather, int64_t ldg,
                                 float *R, int64_t ldr, void *cws, size_t cws_bytes, caqr_stream_t stream);
int caqr_dist_combine_blocks_f64(int P, int64_t n, const double *blocks, double *gather, int64_t ldg,
                                 double *R, int64_t ldr, void *cws, size_t cws_bytes, caqr_stream_t stream);
/* Host-side wait with a deadline for the work a dist call enqueued on
 * `stream`: 0 once the stream is idle; on an NCCL asynchronous error, or when
 * timeout_ms (>= 0; < 0 = no deadline) passes first, the communicator is
 * aborted (ncclCommAbort: a peer that died or never arrived cannot hang this
 * rank) and CAQR_ERR_NCCL / CAQR_ERR_TIMEOUT is returned; the handle then only
 * accepts caqr_dist_destroy.  -1: h NULL; CAQR_ERR_CUDA: the stream failed. */
int caqr_dist_wait(caqr_dist *h, caqr_stream_t stream, int timeout_ms);

/* Peer-memory exchange of the local R factors -- the alternative to the NCCL
 * all-gather of caqr_dist_factor, with the exchange fused into the restack of
 * the combine's input (distributed TSQR; the paper's one-kernel-
 * per-step dataflow, carried across GPUs).  Rank `rank` of P:
 *   1. stores its n x n R (R, ldr; column-major) into slot `rank` of buffer
 *      (epoch & 1) of every rank q's mailbox (peer_mailbox[q], NVLink peer
 *      stores for q != rank);
 *   2. publishes peer_flags[q][rank] = epoch (system fence, then a
 *      system-scope release store);
 *   3. waits (acquire) for its own flags[q] >= epoch from every q and moves
 *      rank q's block to rows [q n, (q+1) n) of `gather` ((P n) x n,
 *      ld = P n, column-major), which caqr_combine_* then factors in place.
 * All P ranks must call it with the same P, n and epoch (1, 2, 3, ... one per
 * exchange; flags zeroed once before the first).  peer_mailbox / peer_flags:
 * DEVICE arrays of P device pointers (rank q's mailbox of
 * caqr_peer_mailbox_bytes(P, n, dtype) bytes and its P ints), mapped into this
 * process (caqr_ipc_open); the two mailbox buffers let a rank run ahead by
 * one exchange.  One CTA per peer, asynchronous on `stream`.
 * status (device int, may be NULL): set to CAQR_ERR_TIMEOUT if a wait exceeded
 * timeout_ms (> 0; 0 = wait forever) -- `gather` is then invalid.
 * info: -1 P < 1, -2 rank, -3 n (0..256), -4 R, -5 ldr, -6 peer_mailbox,
 * -7 peer_flags, -8 gather, -9 epoch < 1; CAQR_ERR_CUDA. */
size_t caqr_peer_mailbox_bytes(int P, int64_t n, int dtype);
int caqr_peer_exchange_f32(int P, int rank, int64_t n, const float *R, int64_t ldr, float *const *peer_mailbox,
                           int *const *peer_flags, float *gather, int epoch, int *status, int timeout_ms,
                           caqr_stream_t stream);
int caqr_peer_exchange_f64(int P, int rank, int64_t n, const double *R, int64_t ldr, double *const *peer_mailbox,
                           int *const *peer_flags, double *gather, int epoch, int *status, int timeout_ms,
                           caqr_stream_t stream);
/* The same exchange for P virtual ranks on ONE device (tests; a single
 * cooperative launch of P x P CTAs, CTA (q, r) playing rank r's sender to /
 * receiver from q, since ranks that wait on one another must be co-resident):
 * Rs / mailboxes / flags / gathers: device arrays of P device pointers. */
int caqr_peer_exchange_emulate_f32(int P, int64_t n, const float *const *Rs, int64_t ldr, float *const *mailboxes,
                                   int *const *flags, float *const *gathers, int epoch, caqr_stream_t stream);
int caqr_peer_exchange_emulate_f64(int P, int64_t n, const double *const *Rs, int64_t ldr,
                                   double *const *mailboxes, int *const *flags, double *const *gathers, int epoch,
                                   caqr_stream_t stream);
/* CUDA IPC of a device allocation (peer pointers across processes): the handle
 * is 64 opaque bytes.  0 / -1 / -2 / CAQR_ERR_CUDA. */
int caqr_ipc_handle(const void *dptr, void *out64);
int caqr_ipc_open(const void *handle64, void **dptr);
int caqr_ipc_close(void *dptr);

/* ---- Least squares through the factorization -------------
 * min ||A x - b||_2 for tall full-rank A, the use of QR the paper opens with
 * (P:L86-92), with LAPACK xGELS semantics: B <- Q^T B, then rows 0..n-1 of B
 * <- R^{-1} B[0:n] (the solution X, n x k); rows n..m-1 keep the residual's
 * components (their column norms are the residual norms; S17: the rows
 * themselves depend on the tree).
 *   m, n, A, lda, ws, opts : exactly as passed to caqr_factor_* (R is read from
 *   A's top n x n upper triangle)                    (info -1..-5 as apply_qt)
 *   k, B, ldb              : as C / ldc of caqr_apply_qt (info -6, -7, -8).
 * An exactly singular R gives Inf/NaN (no rank check, as xGELS). */
int caqr_lstsq_f32(int64_t m, int64_t n, const float *A, int64_t lda, const void *ws, int64_t k,
                   float *B, int64_t ldb, const caqr_opts *opts, caqr_stream_t stream);
int caqr_lstsq_f64(int64_t m, int64_t n, const double *A, int64_t lda, const void *ws, int64_t k,
                   double *B, int64_t ldb, const caqr_opts *opts, caqr_stream_t stream);
/* B (n x k, ldb >= n) <- R^{-1} B, R upper triangular n x n (ldr >= n), on the
 * device (one CTA per column, column-oriented back substitution; n <= 25,600
 * fp64 / 51,200 fp32).  info: -1 n, -2 k, -3 R, -4 ldr, -5 B, -6 ldb. */
int caqr_trsm_upper_f32(int64_t n, int64_t k, const float *R, int64_t ldr, float *B, int64_t ldb,
                        caqr_stream_t stream);
int caqr_trsm_upper_f64(int64_t n, int64_t k, const double *R, int64_t ldr, double *B, int64_t ldb,
                        caqr_stream_t stream);

/* ---- Application layer: SVD via QR and robust PCA (Sec. VI) -----------------
 * The paper's motivating workload: robust PCA of a video matrix
 * (one column per frame) by an alternating-directions method whose
 * main cost is the SVD of a tall-skinny matrix, done as A = QR, SVD(R) = U S V^T,
 * left vectors Q U.  With caqr_factor_f32 and caqr_apply_q_f32 the
 * whole iteration runs on the GPU (the paper takes the small SVD to the CPU,
 * P:L1068-1074; here it is one CTA).  All pointers are device pointers. */

/* SVD of a small square matrix, R = U diag(sigma) V^T, by one-sided (Hestenes)
 * Jacobi rotations in fp64 on one CTA.  R: n x n (ldr >= n, not modified);
 * U, V: n x n outputs (ldu, ldv >= n), orthogonal; sigma: n outputs, descending,
 * >= 0.  A zero singular value gets a zero U column.  0 <= n <= 112.  V may be
 * NULL: the right vectors are then not formed (about half the work; see
 * caqr_svt_core_r_f32, which needs only U, sigma and R).
 * info: -1 n, -2 R, -3 ldr, -4 U, -5 ldu, -6 sigma, -8 ldv; n = 0 quick return. */
int caqr_svd_small_f32(int64_t n, const float *R, int64_t ldr, float *U, int64_t ldu, float *sigma,
                       float *V, int64_t ldv, caqr_stream_t stream);
int caqr_svd_small_f64(int64_t n, const double *R, int64_t ldr, double *U, int64_t ldu, double *sigma,
                       double *V, int64_t ldv, caqr_stream_t stream);

/* Singular value threshold of the small factor (Fig. 11 "threshold these
 * singular values"): W = U diag(max(sigma - tau, 0)) V^T, n x n,
 * from caqr_svd_small's outputs.  The low-rank iterate is then L = Q [W; 0]
 * (caqr_embed_top_f32 + caqr_apply_q_f32).
 * info: -1 n (0..112), -2 U, -3 ldu, -4 sigma, -5 V, -6 ldv, -8 W, -9 ldw. */
int caqr_svt_core_f32(int64_t n, const float *U, int64_t ldu, const float *sigma, const float *V,
                      int64_t ldv, float tau, float *W, int64_t ldw, caqr_stream_t stream);

/* The same W without V: W = U diag(max(sigma - tau, 0) / sigma) U^T R, which equals
 * U diag(max(sigma - tau, 0)) V^T because U^T R = diag(sigma) V^T (only sigma > tau
 * is divided by).  R: the n x n matrix caqr_svd_small_f32 decomposed.
 * info: -1 n, -2 U, -3 ldu, -4 sigma, -5 R, -6 ldr, -8 W, -9 ldw. */
int caqr_svt_core_r_f32(int64_t n, const float *U, int64_t ldu, const float *sigma, const float *R,
                        int64_t ldr, float tau, float *W, int64_t ldw, caqr_stream_t stream);

/* C (m x n, ldc >= m) = [W; 0] with W n x n (ldw >= n), n <= m.
 * info: -1 m, -2 n, -3 W, -4 ldw, -5 C, -6 ldc. */
int caqr_embed_top_f32(int64_t m, int64_t n, const float *W, int64_t ldw, float *C, int64_t ldc,
                       caqr_stream_t stream);

/* One shrinkage + dual step of the alternating-directions iteration (P:L1107-1113,
 * reading S19 of DESIGN.md), elementwise over m x n, given the new low-rank
 * iterate L:
 *   S <- sign(t) max(|t| - lambda/mu, 0),  t = M - L + Y/mu
 *   Y <- Y + mu (M - L - S)
 *   X <- M - S + Y/mu_next                 (the next iteration's SVT input)
 *   resid[0] <- ||M - L - S||_F^2          (fixed-order reduction: deterministic)
 * M, L read; S, Y, X written (X may not alias the others).  resid: device
 * double[CAQR_RPCA_RESID_LEN] scratch.  mu, mu_next > 0, lambda >= 0.
 * info: -1 m, -2 n, -3..-12 the matrices / leading dimensions in order,
 * -13 mu, -14 mu_next, -15 lambda, -16 resid. */
#define CAQR_RPCA_RESID_LEN 1025
int caqr_rpca_update_f32(int64_t m, int64_t n, const float *M, int64_t ldm, const float *L, int64_t ldl,
                         float *S, int64_t lds, float *Y, int64_t ldy, float *X, int64_t ldx, float mu,
                         float mu_next, float lambda, double *resid, caqr_stream_t stream);
/* Start of the iteration: S = 0, Y = yscale M, X = M + Y/mu.
 * info: -1 m, -2 n, -3 M, -4 ldm, -6 S, -7 lds, -8 Y, -9 ldy, -10 X, -11 ldx, -12 mu. */
int caqr_rpca_init_f32(int64_t m, int64_t n, const float *M, int64_t ldm, float yscale, float *S,
                       int64_t lds, float *Y, int64_t ldy, float *X, int64_t ldx, float mu,
                       caqr_stream_t stream);
/* The iteration's scalar schedule on the device (reading S19 of DESIGN.md), so
 * that no step needs a host round trip: sched (device double[CAQR_RPCA_SCHED_LEN])
 * <- mu = mu_factor / sigma[0] (||M||_2 from the QR + small SVD of M), mu_max =
 * mu_max_factor mu, rho, yscale = 1 / max(sigma[0], amax[0] / lambda)
 * (||M||_inf from caqr_absmax_f32), lambda.  The *_sched_f32 variants of
 * rpca_init / svt_core_r / rpca_update read their scalars from it (in double,
 * converted as the by-value entry points receive them), and rpca_update_sched
 * advances mu <- min(rho mu, mu_max) after its pass (stream order).
 * info: -1 sigma, -2 amax, -3 lambda <= 0, -4 mu_factor <= 0,
 * -5 mu_max_factor < 1, -6 rho < 1, -7 sched. */
#define CAQR_RPCA_SCHED_LEN 8
int caqr_rpca_schedule_f32(const float *sigma, const float *amax, double lambda, double mu_factor,
                           double mu_max_factor, double rho, double *sched, caqr_stream_t stream);
/* caqr_rpca_init_f32 with yscale and mu from sched.  info as caqr_rpca_init_f32 with
 * -5 = sched. */
int caqr_rpca_init_sched_f32(int64_t m, int64_t n, const float *M, int64_t ldm, const double *sched, float *S,
                             int64_t lds, float *Y, int64_t ldy, float *X, int64_t ldx, caqr_stream_t stream);
/* caqr_svt_core_r_f32 with tau = 1 / sched[0].  info: -7 sched, otherwise as caqr_svt_core_r_f32. */
int caqr_svt_core_r_sched_f32(int64_t n, const float *U, int64_t ldu, const float *sigma, const float *R,
                              int64_t ldr, const double *sched, float *W, int64_t ldw, caqr_stream_t stream);
/* caqr_rpca_update_f32 with mu = sched[0], mu_next = min(rho mu, mu_max), lambda from sched;
 * sched[0] <- mu_next afterwards.  info: -13 sched, -14 resid, otherwise as caqr_rpca_update_f32. */
int caqr_rpca_update_sched_f32(int64_t m, int64_t n, const float *M, int64_t ldm, const float *L, int64_t ldl,
                               float *S, int64_t lds, float *Y, int64_t ldy, float *X, int64_t ldx, double *sched,
                               double *resid, caqr_stream_t stream);
/* out[0] (device float) = max |M_ij| (0 for an empty M).  info: -1 m, -2 n, -3 M, -4 ldm, -5 out. */
int caqr_absmax_f32(int64_t m, int64_t n, const float *M, int64_t ldm, float *out, caqr_stream_t stream);

/* Diagnostics. */
const char *caqr_strerror(int info);
int caqr_last_cuda_error(void);          /* cudaError_t of the last CAQR_ERR_CUDA (thread-local) */
const char *caqr_build_info(void);       /* "sm_100a ..." */
/* Launch tracing (profiling aid, not needed for correct use).
 * caqr_trace_begin(cap): from now on every kernel the library launches (any
 *   thread) is bracketed by two CUDA events recorded on its launching stream,
 *   up to cap launches; 0, -1 (cap < 1), -2 (already tracing), CAQR_ERR_CUDA.
 * caqr_trace_end(...): stops tracing, waits for the recorded events and fills
 *   up to cap entries: kernel id (caqr_kernel_name), duration in ms, and the
 *   host-computed algorithmic flops and bytes of that launch.  Returns the
 *   number of launches recorded (may exceed cap).  Output pointers may be NULL. */
int caqr_trace_begin(int capacity);
int caqr_trace_end(int *kernel_ids, float *ms, double *flops, double *bytes, int cap);
const char *caqr_kernel_name(int id);
/* Phase profile of the fused TSQR kernel (only when the process runs with
 * CAQR_PROFILE=1): per-phase clock64 cycle sums over all CTAs, then reset.
 * out[0..9] = task fetch, wait for children, stage panel, factor panel, store +
 * V form, G/T, stage C, V^T C, apply, publish; out[10]/out[11] = leaf / merge
 * panel-steps.  Returns 0, or -1 when profiling is off. */
int caqr_debug_profile_read(unsigned long long out[16]);

/* Plan introspection (host only; for tests and the bench's roofline bookkeeping).
 * Fills out[0..7] = {leaf_rows, panel_cols, groups, tiles(group 0),
 * tree_levels(group 0), panels(group 0), kernel_launches(factor), chains(group 0)}.
 * Returns 0 or a negative info. */
int caqr_plan_info(int64_t m, int64_t n, int dtype, const caqr_opts *opts, int64_t out[8]);

/* Plan search (the paper tunes its block sizes by search,
 * P:L796-804 Sec. IV.F, and picks the algorithm by shape).
 * Times caqr_factor of the m x n matrix A (device, column-major, lda; NOT
 * modified: every trial factors a scratch copy) for each candidate plan --
 * leaf_rows in {default, 64, 96, ..., 256} x panel_cols in {default, 32, 64,
 * ..., 256} (< n), keeping only valid plans that differ in (tile height,
 * group width, kernel family) -- as the median of `reps` (1..50) calls after
 * one warm-up, CUDA events on `stream`.
 *   best        out: the fastest plan's options (all-zero when the default
 *               plan is fastest; ties keep the default)           (-7 if NULL)
 *   best_ms     out: its time (ms)                                 (-7 if NULL)
 *   default_ms  out (may be NULL): the default plan's time (ms)
 *   ntried      out (may be NULL): plans timed
 * Info: -1 m < 0, -2 n < 0 or n > m, -3 dtype, -4 A NULL, -5 lda < m; or a
 * factor error; CAQR_ERR_CUDA.  Allocates its scratch (a copy of A, R, the
 * largest workspace) with cudaMalloc and synchronises on `stream`: a setup
 * call, not for graph capture.  Tested: tests/test_gpu_parity.py
 * (test_tune_*). */
int caqr_tune(int64_t m, int64_t n, int dtype, const void *A, int64_t lda, int reps, caqr_opts *best,
              float *best_ms, float *default_ms, int *ntried, caqr_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* CAQR_H */
