/*
 * oracle/householder.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded CPU Householder QR used to check the CUDA
 * path.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code, header,
 * table or constant with the product (paper_conf_ipps_andersonbdk11_b200/).
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md):
 *   - the QR problem A = QR, Q orthogonal, R upper triangular   P:L66-69 (Sec. I)
 *   - unblocked Householder QR: one reflector per column, applied to the
 *     trailing columns; Q = prod_i (I - tau_i u_i u_i^T)           P:L212-224 (Sec. II.A),
 *                                                                  P:L694-703 (Sec. IV.E)
 *   - "for each Householder vector u we first compute A^T u ... then we
 *     update each element of A with the scaled outer product"     P:L704-711 (Sec. IV.E)
 *   - LAPACK SGEQRF semantics: implicit Q (V below the diagonal, R on and
 *     above), explicit Q on request (SORGQR)                      P:L903-910 (Sec. V.C)
 *
 * Readings where the paper is silent or garbled:
 *   S1  reflector normalisation: LAPACK xLARFG.  beta = -copysign(||[alpha;x]||, alpha),
 *       tau = (beta - alpha)/beta, v = [1; x/(alpha - beta)].  The paper's
 *       u = v*(alpha-beta) and tau_paper = 2/||u||^2 = tau/(alpha-beta)^2 give the
 *       same H = I - tau v v^T.
 *   S2  x == 0 (sigma == 0): tau = 0, H = I, R_jj = alpha (LAPACK).
 *   S4  Q = H_0 H_1 ... H_{n-1}; Q^T C applies H_0 first ("repeated
 *       for each Householder vector").
 *   S16 no safmin/overflow rescaling (inputs are O(1)).
 *
 * Arithmetic: each routine exists twice, with accumulation type ACC = double
 * (suffix _d, used for fp32 inputs: the float->double conversion is exact) and
 * ACC = long double (suffix _ld, x87 80-bit, used for fp64 inputs).  All
 * arrays crossing this interface are double, column-major.  Sums run in index
 * order.  Build with -O2 -fno-fast-math -ffp-contract=off.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------------------
 * The three routines, written once as a macro over the accumulation type.
 * ------------------------------------------------------------------------- */
#define DEFINE_ORACLE(SUF, ACC, SQRT, COPYSIGN)                                   \
                                                                                  \
/* Unblocked Householder QR in place (xGEQR2).         \
 * On exit: R in the upper triangle, v_j (unit head implicit) below the          \
 * diagonal, tau[j] for j < min(m,n).  Returns 0, or -1 on bad arguments.    */ \
static int geqr2_##SUF(int64_t m, int64_t n, ACC *A, int64_t lda, ACC *tau)      \
{                                                                                 \
    int64_t k = m < n ? m : n;                                                    \
    for (int64_t j = 0; j < k; ++j) {                                             \
        ACC *x = A + j * lda;                  /* column j */                     \
        ACC alpha = x[j];                                                         \
        ACC sigma = 0;                         /* sum_{i>j} x_i^2 */              \
        for (int64_t i = j + 1; i < m; ++i) sigma += x[i] * x[i];                 \
        ACC t = 0;                                                                \
        if (sigma != 0) {                                                         \
            ACC mu = SQRT(alpha * alpha + sigma);                                 \
            ACC beta = -COPYSIGN(mu, alpha);                                      \
            t = (beta - alpha) / beta;                                            \
            ACC scale = 1 / (alpha - beta);                                       \
            for (int64_t i = j + 1; i < m; ++i) x[i] *= scale;                    \
            x[j] = beta;                                                          \
        }                                                                         \
        tau[j] = t;                                                               \
        if (t == 0) continue;                                                     \
        /* apply H_j = I - t v v^T to the trailing columns:           \
         * s = v^T a_c (matrix-vector product), a_c -= t s v (rank-1 update) */   \
        for (int64_t c = j + 1; c < n; ++c) {                                     \
            ACC *a = A + c * lda;                                                 \
            ACC s = a[j];                                                         \
            for (int64_t i = j + 1; i < m; ++i) s += x[i] * a[i];                 \
            s *= t;                                                               \
            a[j] -= s;                                                            \
            for (int64_t i = j + 1; i < m; ++i) a[i] -= s * x[i];                 \
        }                                                                         \
    }                                                                             \
    return 0;                                                                     \
}                                                                                 \
                                                                                  \
/* C (m x nc) <- Q^T C (trans = 1) or Q C (trans = 0), Q = H_0 ... H_{k-1}      \
 * from the k reflectors stored in V (m x k, as left by geqr2).  (xORM2R)     */  \
static int orm2r_##SUF(int trans, int64_t m, int64_t nc, int64_t k,               \
                       const ACC *V, int64_t ldv, const ACC *tau,                 \
                       ACC *C, int64_t ldc)                                       \
{                                                                                 \
    for (int64_t q = 0; q < k; ++q) {                                             \
        int64_t j = trans ? q : k - 1 - q;     /* Q^T: H_0 first; Q: H_{k-1} first */ \
        ACC t = tau[j];                                                           \
        if (t == 0) continue;                                                     \
        const ACC *v = V + j * ldv;                                               \
        for (int64_t c = 0; c < nc; ++c) {                                        \
            ACC *a = C + c * ldc;                                                 \
            ACC s = a[j];                      /* v_j = 1 */                      \
            for (int64_t i = j + 1; i < m; ++i) s += v[i] * a[i];                 \
            s *= t;                                                               \
            a[j] -= s;                                                            \
            for (int64_t i = j + 1; i < m; ++i) a[i] -= s * v[i];                 \
        }                                                                         \
    }                                                                             \
    return 0;                                                                     \
}                                                                                 \
                                                                                  \
/* public wrappers: double in / double out, ACC inside ----------------------*/ \
int oracle_geqr2_##SUF(int64_t m, int64_t n, double *A, int64_t lda,             \
                       double *tau)                                               \
{                                                                                 \
    if (m < 0 || n < 0 || lda < (m > 1 ? m : 1) || !A || !tau) return -1;         \
    int64_t k = m < n ? m : n;                                                    \
    ACC *W = (ACC *)malloc(sizeof(ACC) * (size_t)(m * n + k + 1));                \
    if (!W) return -2;                                                            \
    ACC *tw = W + m * n;                                                          \
    for (int64_t c = 0; c < n; ++c)                                               \
        for (int64_t i = 0; i < m; ++i) W[c * m + i] = (ACC)A[c * lda + i];       \
    geqr2_##SUF(m, n, W, m, tw);                                                  \
    for (int64_t c = 0; c < n; ++c)                                               \
        for (int64_t i = 0; i < m; ++i) A[c * lda + i] = (double)W[c * m + i];    \
    for (int64_t j = 0; j < k; ++j) tau[j] = (double)tw[j];                       \
    free(W);                                                                      \
    return 0;                                                                     \
}                                                                                 \
                                                                                  \
int oracle_orm2r_##SUF(int trans, int64_t m, int64_t nc, int64_t k,               \
                       const double *V, int64_t ldv, const double *tau,           \
                       double *C, int64_t ldc)                                    \
{                                                                                 \
    if (m < 0 || nc < 0 || k < 0 || k > m || ldv < (m > 1 ? m : 1) ||            \
        ldc < (m > 1 ? m : 1) || !V || !tau || !C) return -1;                     \
    ACC *W = (ACC *)malloc(sizeof(ACC) * (size_t)(m * k + m * nc + k + 1));       \
    if (!W) return -2;                                                            \
    ACC *Vw = W, *Cw = W + m * k, *tw = W + m * k + m * nc;                       \
    for (int64_t c = 0; c < k; ++c)                                               \
        for (int64_t i = 0; i < m; ++i) Vw[c * m + i] = (ACC)V[c * ldv + i];      \
    for (int64_t c = 0; c < nc; ++c)                                              \
        for (int64_t i = 0; i < m; ++i) Cw[c * m + i] = (ACC)C[c * ldc + i];      \
    for (int64_t j = 0; j < k; ++j) tw[j] = (ACC)tau[j];                          \
    orm2r_##SUF(trans, m, nc, k, Vw, m, tw, Cw, m);                               \
    for (int64_t c = 0; c < nc; ++c)                                              \
        for (int64_t i = 0; i < m; ++i) C[c * ldc + i] = (double)Cw[c * m + i];   \
    free(W);                                                                      \
    return 0;                                                                     \
}                                                                                 \
                                                                                  \
/* One call: factor A (m x n, m >= n) and return R (n x n, upper, strict lower   \
 * zeroed, ldr) and, if Q != NULL, the thin Q = H_0...H_{n-1} [I_n; 0] (m x n,   \
 * ldq) -- the SORGQR product of P:L905-910, formed as xORG2R does, all in ACC. */ \
int oracle_qr_##SUF(int64_t m, int64_t n, const double *A, int64_t lda,           \
                    double *R, int64_t ldr, double *Q, int64_t ldq)               \
{                                                                                 \
    if (m < 0 || n < 0 || n > m || lda < (m > 1 ? m : 1) || !A || !R ||           \
        ldr < (n > 1 ? n : 1) || (Q && ldq < (m > 1 ? m : 1))) return -1;         \
    ACC *W = (ACC *)malloc(sizeof(ACC) * (size_t)(2 * m * n + n + 1));           \
    if (!W) return -2;                                                            \
    ACC *Aw = W, *Qw = W + m * n, *tw = W + 2 * m * n;                            \
    for (int64_t c = 0; c < n; ++c)                                               \
        for (int64_t i = 0; i < m; ++i) Aw[c * m + i] = (ACC)A[c * lda + i];      \
    geqr2_##SUF(m, n, Aw, m, tw);                                                 \
    for (int64_t c = 0; c < n; ++c)                                               \
        for (int64_t i = 0; i < n; ++i)                                           \
            R[c * ldr + i] = i <= c ? (double)Aw[c * m + i] : 0.0;                \
    if (Q) {                                                                      \
        memset(Qw, 0, sizeof(ACC) * (size_t)(m * n));                             \
        for (int64_t i = 0; i < n; ++i) Qw[i * m + i] = 1;                        \
        orm2r_##SUF(0, m, n, n, Aw, m, tw, Qw, m);                                \
        for (int64_t c = 0; c < n; ++c)                                           \
            for (int64_t i = 0; i < m; ++i) Q[c * ldq + i] = (double)Qw[c * m + i]; \
    }                                                                             \
    free(W);                                                                      \
    return 0;                                                                     \
}

DEFINE_ORACLE(d, double, sqrt, copysign)
DEFINE_ORACLE(ld, long double, sqrtl, copysignl)

/* Same-precision fp32 variant (ACC = float): only used to calibrate what a
 * plain fp32 Householder reaches against the BASELINE bounds. */
DEFINE_ORACLE(f, float, sqrtf, copysignf)

/* LAPACK flop count of xGEQRF used by the metric (BASELINE.json "metric"):
 * 2 m n^2 - 2 n^3 / 3. */
double oracle_geqrf_flops(int64_t m, int64_t n)
{
    return 2.0 * (double)m * (double)n * (double)n - 2.0 * (double)n * (double)n * (double)n / 3.0;
}
