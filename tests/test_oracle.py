"""Pins for the CPU oracle (oracle/), run with -m "not gpu".

The oracle is pinned to things other than itself:
  * hand-derived closed forms (tests/golden/closed_forms.json)
  * LAPACK dgeqrf/dormqr through scipy (an independent implementation of the
    same xLARFG convention): same V, tau, R, and same Q^T C
  * Cholesky of A^T A (R^T R = A^T A, a different algorithm)
  * classical Gram-Schmidt at 50 digits (mpmath) on tiny inputs
  * invariants: orthogonality, reconstruction, column norms, row permutation,
    zero-row padding (exact), power-of-2 column scaling (bitwise)
"""
import json
import math
import os

import numpy as np
import pytest
import scipy.linalg.lapack as lapack

import oracle
from oracle.cgs import cgs_qr
from paper_conf_ipps_andersonbdk11_b200 import workloads

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "closed_forms.json")


def _ev(x):
    if isinstance(x, str):
        return float(eval(x, {"__builtins__": {}}, {"sqrt": math.sqrt}))
    return float(x)


def _arr(rows):
    return np.array([[_ev(v) for v in r] for r in rows], dtype=np.float64)


def _cases():
    with open(GOLDEN) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("acc", ["d", "ld"])
@pytest.mark.parametrize("case", _cases(), ids=lambda c: c["name"])
def test_closed_forms(case, acc):
    A = _arr(case["A"])
    VR, tau = oracle.geqr2(A, acc=acc)
    n = A.shape[1]
    R = np.triu(VR[:n, :])
    np.testing.assert_allclose(R, _arr(case["R"]), rtol=0, atol=1e-15)
    np.testing.assert_allclose(tau, [_ev(t) for t in case["tau"]], rtol=0, atol=1e-15)
    Rq, Q = oracle.qr(A, acc=acc)
    np.testing.assert_allclose(oracle.normalize_signs(Rq), _arr(case["R_normalized"]), rtol=0, atol=1e-15)
    # Q is orthonormal and reproduces A
    np.testing.assert_allclose(Q.T @ Q, np.eye(n), atol=1e-15)
    np.testing.assert_allclose(Q @ Rq, A, atol=1e-14)


def test_closed_forms_fp32_mode():
    for case in _cases():
        A = _arr(case["A"])
        R = oracle.qr(A, want_q=False, acc="f")
        np.testing.assert_allclose(oracle.normalize_signs(R), _arr(case["R_normalized"]), atol=2e-6)


def test_identity_exact():
    for n in (1, 5, 16):
        A = np.eye(n)
        R, Q = oracle.qr(A)
        assert np.array_equal(R, np.eye(n))
        assert np.array_equal(Q, np.eye(n))
        _, tau = oracle.geqr2(np.vstack([np.eye(n), np.zeros((3, n))]))
        assert np.all(tau == 0)


@pytest.mark.parametrize("shape", [(7, 3), (50, 5), (200, 16), (64, 64), (333, 31)])
def test_matches_lapack_representation(shape):
    """Same reflectors, taus and R as LAPACK dgeqrf (xLARFG convention)."""
    m, n = shape
    A = np.random.default_rng(m * 1000 + n).standard_normal(shape)
    VR, tau = oracle.geqr2(A, acc="d")
    qr_l, tau_l, _, info = lapack.dgeqrf(np.asfortranarray(A))
    assert info == 0
    scale = np.abs(qr_l).max()
    np.testing.assert_allclose(VR, qr_l, rtol=0, atol=1e-12 * scale * n)
    np.testing.assert_allclose(tau, tau_l, rtol=0, atol=1e-12)
    # Q^T C and Q C agree with LAPACK dormqr applied to the same reflectors
    C = np.random.default_rng(7).standard_normal((m, 4))
    for trans, ltrans in ((True, "T"), (False, "N")):
        ours = oracle.orm2r(VR, tau, C, trans=trans)
        cq, _, info = lapack.dormqr("L", ltrans, qr_l, tau_l, np.asfortranarray(C), max(1, 4 * 64))
        assert info == 0
        np.testing.assert_allclose(ours, cq, atol=1e-12 * n)


@pytest.mark.parametrize("acc", ["d", "ld"])
def test_cholesky_of_gram(acc):
    """Normalised R = chol(A^T A)^T  (R^T R = A^T A with positive diagonal)."""
    A = np.random.default_rng(3).standard_normal((50, 5))
    R = oracle.normalize_signs(oracle.qr(A, want_q=False, acc=acc))
    L = np.linalg.cholesky(A.T @ A)
    np.testing.assert_allclose(R, L.T, rtol=0, atol=1e-13 * np.abs(L).max())


@pytest.mark.parametrize("seed", range(8))
def test_mpmath_cgs_tiny(seed):
    """Brute force: classical Gram-Schmidt at 50 digits on tiny inputs."""
    rng = np.random.default_rng(100 + seed)
    m = int(rng.integers(2, 13))
    n = int(rng.integers(1, min(m, 6) + 1))
    A = rng.standard_normal((m, n))
    R_ref, Q_ref = cgs_qr(A)
    for acc, tol in (("d", 1e-14), ("ld", 1e-15)):
        R, Q = oracle.qr(A, acc=acc)
        Rn, Qn = oracle.normalize_signs(R, Q)
        assert np.linalg.norm(Rn - R_ref) / np.linalg.norm(R_ref) <= tol
        assert np.linalg.norm(Qn - Q_ref) <= 10 * tol


def test_mpmath_cgs_hilbert_block():
    """Ill-conditioned tiny case (10 x 6 Hilbert block, kappa ~ 2.5e6)."""
    A = np.array([[1.0 / (i + j + 1) for j in range(6)] for i in range(10)])
    R_ref, _ = cgs_qr(A, dps=60)
    R = oracle.normalize_signs(oracle.qr(A, want_q=False, acc="ld"))
    assert np.linalg.norm(R - R_ref) / np.linalg.norm(R_ref) <= 1e-14


@pytest.mark.parametrize("acc", ["d", "ld"])
def test_invariants(acc):
    rng = np.random.default_rng(11)
    A = rng.standard_normal((300, 12))
    R, Q = oracle.qr(A, acc=acc)
    n = A.shape[1]
    # Q orthonormal, A = QR
    assert np.linalg.norm(Q.T @ Q - np.eye(n)) <= 1e-14
    assert np.linalg.norm(A - Q @ R) / np.linalg.norm(A) <= 1e-15 * 10
    # column norms ||R e_j|| = ||A e_j||
    np.testing.assert_allclose(np.linalg.norm(R, axis=0), np.linalg.norm(A, axis=0), rtol=1e-14)
    Rn = oracle.normalize_signs(R)
    # row permutation invariance R(PA) = R(A)
    Rp = oracle.normalize_signs(oracle.qr(A[rng.permutation(A.shape[0])], want_q=False, acc=acc))
    assert np.linalg.norm(Rp - Rn) / np.linalg.norm(Rn) <= 1e-14
    # zero-row padding R([A; 0]) = R(A), exactly
    Rz = oracle.qr(np.vstack([A, np.zeros((17, n))]), want_q=False, acc=acc)
    assert np.array_equal(Rz, R)
    # power-of-2 column scaling: R(A diag(2^e)) = R(A) diag(2^e), bitwise
    e = rng.integers(-20, 20, size=n)
    s = np.ldexp(1.0, e)
    Rs = oracle.qr(A * s[None, :], want_q=False, acc=acc)
    assert np.array_equal(Rs, R * s[None, :])


def test_apply_qt_gives_r():
    """Q^T A = [R; 0] and ||Q^T C|| = ||C||."""
    rng = np.random.default_rng(5)
    A = rng.standard_normal((120, 9))
    VR, tau = oracle.geqr2(A)
    QtA = oracle.orm2r(VR, tau, A, trans=True)
    np.testing.assert_allclose(QtA[:9], np.triu(VR[:9]), atol=1e-13)
    assert np.abs(QtA[9:]).max() <= 1e-13
    C = rng.standard_normal((120, 5))
    QtC = oracle.orm2r(VR, tau, C, trans=True)
    np.testing.assert_allclose(np.linalg.norm(QtC, axis=0), np.linalg.norm(C, axis=0), rtol=1e-14)
    # round trip Q (Q^T C) = C
    np.testing.assert_allclose(oracle.orm2r(VR, tau, QtC, trans=False), C, atol=1e-13)


def test_fp32_calibration_level():
    """A plain fp32 Householder (acc='f') sits ~1e-7 from the double oracle on
    a 4096 x 16 Gaussian: the scale the fp32 BASELINE bounds are set against."""
    A = workloads.gaussian(4096, 16, seed=0).astype(np.float64)
    Rd = oracle.normalize_signs(oracle.qr(A, want_q=False, acc="d"))
    Rf = oracle.normalize_signs(oracle.qr(A, want_q=False, acc="f"))
    rel = np.linalg.norm(Rf - Rd) / np.linalg.norm(Rd)
    assert 1e-9 < rel < 1e-5


def test_flop_count():
    # 2 m n^2 - 2 n^3 / 3 (BASELINE metric); 1M x 192 -> 73.72 GFLOP
    assert abs(oracle.geqrf_flops(1_000_000, 192) - 73.7233e9) / 73.72e9 < 1e-4
    # brute-force count of the unblocked algorithm's multiply-adds (4 flops per
    # trailing-column element per reflector) approaches the LAPACK count
    m, n = 4000, 40
    brute = sum(4 * (m - j) * (n - j - 1) + 3 * (m - j) for j in range(n))
    assert abs(brute / oracle.geqrf_flops(m, n) - 1) < 0.05


def test_workloads_deterministic():
    a = workloads.gaussian(100, 7, seed=3)
    b = workloads.gaussian(100, 7, seed=3)
    assert a.dtype == np.float32 and a.flags.f_contiguous and np.array_equal(a, b)
    k = workloads.krylov_basis(grid=40, s=6, seed=1, dtype=np.float64)
    np.testing.assert_allclose(np.linalg.norm(k, axis=0), 1.0, rtol=1e-12)
    ks = workloads.krylov_basis(grid=40, s=6, seed=1, shifted=True, dtype=np.float64)
    assert np.linalg.cond(ks) < np.linalg.cond(k)
    v = workloads.video(frames=5, h=24, w=32, seed=0)
    assert v.shape == (24 * 32, 5) and v.min() >= 0 and v.max() <= 1
