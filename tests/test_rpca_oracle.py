"""Pins for the robust-PCA oracle (oracle/rpca.py), -m "not gpu".

Pinned against things other than the oracle's own formulas:
  * closed forms: the singular values of [[3, 0], [4, 5]] are sqrt(45) and sqrt(5)
    (eigenvalues of A^T A = [[25, 20], [20, 25]]: 45 and 5), so svt at tau = 1 is
    known entry by entry; a rank-one matrix s u v^T thresholds to (s - tau) u v^T;
    tau >= sigma_max gives 0; tau = 0 gives X back;
  * shrink at hand-computed points;
  * exact recovery of a planted low-rank + sparse matrix by the iteration
    (Candes, Li, Ma, Wright; the property robust PCA, is built on).
"""
import numpy as np

from oracle import rpca


def test_svt_closed_form_2x2():
    A = np.array([[3.0, 0.0], [4.0, 5.0]])
    s = np.linalg.svd(A, compute_uv=False)
    assert np.allclose(s, [np.sqrt(45.0), np.sqrt(5.0)], rtol=0, atol=1e-14)
    # A^T A = [[25, 20], [20, 25]]: right singular vectors (1,1)/sqrt2, (1,-1)/sqrt2
    v1, v2 = np.array([1.0, 1.0]) / np.sqrt(2), np.array([1.0, -1.0]) / np.sqrt(2)
    u1, u2 = A @ v1 / np.sqrt(45.0), A @ v2 / np.sqrt(5.0)
    want = (np.sqrt(45.0) - 1) * np.outer(u1, v1) + (np.sqrt(5.0) - 1) * np.outer(u2, v2)
    assert np.abs(rpca.svt(A, 1.0) - want).max() <= 1e-14
    # only the top singular value survives tau = 2.5 (sqrt 5 = 2.236 < 2.5)
    assert np.abs(rpca.svt(A, 2.5) - (np.sqrt(45.0) - 2.5) * np.outer(u1, v1)).max() <= 1e-14


def test_svt_rank_one_and_limits():
    rng = np.random.default_rng(0)
    u = rng.standard_normal(50)
    u /= np.linalg.norm(u)
    v = rng.standard_normal(7)
    v /= np.linalg.norm(v)
    X = 4.0 * np.outer(u, v)
    assert np.abs(rpca.svt(X, 1.5) - 2.5 * np.outer(u, v)).max() <= 1e-14
    assert np.abs(rpca.svt(X, 4.0)).max() <= 1e-14
    Y = rng.standard_normal((30, 6))
    assert np.abs(rpca.svt(Y, 0.0) - Y).max() <= 1e-13
    assert np.abs(rpca.svt(Y, 1e9)).max() == 0.0


def test_shrink_points():
    x = np.array([-3.0, -1.0, -0.5, 0.0, 0.25, 2.0])
    assert np.array_equal(rpca.shrink(x, 1.0), np.array([-2.0, 0.0, 0.0, 0.0, 0.0, 1.0]))
    assert np.array_equal(rpca.shrink(x, 0.0), x)


def test_planted_recovery():
    """M = L0 + S0, rank(L0) = 2, 5 % sparse S0: the iteration recovers both."""
    rng = np.random.default_rng(3)
    m, n, r = 300, 40, 2
    L0 = rng.standard_normal((m, r)) @ rng.standard_normal((r, n))
    S0 = np.zeros((m, n))
    mask = rng.random((m, n)) < 0.05
    S0[mask] = rng.uniform(-10, 10, mask.sum())
    M = L0 + S0
    st = rpca.ialm(M, 60)
    assert np.linalg.norm(st["L"] - L0) / np.linalg.norm(L0) <= 1e-5
    assert np.linalg.norm(st["S"] - S0) / np.linalg.norm(S0) <= 1e-5
    assert st["resid"] / np.linalg.norm(M) <= 1e-7
    assert np.linalg.matrix_rank(st["L"], tol=1e-6 * np.linalg.norm(st["L"], 2)) == r
