"""Robust PCA oracle -- TEST INFRASTRUCTURE ONLY (not part of the product).

Plain numpy float64 definitions of the paper's application:

* ``svt``     singular value thresholding, the step that "thresholds (sets to
              zero) the smallest singular values of L0" (Fig. 11),
              written as its definition U diag(max(sigma - tau, 0)) V^T with the
              SVD taken directly of X (numpy/LAPACK gesdd).  The GPU path reaches
              the same matrix through A = QR, SVD(R), (QU); the
              oracle deliberately does not.
* ``shrink``  the shrinkage operator "pushing the values of the matrix towards
              zero": sign(x) max(|x| - t, 0).
* ``ialm_*``  the alternating-directions method the paper cites ([19])
              in its inexact augmented-Lagrangian form (Lin, Chen, Ma): reading
              S19 of DESIGN.md fixes its parameters (lambda = 1/sqrt(max(m, n)),
              mu0 = 1.25 / ||M||_2, rho = 1.5, mu_max = 1e7 mu0,
              Y0 = M / max(||M||_2, ||M||_inf / lambda)).

Pins (tests/test_rpca_oracle.py, -m "not gpu"): closed forms of svt / shrink,
the 2 x 2 singular values, and exact recovery of a planted low-rank + sparse
matrix (the property robust PCA is built on), none of which re-types these
formulas.
"""
from __future__ import annotations

import numpy as np


def svt(X: np.ndarray, tau: float) -> np.ndarray:
    """U diag(max(sigma - tau, 0)) V^T of X."""
    U, s, Vt = np.linalg.svd(np.asarray(X, dtype=np.float64), full_matrices=False)
    d = np.maximum(s - tau, 0.0)
    return (U * d) @ Vt


def shrink(X: np.ndarray, t: float) -> np.ndarray:
    """sign(x) max(|x| - t, 0), elementwise."""
    X = np.asarray(X, dtype=np.float64)
    return np.sign(X) * np.maximum(np.abs(X) - t, 0.0)


def ialm_params(M: np.ndarray) -> dict:
    """Starting state of the alternating-directions iteration (reading S19)."""
    M = np.asarray(M, dtype=np.float64)
    m, n = M.shape
    lam = 1.0 / np.sqrt(max(m, n))
    norm2 = np.linalg.svd(M, compute_uv=False)[0]
    norminf = np.abs(M).max()
    J = max(norm2, norminf / lam)
    mu = 1.25 / norm2
    return dict(lam=lam, mu=mu, rho=1.5, mu_max=mu * 1e7, Y=M / J, S=np.zeros_like(M), L=np.zeros_like(M))


def ialm_step(M: np.ndarray, st: dict) -> dict:
    """One iteration (Fig. 11): L = svt(M - S + Y/mu, 1/mu); S = shrink(M - L + Y/mu,
    lam/mu); Y += mu (M - L - S); mu = min(rho mu, mu_max).  Returns the new state
    and the residual ||M - L - S||_F."""
    M = np.asarray(M, dtype=np.float64)
    mu, lam = st["mu"], st["lam"]
    L = svt(M - st["S"] + st["Y"] / mu, 1.0 / mu)
    S = shrink(M - L + st["Y"] / mu, lam / mu)
    Z = M - L - S
    Y = st["Y"] + mu * Z
    out = dict(st)
    out.update(L=L, S=S, Y=Y, mu=min(st["rho"] * mu, st["mu_max"]), resid=float(np.linalg.norm(Z)))
    return out


def ialm(M: np.ndarray, iters: int) -> dict:
    st = ialm_params(M)
    for _ in range(iters):
        st = ialm_step(M, st)
    return st
