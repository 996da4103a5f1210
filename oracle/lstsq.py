"""Least-squares oracle -- TEST INFRASTRUCTURE ONLY (not part of the product).

min ||A x - b||_2 for a tall A (m >= n, full column rank) the way the paper's
QR serves it ("... least squares problems", LAPACK
xGELS semantics): x = R^{-1} (Q^T b)[0:n] with Q, R from the oracle's own
Householder QR (householder.py: xGEQR2 + xORM2R in double / long double) and a
plain back substitution written out below.  Rows n..m-1 of Q^T b are the
residual's components: ||(Q^T b)[n:m]|| = min ||A x - b||.

Pins (tests/test_lstsq_oracle.py, -m "not gpu"): numpy's lstsq (LAPACK gelsd, an
SVD-based independent implementation), the exact solution of a consistent system
b = A x0, the normal equations A^T (A x - b) = 0, and a 3 x 2 closed form.
"""
from __future__ import annotations

import numpy as np

from .householder import geqr2, orm2r


def back_substitute(R: np.ndarray, B: np.ndarray) -> np.ndarray:
    """X = R^{-1} B for upper-triangular R (n x n), B (n x k): x_i = (b_i - sum_{j>i} R_ij x_j) / R_ii."""
    R = np.asarray(R, dtype=np.float64)
    X = np.array(B, dtype=np.float64, copy=True).reshape(R.shape[0], -1)
    n = R.shape[0]
    for i in range(n - 1, -1, -1):
        X[i] = (X[i] - R[i, i + 1:] @ X[i + 1:]) / R[i, i]
    return X


def lstsq(A: np.ndarray, B: np.ndarray, acc: str = "d"):
    """(X, residual norms): X = argmin ||A X - B||_F column by column."""
    A = np.asarray(A, dtype=np.float64)
    B2 = np.asarray(B, dtype=np.float64).reshape(A.shape[0], -1)
    n = A.shape[1]
    VR, tau = geqr2(A, acc=acc)
    QtB = orm2r(VR, tau, B2, trans=True, acc=acc)
    X = back_substitute(np.triu(VR[:n, :n]), QtB[:n])
    return X, np.linalg.norm(QtB[n:], axis=0)
