"""Classical Gram-Schmidt in extended precision -- TEST INFRASTRUCTURE ONLY.

The independent brute-force pin for tiny inputs named by BASELINE.json's
north_star ("brute-force classical Gram-Schmidt in extended precision on tiny
inputs").  Gram-Schmidt is one of the QR algorithms the paper lists
(Sec. II); it is numerically weaker than Householder in working
precision, which is why it runs here at 50 significant digits (mpmath), where
the weakness is irrelevant for the small, well-conditioned inputs it is used on.

    r_ij = q_i^T a_j  (i < j),   w = a_j - sum_i r_ij q_i,   r_jj = ||w||,  q_j = w / r_jj

It returns R with a nonnegative diagonal, i.e. the normalised R of
SURVEY 8(c) step 5, and the thin Q.  Pure Python loops: only for m <= ~32.
"""
from __future__ import annotations

import mpmath
import numpy as np


def cgs_qr(A, dps: int = 50):
    """Return (R, Q) as float64 arrays, computed in `dps`-digit arithmetic."""
    A = np.asarray(A, dtype=np.float64)
    m, n = A.shape
    with mpmath.workdps(dps):
        a = [[mpmath.mpf(float(A[i, j])) for i in range(m)] for j in range(n)]
        q = []
        R = [[mpmath.mpf(0)] * n for _ in range(n)]
        for j in range(n):
            w = list(a[j])
            for i in range(j):
                rij = mpmath.fsum(q[i][k] * a[j][k] for k in range(m))
                R[i][j] = rij
                w = [w[k] - rij * q[i][k] for k in range(m)]
            rjj = mpmath.sqrt(mpmath.fsum(x * x for x in w))
            R[j][j] = rjj
            if rjj == 0:
                raise ValueError("cgs_qr: rank-deficient input")
            q.append([x / rjj for x in w])
        Rf = np.array([[float(R[i][j]) for j in range(n)] for i in range(n)])
        Qf = np.array([[float(q[j][i]) for j in range(n)] for i in range(m)])
    return Rf, Qf
