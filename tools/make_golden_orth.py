"""tests/golden/oracle_f_orth.json: ||Q^T Q - I||_F of the oracle's fp32
Householder QR (acc="f": float accumulation) on the square C5 input family,
the calibration of the fp32 orthogonality bound for n > 192 (SURVEY 9.1,
DESIGN.md section 6).  Calls only oracle/ and workloads.gaussian.  Slow
(8192^2: minutes on one core).  TEST INFRASTRUCTURE."""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from paper_conf_ipps_andersonbdk11_b200 import workloads  # noqa: E402

out = {"oracle": "oracle.qr(acc='f'), ||Q^T Q - I||_F", "generator": "workloads.gaussian(n, n, seed=7) fp32"}
for n in (2048, 4096, 8192):
    t0 = time.time()
    A = workloads.gaussian(n, n, seed=7).astype(np.float64)
    _, Q = oracle.qr(A, want_q=True, acc="f")
    G = Q.T @ Q
    G[np.diag_indices(n)] -= 1.0
    out[str(n)] = float(np.linalg.norm(G))
    print(n, out[str(n)], f"{time.time() - t0:.0f} s", flush=True)
    with open(os.path.join(ROOT, "tests", "golden", "oracle_f_orth.json"), "w") as f:
        json.dump(out, f, indent=1)
