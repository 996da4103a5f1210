"""Write tests/golden/*.npz: the CPU oracle's sign-normalised R factors at the
full BASELINE sizes, for element-by-element GPU parity (tests/test_gpu_parity.py
test_full_size_r_vs_oracle_golden).  Calls only oracle/ and the seeded input
generator workloads.gaussian (numpy PCG64; the GPU test regenerates the same
input bit for bit).  TEST INFRASTRUCTURE: never imported by the product.

    python tools/make_golden.py            # ~1-2 minutes on one core
"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from paper_conf_ipps_andersonbdk11_b200 import workloads  # noqa: E402

CASES = [
    # (name, m, n, seed, input dtype, oracle accumulation)
    ("r_1000000x192_f32_seed0", 1_000_000, 192, 0, np.float32, "d"),   # config C4 (fp32)
    ("r_200000x192_f64_seed1", 200_000, 192, 1, np.float64, "ld"),     # config C4 fp64 variant, 200k rows
]

for name, m, n, seed, dt, acc in CASES:
    t0 = time.time()
    A = workloads.gaussian(m, n, seed=seed, dtype=dt)
    R = oracle.normalize_signs(oracle.qr(A.astype(np.float64), want_q=False, acc=acc))
    path = os.path.join(ROOT, "tests", "golden", name + ".npz")
    np.savez_compressed(path, R=R, m=m, n=n, seed=seed, dtype=np.dtype(dt).name, acc=acc,
                        generator="workloads.gaussian (numpy default_rng PCG64, float64 rounded to dtype)",
                        oracle="oracle.qr (householder.c xGEQR2, accumulation %s), sign-normalised" % acc)
    print(f"{name}: {time.time() - t0:.1f} s -> {path} ({os.path.getsize(path)} B)", flush=True)
