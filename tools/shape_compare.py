"""Time caqr_factor on several shapes with the round-1 fused path (CAQR_CHAIN=0)
and the chain kernel (CAQR_CHAIN=1, tcgen05), median of 5 (diagnostics)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
shapes = [(110592, 100), (8192, 256), (100000, 256), (1000000, 128), (1000000, 64), (1000000, 32), (4096, 192),
          (200000, 192), (1000000, 192)]
for m, n in shapes:
    A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
    A = caqr.colmajor_empty(m, n, torch.float32)
    res = []
    for ch in ("0", "1"):
        os.environ["CAQR_CHAIN"] = ch
        A.copy_(A0)
        R, ws = caqr.caqr_factor(A)
        ts = []
        for _ in range(5):
            A.copy_(A0)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); caqr.caqr_factor(A, R=R, ws=ws); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        res.append(sorted(ts)[2])
    fl = 2.0 * m * n * n - 2.0 * n ** 3 / 3
    print(f"{m:8d} x {n:3d}: fused {res[0]:7.3f} ms  chain {res[1]:7.3f} ms  ({fl / res[0] / 1e9:.1f} / {fl / res[1] / 1e9:.1f} TF/s)", flush=True)
