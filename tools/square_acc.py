"""Square CAQR: time + residual / orthogonality / R^T R for the tensor-core
(3xTF32) vs FFMA trailing update (CAQR_MMA), n = 2048 and 8192 (diagnostics)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
for n in (2048, 8192):
    A0 = workloads.device_gaussian(n, n, seed=7, dtype=torch.float32, device="cuda").t()
    for mma in ("1", "0"):
        os.environ["CAQR_MMA"] = mma
        A = caqr.colmajor_empty(n, n, torch.float32)
        A.copy_(A0)
        R, ws = caqr.caqr_factor(A)
        ts = []
        for _ in range(3):
            A.copy_(A0)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); caqr.caqr_factor(A, R=R, ws=ws); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        Q = caqr.caqr_form_q(A, ws)
        torch.cuda.synchronize()
        A64, R64, Q64 = A0.double(), R.double(), Q.double()
        G = A64.t() @ A64
        print(f"n={n} CAQR_MMA={mma}: {sorted(ts)[1]:8.2f} ms  RtR {(torch.linalg.norm(R64.t() @ R64 - G) / torch.linalg.norm(G)).item():.2e}"
              f"  res {(torch.linalg.norm(A64 - Q64 @ R64) / torch.linalg.norm(A64)).item():.2e}"
              f"  orth {torch.linalg.norm(Q64.t() @ Q64 - torch.eye(n, dtype=torch.float64, device='cuda')).item():.2e}", flush=True)
        del A64, R64, Q64, G, Q
