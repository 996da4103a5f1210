"""Width sweep for tall matrices (plan-cliff check): caqr_factor
GFLOP/s at m = 1,000,000 and 100,000 over n = 8 ... 512, plan printed beside."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads


def t_factor(m, n, reps=3):
    A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
    A = caqr.colmajor_empty(m, n)
    ts = []
    for r in range(reps + 1):
        A.copy_(A0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        caqr.caqr_factor(A)
        e1.record()
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    ms = sorted(ts)[len(ts) // 2]
    del A0, A
    torch.cuda.empty_cache()
    return ms, (2.0 * m * n * n - 2.0 * n ** 3 / 3) / ms / 1e9


for m in (1_000_000, 100_000):
    for n in (8, 16, 17, 24, 32, 48, 64, 96, 128, 160, 192, 200, 224, 232, 256, 288, 320, 384, 512):
        ms, tf = t_factor(m, n)
        p = caqr.caqr_plan_info(m, n)
        print(f"{m:8d} x {n:4d}: {ms:8.3f} ms {tf:6.2f} TF/s  b={p['leaf_rows']} nb={p['panel_cols']} "
              f"groups={p['groups']} chains={p['chains']}", flush=True)
