"""Time caqr_factor on every BASELINE config shape (device-generated inputs)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads

cfgs = [("c1_4096x16", 4096, 16, torch.float32, 0), ("c2_4Mx8", 4_000_000, 8, torch.float32, 0),
        ("c3_110592x100", 110_592, 100, torch.float32, 0), ("c4_1Mx192_f32", 1_000_000, 192, torch.float32, 0),
        ("c4_1Mx192_f64", 1_000_000, 192, torch.float64, 0), ("c5_8192sq", 8192, 8192, torch.float32, 64)]
only = sys.argv[1:] or None
for name, m, n, dt, nb in cfgs:
    if only and name not in only:
        continue
    A0 = workloads.device_gaussian(m, n, seed=0, dtype=dt, device="cuda").t()
    A = caqr.colmajor_empty(m, n, dt)
    opts = caqr.make_opts(0, nb)
    reps = 3 if m * n > 1e8 else 10
    ts = []
    for r in range(reps + 1):
        A.copy_(A0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        R, ws = caqr.caqr_factor(A, opts=opts)
        e1.record()
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    ms = sorted(ts)[len(ts) // 2]
    fl = 2.0 * m * n * n - 2.0 * n ** 3 / 3
    print(f"{name:16s} {ms:9.3f} ms  {fl / ms / 1e9:8.1f} TFLOP/s  plan={caqr.caqr_plan_info(m, n, 0 if dt == torch.float32 else 1, opts)}")
    del A0, A, ws
    torch.cuda.empty_cache()
