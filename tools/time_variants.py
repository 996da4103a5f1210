"""Time caqr_factor at 1M x 192 fp32 for several plan options (panel group width
nb, tile height b), with the per-kernel split from the launch trace.

    python tools/time_variants.py [m] [n]
"""
import collections
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads

m = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
n = int(sys.argv[2]) if len(sys.argv) > 2 else 192
variants = [("1", 0, 0), ("0", 0, 0)] + ([("1", 0, 64), ("1", 0, 96)] if os.environ.get("VAR_ALL") else [])
A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
A = caqr.colmajor_empty(m, n, torch.float32)
fl = 2.0 * m * n * n - 2.0 * n ** 3 / 3
for ch, b, nb in variants:
    os.environ["CAQR_CHAIN"] = ch
    opts = caqr.make_opts(b, nb)
    try:
        A.copy_(A0)
        R, ws = caqr.caqr_factor(A, opts=opts)
    except Exception as e:  # noqa: BLE001
        print(f"b={b} nb={nb}: {e}")
        continue
    ts = []
    for _ in range(5):
        A.copy_(A0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        caqr.caqr_factor(A, R=R, ws=ws, opts=opts)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    t = sorted(ts)[len(ts) // 2]
    A.copy_(A0)
    caqr.caqr_trace_begin(1 << 17)
    caqr.caqr_factor(A, R=R, ws=ws, opts=opts)
    torch.cuda.synchronize()
    tr = caqr.caqr_trace_end(1 << 17)
    agg = collections.defaultdict(lambda: [0, 0.0])
    for name, kms, _, _ in tr:
        agg[name][0] += 1
        agg[name][1] += kms
    split = "  ".join(f"{k}: {v[0]}x {v[1]:.3f}ms" for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1]))
    print(f"chain={ch} b={b:3d} nb={nb:3d}  {t:7.3f} ms  {fl / t / 1e9:6.2f} TF/s  plan={caqr.caqr_plan_info(m, n, opts=opts)}")
    print("     ", split)
