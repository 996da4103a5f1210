"""C3 (110,592 x 100 video matrix) plan sweep: chains (CAQR_CHAIN_TARGET) x tile
height; plus the n in (224, 256] shapes (diagnostics)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads


def t_factor(A0, opts=None):
    m, n = A0.shape
    A = caqr.colmajor_empty(m, n, A0.dtype)
    A.copy_(A0)
    R, ws = caqr.caqr_factor(A, opts=opts)
    ts = []
    for _ in range(7):
        A.copy_(A0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); caqr.caqr_factor(A, R=R, ws=ws, opts=opts); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return sorted(ts)[3]


V = workloads.video(seed=0)
A0 = caqr.colmajor_empty(*V.shape, torch.float32)
A0.copy_(torch.from_numpy(np.ascontiguousarray(V)))
for ct in ("", "74", "124", "148", "200", "247", "296", "400"):
    if ct:
        os.environ["CAQR_CHAIN_TARGET"] = ct
    else:
        os.environ.pop("CAQR_CHAIN_TARGET", None)
    row = []
    for b in (128, 160, 192, 224, 256):
        try:
            row.append(f"b={b}: {t_factor(A0, caqr.make_opts(leaf_rows=b)):.3f}")
        except Exception as e:  # noqa: BLE001
            row.append(f"b={b}: err")
    print(f"chain_target={ct or 'default'}: " + "  ".join(row), flush=True)
os.environ.pop("CAQR_CHAIN_TARGET", None)
for m, n in [(8192, 256), (100000, 256), (8192, 240), (1000000, 256)]:
    A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
    print(f"{m}x{n}: {t_factor(A0):.3f} ms  plan={caqr.caqr_plan_info(m, n)}", flush=True)
