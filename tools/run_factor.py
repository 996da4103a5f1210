"""Profiling driver: run caqr_factor on an m x n Gaussian a few times (for ncu)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=1_000_000)
ap.add_argument("--n", type=int, default=192)
ap.add_argument("--dtype", default="f32")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--leaf-rows", type=int, default=0)
ap.add_argument("--apply", action="store_true")
a = ap.parse_args()
dt = torch.float32 if a.dtype == "f32" else torch.float64
A0 = workloads.device_gaussian(a.m, a.n, seed=0, dtype=dt, device="cuda").t()
A = caqr.colmajor_empty(a.m, a.n, dt)
opts = caqr.make_opts(a.leaf_rows)
for _ in range(a.reps):
    A.copy_(A0)
    R, ws = caqr.caqr_factor(A, opts=opts)
    if a.apply:
        Q = caqr.caqr_form_q(A, ws, opts=opts)
torch.cuda.synchronize()
print("done")
if os.environ.get("CAQR_PROFILE") == "1":
    import ctypes
    L = caqr.lib()
    out = (ctypes.c_ulonglong * 16)()
    L.caqr_debug_profile_read.argtypes = [ctypes.c_void_p]
    L.caqr_debug_profile_read(out)
    names = {0: "fetch", 1: "wait", 2: "stage_panel", 3: "factor", 4: "G=V^T V", 12: "build_t",
             5: "fence/publish", 6: "stage_C", 7: "VtC", 8: "apply", 9: "publish"}
    tot = sum(out[i] for i in names)
    for i, nm in names.items():
        print(f"{nm:14s} {out[i] / tot * 100:5.1f}%  {out[i] / 1.965e9 / max(1, a.reps):.4f} CTA-s")
    print("leaf panel-steps", out[10], "merge panel-steps", out[11], "total CTA-s", tot / 1.965e9 / a.reps)
    t0 = (2**64 - 1) - out[15]
    print(f"timeline (last rep): chains done by {(out[13] - t0) / 1e3:.1f} us (last chain end), "
          f"kernel end {(out[14] - t0) / 1e3:.1f} us")
