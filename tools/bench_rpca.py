"""Robust PCA iterations/s (the paper's Table II metric) on the
synthetic 110,592 x 100 video (config C3 shape), fp32, one B200: every step of
the iteration on the GPU (CAQR + one-CTA SVD of R + Q[W;0] + fused update).
Prints one JSON line; with --trace also the per-kernel time split."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
from paper_conf_ipps_andersonbdk11_b200.rpca import RobustPCA

ap = argparse.ArgumentParser()
ap.add_argument("--iters", type=int, default=50)
ap.add_argument("--warmup", type=int, default=5)
ap.add_argument("--trace", action="store_true")
a = ap.parse_args()
M = workloads.video(seed=0).astype(np.float32)
m, n = M.shape
Md = caqr.colmajor_empty(m, n)
Md.copy_(torch.from_numpy(M))
rp = RobustPCA(Md)
for _ in range(a.warmup):
    rp.step()
torch.cuda.synchronize()
if a.trace:
    caqr.caqr_trace_begin()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(a.iters):
    rp.step()
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / a.iters
out = {"metric": "Robust PCA iterations/s (110592 x 100 synthetic video, fp32)", "value": 1000.0 / ms,
       "unit": "it/s", "ms_per_iter": ms, "iters": a.iters, "warmup": a.warmup,
       "residual_rel": rp.residual() / float(np.linalg.norm(M)),
       "paper": "27.0 it/s CAQR on GTX480 (Table II, P:L1141-1145) -- other hardware, context only"}
if a.trace:
    tr = caqr.caqr_trace_end()
    agg = {}
    for k, t, _, _ in tr:
        agg[k] = agg.get(k, 0.0) + t
    out["kernel_ms_per_iter"] = {k: v / a.iters for k, v in sorted(agg.items(), key=lambda kv: -kv[1])}
print(json.dumps(out))
