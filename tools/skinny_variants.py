"""Time the streaming skinny TSQR (n <= 8) with 8 warps x two tile buffers
(CAQR_STREAM_W16B=0) against 16 warps x one buffer (default), with an R
check against the Cholesky factor of the fp64 Gram matrix.

    python tools/skinny_variants.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads

for m, n in [(4_000_000, 8), (1_000_000, 8), (200_000, 8), (4_000_000, 4), (65536, 8), (4096, 8), (4_000_000, 1)]:
    A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
    A = caqr.colmajor_empty(m, n)
    A64 = A0.double()
    Lc = torch.linalg.cholesky(A64.t() @ A64).t()
    line = f"{m}x{n}:"
    for w in ("0", "1"):
        os.environ["CAQR_STREAM_W16B"] = w
        A.copy_(A0)
        R, ws = caqr.caqr_factor(A)
        ts = []
        for _ in range(20):
            A.copy_(A0)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            caqr.caqr_factor(A, R=R, ws=ws)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        d = torch.sign(torch.diagonal(R.double()))
        err = ((R.double() * d[:, None]) - Lc).norm() / Lc.norm()
        t = sorted(ts)[len(ts) // 2] * 1e3
        line += f"  w16b={w}: {t:7.1f} us ({2 * m * n * 4 / t / 1e3:6.0f} GB/s) err={err:.1e}"
        # apply / form_q still consistent
        C = caqr.colmajor(A0.clone())
        caqr.caqr_apply_qt(A, ws, C)
        Q = caqr.caqr_form_q(A, ws)
        e2 = (C[:n].double() - R.double()).norm() / R.double().norm()
        e3 = (Q.double() @ R.double() - A64).norm() / A64.norm()
        line += f" qtA={e2:.1e} QR={e3:.1e}"
    print(line, f"plan={caqr.caqr_plan_info(m, n)}", flush=True)
