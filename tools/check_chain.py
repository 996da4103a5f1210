"""Quick GPU check of the chain-kernel path against the round-1 fused path and
an fp64 reference (diagnostics; the real parity tests are tests/test_gpu_*).

    python tools/check_chain.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads


def signfix(R):
    d = torch.sign(torch.diagonal(R))
    d[d == 0] = 1
    return R * d[:, None]


def run(m, n, seed=0):
    A0 = workloads.device_gaussian(m, n, seed=seed, dtype=torch.float32, device="cuda").t()
    out = {}
    for ch in ("1", "0"):
        os.environ["CAQR_CHAIN"] = ch
        A = caqr.colmajor_empty(m, n, torch.float32)
        A.copy_(A0)
        R, ws = caqr.caqr_factor(A)
        C = caqr.colmajor(A0.clone())
        caqr.caqr_apply_qt(A, ws, C)
        Q = caqr.caqr_form_q(A, ws)
        torch.cuda.synchronize()
        out[ch] = (R.double(), C.double(), Q.double())
    A64 = A0.double()
    G = A64.t() @ A64
    Rc, Cc, Qc = out["1"]
    Rr = out["0"][0]
    Lc = torch.linalg.cholesky(G).t()
    err_chol = (signfix(Rc) - Lc).norm() / Lc.norm()
    err_r = (signfix(Rc) - signfix(Rr)).norm() / Rr.norm()
    err_top = (Cc[:n] - Rc).norm() / Rc.norm()
    err_bot = Cc[n:].norm() / A64.norm()
    err_orth = (Qc.t() @ Qc - torch.eye(n, dtype=torch.float64, device="cuda")).norm()
    err_res = (A64 - Qc @ Rc).norm() / A64.norm()
    tril = torch.tril(Rc, -1).abs().max().item()
    print(f"{m}x{n}: plan={caqr.caqr_plan_info(m, n)}\n   |R-chol|/|R|={err_chol:.2e} |R-R_round1|={err_r:.2e} "
          f"|QtA top - R|={err_top:.2e} |QtA bottom|={err_bot:.2e} |QtQ-I|={err_orth:.2e} |A-QR|={err_res:.2e} "
          f"tril={tril}", flush=True)


os.environ["CAQR_CHAIN"] = "1"
for m, n in [(4096, 32), (5000, 40), (20000, 100), (20000, 130), (777, 100), (50000, 192), (12345, 192),
             (100000, 200), (30000, 256), (1000, 192), (193, 192), (1_000_000, 192)]:
    run(m, n)
