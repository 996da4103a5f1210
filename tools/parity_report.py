"""Achieved parity errors of the CUDA path against the oracle on the BASELINE
configs (writes profiles/parity_r02.json).  Diagnostics / evidence; the pass /
fail gates are tests/test_gpu_parity.py.  Uses the oracle (test infrastructure)
and the golden R's of tools/make_golden.py.

    python tools/parity_report.py
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads  # noqa: E402

out = {"when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime()), "gpu": torch.cuda.get_device_name(0),
       "note": "errors of the default plan; R sign-normalised (reading S17); fp32 bounds 1e-5/1e-5/1e-4"}


def dev(A):
    t = caqr.colmajor_empty(A.shape[0], A.shape[1], torch.float32 if A.dtype == np.float32 else torch.float64)
    t.copy_(torch.from_numpy(np.ascontiguousarray(A)))
    return t


def host_case(name, A, Ro=None, acc="d", want_q=True):
    t0 = time.time()
    m, n = A.shape
    Ad = dev(A)
    R, ws = caqr.caqr_factor(Ad)
    Q = caqr.caqr_form_q(Ad, ws) if want_q else None
    torch.cuda.synchronize()
    R = R.cpu().double().numpy()
    A64 = A.astype(np.float64)
    if Ro is None:
        Ro = oracle.normalize_signs(oracle.qr(A64, want_q=False, acc=acc))
    rec = {"shape": [m, n], "dtype": str(A.dtype),
           "r_vs_oracle": float(np.linalg.norm(oracle.normalize_signs(R) - Ro) / np.linalg.norm(Ro))}
    if want_q:
        Q = Q.cpu().double().numpy()
        rec["residual"] = float(np.linalg.norm(A64 - Q @ R) / np.linalg.norm(A64))
        rec["orthogonality"] = float(np.linalg.norm(Q.T @ Q - np.eye(n)))
    rec["seconds"] = round(time.time() - t0, 1)
    out[name] = rec
    print(name, rec, flush=True)


host_case("C1_4096x16", workloads.gaussian(4096, 16, seed=0))
host_case("C2_krylov_4Mx8_shifted", workloads.krylov_basis(grid=2000, s=8, seed=0, shifted=True), want_q=False)
host_case("C3_video_110592x100", workloads.video(seed=0))
for name, dt in [("r_1000000x192_f32_seed0", np.float32), ("r_200000x192_f64_seed1", np.float64)]:
    g = np.load(os.path.join(ROOT, "tests", "golden", name + ".npz"))
    A = workloads.gaussian(int(g["m"]), int(g["n"]), seed=int(g["seed"]), dtype=dt)
    host_case("C4_" + name, A, Ro=g["R"], want_q=(dt == np.float32))
A = workloads.gaussian(2048, 2048, seed=3)
host_case("square_2048", A)
_, Qf = oracle.qr(A.astype(np.float64), want_q=True, acc="f")
out["square_2048"]["oracle_fp32_orthogonality"] = float(np.linalg.norm(Qf.T @ Qf - np.eye(2048)))
# C5 8192^2 (device-side fp64 checks)
n = 8192
A = workloads.device_gaussian(n, n, seed=7, dtype=torch.float32, device="cuda").t()
A0 = A.clone()
R, ws = caqr.caqr_factor(A)
Q = caqr.caqr_form_q(A, ws)
torch.cuda.synchronize()
A64, R64, Q64 = A0.double(), R.double(), Q.double()
G = A64.t() @ A64
out["C5_8192sq"] = {
    "RtR_vs_AtA": (torch.linalg.norm(R64.t() @ R64 - G) / torch.linalg.norm(G)).item(),
    "residual": (torch.linalg.norm(A64 - Q64 @ R64) / torch.linalg.norm(A64)).item(),
    "orthogonality": torch.linalg.norm(Q64.t() @ Q64 - torch.eye(n, dtype=torch.float64, device="cuda")).item()}
print("C5", out["C5_8192sq"], flush=True)
with open(os.path.join(ROOT, "profiles", "parity_r02.json"), "w") as f:
    json.dump(out, f, indent=1)
