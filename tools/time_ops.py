"""Time factor / apply_qt (k columns) / form_q on one shape."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
m, n, k = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
dt = torch.float64 if os.environ.get("DT") == "f64" else torch.float32
A0 = workloads.device_gaussian(m, n, seed=0, dtype=dt, device="cuda").t()
A = caqr.colmajor_empty(m, n, dt); A.copy_(A0)
R, ws = caqr.caqr_factor(A)
C0 = workloads.device_gaussian(m, k, seed=1, dtype=dt, device="cuda").t()
C = caqr.colmajor_empty(m, k, dt)
def t(f, reps=3):
    ts = []
    for _ in range(reps + 1):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); f(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    return sorted(ts[1:])[len(ts[1:]) // 2]
def fac():
    A.copy_(A0); caqr.caqr_factor(A, R=R, ws=ws)
def app():
    C.copy_(C0); caqr.caqr_apply_qt(A, ws, C)
Q = caqr.colmajor_empty(m, n, dt)
def fq():
    caqr.caqr_form_q(A, ws, Q=Q)
fl = 2.0 * m * n * n - 2.0 * n ** 3 / 3
print(f"{m}x{n} factor {t(fac):.3f} ms ({fl / t(fac) / 1e9:.1f} TF/s); apply_qt k={k} {t(app):.3f} ms "
      f"({(4.0 * m * n * k - 2.0 * n * n * k) / t(app) / 1e9:.1f} TF/s); form_q {t(fq):.3f} ms ({fl / t(fq) / 1e9:.1f} TF/s)")
