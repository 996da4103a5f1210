"""Per-kernel device time of caqr_apply_qt / caqr_form_q (launch tracing)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
m, n, k = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
A = caqr.colmajor_empty(m, n)
A.copy_(workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t())
R, ws = caqr.caqr_factor(A)
C = caqr.colmajor_empty(m, k)
C.copy_(workloads.device_gaussian(m, k, seed=1, dtype=torch.float32, device="cuda").t())
caqr.caqr_apply_qt(A, ws, C); caqr.caqr_form_q(A, ws); torch.cuda.synchronize()
for name, f in (("apply_qt", lambda: caqr.caqr_apply_qt(A, ws, C)), ("form_q", lambda: caqr.caqr_form_q(A, ws))):
    caqr.caqr_trace_begin()
    f()
    tr = caqr.caqr_trace_end()
    agg = {}
    for kname, t, fl, by in tr:
        a = agg.setdefault(kname, [0, 0.0, 0.0])
        a[0] += 1; a[1] += t; a[2] += by
    print(f"{m}x{n} {name}: " + ", ".join(f"{kk} x{v[0]} {v[1]*1e3:.1f} us ({v[2]/max(v[1],1e-9)/1e6:.0f} GB/s alg)" for kk, v in agg.items()))
