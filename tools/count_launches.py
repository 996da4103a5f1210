"""Kernel launches of caqr_factor / apply_qt / form_q on one shape (launch trace)."""
import collections
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads

m, n, nb = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]) if len(sys.argv) > 3 else 0
opts = caqr.make_opts(0, nb)
A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
A = caqr.colmajor_empty(m, n)
A.copy_(A0)
R, ws = caqr.caqr_factor(A, opts=opts)
C = caqr.colmajor(A0[:, :8].clone())
torch.cuda.synchronize()
for name, f in (("factor", lambda: (A.copy_(A0), caqr.caqr_factor(A, R=R, ws=ws, opts=opts))),
                ("apply_qt", lambda: caqr.caqr_apply_qt(A, ws, C, opts=opts)),
                ("form_q", lambda: caqr.caqr_form_q(A, ws, opts=opts))):
    caqr.caqr_trace_begin(1 << 16)
    f()
    torch.cuda.synchronize()
    tr = caqr.caqr_trace_end(1 << 16)
    cnt = collections.Counter(t[0] for t in tr)
    print(f"{m}x{n} nb={nb} {name}: {len(tr)} launches {dict(cnt)}", flush=True)
