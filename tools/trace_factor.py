"""Per-kernel device time of one caqr_factor (library launch tracing)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
m, n, nb = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]) if len(sys.argv) > 3 else 0
dt = torch.float64 if os.environ.get("DT") == "f64" else torch.float32
A0 = workloads.device_gaussian(m, n, seed=0, dtype=dt, device="cuda").t()
A = caqr.colmajor_empty(m, n, dt)
opts = caqr.make_opts(0, nb)
A.copy_(A0); caqr.caqr_factor(A, opts=opts); torch.cuda.synchronize()
A.copy_(A0); torch.cuda.synchronize()
caqr.caqr_trace_begin(1 << 16)
caqr.caqr_factor(A, opts=opts)
tr = caqr.caqr_trace_end(1 << 16)
per = {}
for name, ms, fl, by in tr:
    d = per.setdefault(name, [0, 0.0, 0.0]); d[0] += 1; d[1] += ms; d[2] += fl
tot = sum(v[1] for v in per.values())
for k, (c, ms, fl) in sorted(per.items(), key=lambda kv: -kv[1][1]):
    print(f"{k:14s} launches {c:5d}  {ms:9.3f} ms ({ms/tot*100:5.1f}%)  {fl/ms/1e9 if ms > 0 else 0:8.2f} TFLOP/s")
print(f"total {tot:.3f} ms")
