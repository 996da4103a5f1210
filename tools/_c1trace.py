import os, sys
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
m, n = 4096, 16
A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
A = caqr.colmajor_empty(m, n)
R = caqr.colmajor_empty(n, n)
ws = torch.empty(caqr.caqr_workspace_bytes(m, n), dtype=torch.uint8, device="cuda")
print("ws bytes", ws.numel())
for _ in range(5):
    A.copy_(A0); caqr.caqr_factor(A, R=R, ws=ws)
torch.cuda.synchronize()
# graph of the bare call
g = torch.cuda.CUDAGraph()
s = torch.cuda.Stream()
with torch.cuda.stream(s):
    A.copy_(A0)
    torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=s):
        caqr.caqr_factor(A, R=R, ws=ws, stream=s)
torch.cuda.synchronize()
ts = []
for _ in range(50):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); g.replay(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
ts.sort(); print("graph replay median ms", ts[len(ts)//2])
caqr.caqr_trace_begin(1 << 10)
caqr.caqr_factor(A, R=R, ws=ws)
tr = caqr.caqr_trace_end(1 << 10)
for t in tr: print(t)
