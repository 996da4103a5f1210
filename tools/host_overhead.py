"""Host cost of one caqr_factor call (Python + ctypes + C-ABI plan + launches)
on a small shape, vs the device time of the same call replayed from a CUDA
graph.  python tools/host_overhead.py [m n]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads

m = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
n = int(sys.argv[2]) if len(sys.argv) > 2 else 16
A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
A = caqr.colmajor_empty(m, n)
A.copy_(A0)
R, ws = caqr.caqr_factor(A)
torch.cuda.synchronize()
N = 500
hs, rs = [], []
for _ in range(200):  # GPU idle before each call: pure host cost (no queue back-pressure)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    caqr.caqr_factor(A, R=R, ws=ws)
    hs.append(time.perf_counter() - t0)
L = caqr.lib()
st = torch.cuda.current_stream().cuda_stream
for _ in range(200):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    L.caqr_factor_f32(m, n, A.data_ptr(), m, R.data_ptr(), n, ws.data_ptr(), ws.numel(), None, st)
    rs.append(time.perf_counter() - t0)
torch.cuda.synchronize()
med = lambda v: 1e6 * sorted(v)[len(v) // 2]  # noqa: E731
print(f"{m}x{n}: host cost per call {med(hs):.1f} us (caqr.py), {med(rs):.1f} us (raw ctypes C-ABI)")
g = torch.cuda.CUDAGraph()
s = torch.cuda.Stream()
s.wait_stream(torch.cuda.current_stream())
with torch.cuda.stream(s):
    caqr.caqr_factor(A, R=R, ws=ws)
torch.cuda.current_stream().wait_stream(s)
with torch.cuda.graph(g):
    caqr.caqr_factor(A, R=R, ws=ws)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for _ in range(5):
    g.replay()
e0.record()
for _ in range(N):
    g.replay()
e1.record()
torch.cuda.synchronize()
print(f"   graph replay back to back: {1e3 * e0.elapsed_time(e1) / N:.1f} us/call (device)")
ts = []
for _ in range(50):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    g.replay()
    b.record()
    torch.cuda.synchronize()
    ts.append(a.elapsed_time(b))
print(f"   graph replay, one at a time: {1e3 * sorted(ts)[len(ts) // 2]:.1f} us/call")
