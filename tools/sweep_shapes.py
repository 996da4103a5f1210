"""SURVEY 8(f) f3 measurements (the paper's Fig. 7 / Fig. 9 analogues, P:L796-824,
P:L915-922): caqr_factor GFLOP/s (LAPACK count) over
  * height 8192 x width 64 ... 8192 (CAQR panel width nb = 64 for n > 224),
  * leaf (tile) height b for the tall-skinny shapes 1M x 192 and 110,592 x 100,
  * panel width nb for 8192 x 8192.
Median of a few calls, CUDA events, A restored outside the timed call."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads


def t_factor(m, n, leaf=0, nb=0, reps=3):
    A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
    A = caqr.colmajor_empty(m, n)
    opts = caqr.make_opts(leaf, nb)
    ts = []
    for r in range(reps + 1):
        A.copy_(A0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        caqr.caqr_factor(A, opts=opts)
        e1.record()
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    ms = sorted(ts)[len(ts) // 2]
    del A0, A
    torch.cuda.empty_cache()
    return ms, (2.0 * m * n * n - 2.0 * n ** 3 / 3) / ms / 1e9


print("# height 8192, width sweep (Fig. 9 analogue): n, ms, TFLOP/s")
for n in (64, 128, 192, 256, 512, 1024, 2048, 4096, 8192):
    ms, tf = t_factor(8192, n, nb=64 if n > 224 else 0)
    print(f"8192 x {n:5d}  {ms:9.3f} ms  {tf:6.2f} TFLOP/s")
print("# leaf (tile) height sweep (Fig. 7 analogue)")
for m, n in ((1_000_000, 192), (110_592, 100)):
    for b in (128, 160, 192, 224):
        ms, tf = t_factor(m, n, leaf=b)
        print(f"{m} x {n}  b = {b:3d}  {ms:8.3f} ms  {tf:6.2f} TFLOP/s")
print("# panel width nb for 8192 x 8192")
for nb in (32, 64, 96, 128, 192):
    ms, tf = t_factor(8192, 8192, nb=nb, reps=1)
    print(f"8192 x 8192  nb = {nb:3d}  {ms:8.2f} ms  {tf:6.2f} TFLOP/s")
