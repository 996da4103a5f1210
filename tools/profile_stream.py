"""Timeline of the streaming skinny kernel (CAQR_PROFILE=1): chain phase vs
tree tail, from the kernel's globaltimer stamps (one factor call)."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["CAQR_PROFILE"] = "1"
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads

m, n = int(sys.argv[1]), int(sys.argv[2])
A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
A = caqr.colmajor_empty(m, n)
L = caqr.lib()
L.caqr_debug_profile_read.argtypes = [ctypes.c_void_p]
out = (ctypes.c_ulonglong * 16)()
for rep in range(3):
    A.copy_(A0)
    torch.cuda.synchronize()
    L.caqr_debug_profile_read(out)  # clears
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    R, ws = caqr.caqr_factor(A)
    e1.record()
    torch.cuda.synchronize()
    L.caqr_debug_profile_read(out)
    info = caqr.caqr_plan_info(m, n)
    chains = info["chains"]
    t0, t1, t2 = out[0], out[1], out[2]
    print(f"{m}x{n}: call {e0.elapsed_time(e1) * 1e3:.1f} us | chain phase {(t1 - t0) / 1e3:.1f} us "
          f"(mean chain {out[3] / chains / 1e3:.1f} us, mean tile wait {out[4] / chains / 1.9e3:.1f} us) | "
          f"tree tail after the last chain {(t2 - t1) / 1e3:.1f} us")
    if out[15]:
        print(f"   root path: in-CTA levels {(out[9] - out[8]) / 1e3:.2f} us, {out[14]} cross-CTA merges: publish "
              f"{out[10] / 1e3:.2f} ticket {out[11] / 1e3:.2f} load {out[12] / 1e3:.2f} merge {out[13] / 1e3:.2f} us; "
              f"tree start -> root {(out[15] - out[8]) / 1e3:.2f} us; root tree start - last chain end "
              f"{(out[8] - t1) / 1e3:.2f} us")
