"""CAQR_PROFILE=1 phase profile of the chain kernel (diagnostics)."""
import ctypes, os, sys
os.environ["CAQR_PROFILE"] = "1"
os.environ.setdefault("CAQR_CHAIN", "1")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
m = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
n = int(sys.argv[2]) if len(sys.argv) > 2 else 192
A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
A = caqr.colmajor_empty(m, n, torch.float32)
L = caqr.lib()
L.caqr_debug_profile_read.argtypes = [ctypes.c_void_p]
out = (ctypes.c_ulonglong * 16)()
for it in range(3):
    A.copy_(A0)
    caqr.caqr_factor(A)
    torch.cuda.synchronize()
    L.caqr_debug_profile_read(out)
names = ["load_panel", "factor_loop", "post_factor(conv+G+T)", "stage_wait(+xload)", "conv C+GEMM1 | mma.sync", "chain_end", "W,T,W2 conv", "GEMM2 wait", "epilogue"]
tot = sum(out[i] for i in range(9)) or 1
for i, nm in enumerate(names):
    print(f"{nm:18s} {out[i] / tot * 100:5.1f}%  {out[i] / 1.9e9:.4f} CTA-s")
print("total CTA-s", tot / 1.9e9)
