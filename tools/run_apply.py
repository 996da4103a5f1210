"""Profiling driver: factor once, then caqr_apply_qt (k columns) a few times."""
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
for _ in range(2):
    caqr.caqr_apply_qt(A, ws, C)
torch.cuda.synchronize()
print("done")
