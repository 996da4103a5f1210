import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
m, n = int(sys.argv[1]), int(sys.argv[2])
A0 = workloads.device_gaussian(m, n, seed=0, dtype=torch.float32, device="cuda").t()
A = caqr.colmajor_empty(m, n)
for _ in range(2):
    A.copy_(A0)
    R, ws = caqr.caqr_factor(A)
torch.cuda.synchronize()
