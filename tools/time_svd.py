"""Time caqr_svd_small on the R of the video robust-PCA input (diagnostics)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
M = workloads.video(seed=0).astype(np.float32)
A = caqr.colmajor_empty(*M.shape); A.copy_(torch.from_numpy(M))
R, ws = caqr.caqr_factor(A)
U = caqr.colmajor_empty(100, 100); s = torch.empty(100, device="cuda")
for _ in range(3):
    caqr.caqr_svd_small(R, U, s, want_v=False)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10):
    caqr.caqr_svd_small(R, U, s, want_v=False)
e1.record(); torch.cuda.synchronize()
print(os.environ.get("CAQR_SVD_SWEEPS", "30"), "sweeps max:", e0.elapsed_time(e1) / 10, "ms;  sigma[0..3]", s[:3].tolist(), "sigma[-1]", s[-1].item())
