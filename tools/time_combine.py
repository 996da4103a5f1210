"""Device time of the distributed TSQR's post-exchange half (caqr_dist_combine_blocks:
restack + structured combine tree) for P stacked n x n R factors, one GPU."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_andersonbdk11_b200 import caqr

for P in (2, 4, 8):
    for n in (8, 100, 192):
        blocks = torch.triu(torch.randn(P, n, n, device="cuda")).transpose(1, 2).contiguous().reshape(-1)
        R, gather, cws = caqr.caqr_dist_combine_blocks(blocks, P, n)
        ts = []
        for r in range(12):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            caqr.caqr_dist_combine_blocks(blocks, P, n, gather=gather, R=R, cws=cws)
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        ts.sort()
        print(f"P={P} n={n:3d}: combine {ts[len(ts) // 2] * 1e3:8.1f} us", flush=True)
