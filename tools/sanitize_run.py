"""Small invocations of every kernel family, for compute-sanitizer (memcheck /
racecheck / synccheck): fused TSQR (fp32/fp64, chains + tree), streaming skinny
kernel, split path, CAQR panel loop, Q^T C / Q C / form_q, combine, robust PCA."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
from paper_conf_ipps_andersonbdk11_b200.rpca import RobustPCA


def run(m, n, dt=torch.float32, opts=None):
    A = caqr.colmajor_empty(m, n, dt)
    A.copy_(torch.from_numpy(workloads.gaussian(m, n, seed=1, dtype=np.float32 if dt == torch.float32 else np.float64)))
    R, ws = caqr.caqr_factor(A, opts=opts)
    Q = caqr.caqr_form_q(A, ws, opts=opts)
    C = caqr.colmajor_empty(m, 3, dt)
    C.copy_(torch.from_numpy(workloads.gaussian(m, 3, seed=2, dtype=np.float32 if dt == torch.float32 else np.float64)))
    caqr.caqr_apply_qt(A, ws, C, opts=opts)
    caqr.caqr_apply_q(A, ws, C, opts=opts)
    torch.cuda.synchronize()


which = sys.argv[1] if len(sys.argv) > 1 else "all"
if which in ("all", "fused"):
    run(20000, 48)                     # fused, chains + tree
    run(30000, 100)                    # fused: 4 panels, ragged last (4 columns), 3-block trailing updates
    run(5000, 40, torch.float64)       # fused fp64
if which in ("all", "stream"):
    run(300_000, 8)                    # streaming skinny kernel
if which in ("all", "caqr"):
    run(600, 300, opts=caqr.make_opts(panel_cols=64))  # CAQR panel loop (split + early start)
if which in ("all", "peer"):
    P, n = 3, 24
    Rs = [torch.triu(torch.randn(n, n, device="cuda")).t().contiguous().t() for _ in range(P)]
    mb = [torch.zeros(caqr.caqr_peer_mailbox_bytes(P, n, caqr.CAQR_F32) // 4, device="cuda") for _ in range(P)]
    fl = [torch.zeros(P, dtype=torch.int32, device="cuda") for _ in range(P)]
    for ep in (1, 2):
        gs = [caqr.colmajor_empty(P * n, n) for _ in range(P)]
        caqr.caqr_peer_exchange_emulate(Rs, mb, fl, gs, ep)
    torch.cuda.synchronize()
if which in ("all", "rpca"):
    M = workloads.video(frames=20, h=48, w=64).astype(np.float32)
    Md = caqr.colmajor_empty(*M.shape)
    Md.copy_(torch.from_numpy(M))
    rp = RobustPCA(Md)
    for _ in range(2):
        rp.step()
    torch.cuda.synchronize()
print("ok", which)
