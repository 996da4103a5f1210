"""Multi-GPU paths on real ranks (one process per GPU).  Skipped on boxes with
fewer than 2 GPUs (gpurun and the driver's round-end tests have one): the
per-rank kernels wait on one another, so they must not be emulated as several
launches on one device (the emulated form is test_gpu_parity's
test_peer_exchange_emulated_ranks, one cooperative launch)."""
import os
import socket

import numpy as np
import pytest

import oracle
from paper_conf_ipps_andersonbdk11_b200 import workloads

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

NGPU = torch.cuda.device_count() if torch.cuda.is_available() else 0


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, m, n, out_q):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_andersonbdk11_b200 import caqr
    from paper_conf_ipps_andersonbdk11_b200 import dist as cdist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", rank))
    A = workloads.gaussian(m, n, seed=7, dtype=np.float32)
    s0, rows = cdist.shard_rows(m, world, rank)
    res = {}
    for name, mk in (("nccl", lambda: cdist.DistTSQR()), ("peer", lambda: cdist.PeerTSQR(n, torch.float32))):
        eng = mk()
        for _ in range(3):  # three epochs through the peer mailboxes
            Al = caqr.colmajor_empty(rows, n, torch.float32)
            Al.copy_(torch.from_numpy(A[s0:s0 + rows]))
            R, ws, gather, cws = eng.factor(Al)
        torch.cuda.synchronize()
        res[name] = R.cpu().numpy()
        eng.close()
    out_q.put((rank, res))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.skipif(NGPU < 2, reason="needs 2 GPUs")
def test_peer_exchange_matches_nccl_two_ranks():
    import torch.multiprocessing as mp

    m, n = 20000, 96
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, m, n, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(2)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    A = workloads.gaussian(m, n, seed=7, dtype=np.float32)
    Ro = oracle.normalize_signs(oracle.qr(A.astype(np.float64), want_q=False))
    for _, r in res:
        # the peer exchange delivers the same stack as the all-gather: same bits
        assert np.array_equal(r["peer"], r["nccl"])
        Rn = oracle.normalize_signs(r["peer"].astype(np.float64))
        assert np.linalg.norm(Rn - Ro) / np.linalg.norm(Ro) <= 1e-4
    assert np.array_equal(res[0][1]["peer"], res[1][1]["peer"])
