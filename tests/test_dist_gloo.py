"""Multi-process host logic of the row-sharded TSQR on CPU (gloo, world size 2).

The GPU math (local TSQR + NCCL all-gather + combine) needs >= 2 GPUs; here the
same exchange (dist.allgather_r through torch.distributed) and sharding run
with the oracle as the local and combine QR (tests may use the oracle), and the
result must equal the single-shot R: R is unique up to row signs, so a tree
whose leaves are ranks gives the oracle's R."""
import os
import socket

import numpy as np
import pytest

import oracle
from paper_conf_ipps_andersonbdk11_b200 import dist as cdist
from paper_conf_ipps_andersonbdk11_b200 import workloads


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, m, n, out_q):
    import torch
    import torch.distributed as dist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    A = workloads.gaussian(m, n, seed=3, dtype=np.float64)
    start, rows = cdist.shard_rows(m, world, rank)
    R_local = oracle.qr(A[start:start + rows], want_q=False, acc="d")
    stacked = cdist.allgather_r(torch.from_numpy(np.ascontiguousarray(R_local)))
    R = oracle.qr(stacked.numpy(), want_q=False, acc="d")
    out_q.put((rank, R, stacked.numpy()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("m,n", [(1000, 16), (777, 33)])
def test_two_rank_tsqr_matches_single_shot(m, n):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, m, n, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort(key=lambda t: t[0])
    A = workloads.gaussian(m, n, seed=3, dtype=np.float64)
    R_ref = oracle.normalize_signs(oracle.qr(A, want_q=False, acc="d"))
    for _, R, stacked in res:
        assert np.linalg.norm(oracle.normalize_signs(R) - R_ref) / np.linalg.norm(R_ref) < 1e-13
    # rank order of the exchange: block r of the stack is rank r's local R
    s0, r0 = cdist.shard_rows(m, 2, 0)
    R0 = oracle.qr(A[s0:s0 + r0], want_q=False, acc="d")
    assert np.array_equal(res[0][2][:n], R0)
    # both ranks hold bitwise-identical combined R (same inputs, same order)
    assert np.array_equal(res[0][1], res[1][1])


def test_shard_rows():
    for m, w in [(10, 3), (8_000_000, 8), (1000, 7)]:
        spans = [cdist.shard_rows(m, w, r) for r in range(w)]
        assert spans[0][0] == 0
        for (s, c), (s2, _) in zip(spans, spans[1:]):
            assert s + c == s2
        assert spans[-1][0] + spans[-1][1] == m
    with pytest.raises(ValueError):
        cdist.check_shards(100, 60, 2)
    cdist.check_shards(8_000_000, 192, 8)


def _agree_worker(rank, world, port, rows, n, out_q):
    import torch.distributed as dist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cdist.agree_shards(rows[rank], n)
        out_q.put((rank, "ok"))
    except ValueError:
        out_q.put((rank, "raised"))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("rows,expect", [((500, 400), "ok"), ((500, 40), "raised"), ((10, 500), "raised")])
def test_agree_shards_all_or_none(rows, expect):
    """DistTSQR.factor's pre-collective check (agree_shards): every rank checks
    its own shard and the verdict is all-reduced, so either every rank enters
    the NCCL all-gather or every rank raises -- one bad shard (rank 1: 40 rows <
    n = 64) must not leave the other rank blocked in the collective."""
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_agree_worker, args=(r, 2, port, rows, 64, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res == {0: expect, 1: expect}
