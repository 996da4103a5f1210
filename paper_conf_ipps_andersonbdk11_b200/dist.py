"""Row-sharded multi-GPU TSQR: host-side plumbing (one process per GPU).

The math runs in libcaqr.so: ``caqr_dist_factor_*`` = local TSQR of the shard,
``ncclAllGather`` of the n x n local R factors over NVLink, and the same
deterministic combine tree on every rank (``caqr_combine_*``) -- the
distributed TSQR the paper cites with the GPUs as the leaves of
one more tree level.  This module only
  * decides the contiguous row shards (``shard_rows``),
  * creates the NCCL communicator inside libcaqr from a ``ncclUniqueId`` that
    rank 0 makes and torch.distributed broadcasts (``DistTSQR``),
  * offers ``allgather_r`` -- the same exchange through torch.distributed
    (any backend, incl. gloo on CPU), used to test the exchange order and by
    callers that already hold a torch process group.
"""
from __future__ import annotations

import ctypes
from typing import Tuple


def shard_rows(m: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous row shard of rank `rank`: (first_row, rows).  Even split,
    remainder to the last rank."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    base = m // world
    start = rank * base
    rows = base if rank < world - 1 else m - start
    return start, rows


def check_shards(m: int, n: int, world: int) -> None:
    """Every shard must hold at least n rows (each local R is n x n)."""
    for r in range(world):
        _, rows = shard_rows(m, world, r)
        if rows < n:
            raise ValueError(f"rank {r} would get {rows} < n = {n} rows; use fewer ranks")


def allgather_r(R_local, group=None):
    """Stack every rank's n x n R (rank order) into a (world*n) x n tensor via
    torch.distributed.all_gather (works for gloo CPU tensors and NCCL CUDA
    tensors).  Returns the stacked tensor (row-major torch layout)."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    parts = [torch.empty_like(R_local) for _ in range(world)]
    dist.all_gather(parts, R_local.contiguous(), group=group)
    return torch.cat(parts, dim=0)


def local_form_q(A_local, ws, gather, cws, rank: int, world: int, opts=None, stream=None):
    """Rows of the global thin Q held by rank `rank` (the
    explicit basis of a row-sharded matrix, e.g. an s-step Krylov basis).

    With A_p = Q_p R_p locally and [R_1; ...; R_P] = Q_c R (the combine), the
    global factor is A = diag(Q_1 ... Q_P) Q_c R, so rank p's rows of Q are
    Q_p Q_c[p n:(p+1) n, :] = Q_p_full [Q_c,p; 0].  Every rank forms the small
    Q_c (P n x n) from the combine it already holds (identical bits on every
    rank) and applies its local Q: no communication beyond the factor's
    all-gather.  All steps are libcaqr kernels."""
    from . import caqr

    import contextlib

    import torch

    m, n = A_local.shape
    # every step -- the library calls and the torch copy between them -- on
    # the caller's stream (the copy would otherwise run on torch's current
    # stream, unordered with the library calls)
    ctx = torch.cuda.stream(stream) if isinstance(stream, torch.cuda.Stream) else contextlib.nullcontext()
    with ctx:
        Qc = caqr.colmajor_empty(world * n, n, A_local.dtype, A_local.device)
        caqr.caqr_set_identity(Qc, stream=stream)
        caqr.caqr_combine_apply(gather, world, cws, Qc, trans=False, stream=stream)
        Q = caqr.colmajor_empty(m, n, A_local.dtype, A_local.device)
        caqr.caqr_set_identity(Q, stream=stream)  # then overwrite the top n x n with Q_c,p
        Q[:n].copy_(Qc[rank * n:(rank + 1) * n])
        caqr.caqr_apply_q(A_local, ws, Q, opts=opts, stream=stream)
    return Q


def agree_shards(m_local: int, n: int, group=None) -> None:
    """Every rank checks its own shard (m_local >= n >= 0, n <= 256) and the
    ranks all-reduce the verdict, so that either all of them enter the NCCL
    collective or all of them raise (a rank that bailed out alone would leave
    the others blocked in the all-gather).  Works with any torch.distributed
    backend (gloo on CPU in the tests)."""
    import torch
    import torch.distributed as dist

    ok = 1 if (0 <= n <= 256 and m_local >= n) else 0
    backend = dist.get_backend(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")
    t = torch.tensor([ok], dtype=torch.int32, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
    if int(t.item()) != 1:
        raise ValueError(f"some rank's shard is unusable (this rank: {m_local} rows, n = {n}; every shard needs "
                         f"m_local >= n and n <= 256)")


class DistTSQR:
    """NCCL communicator owned by libcaqr (caqr_dist_create) for the ranks of a
    torch.distributed group; `factor` runs caqr_dist_factor_* on a local shard."""

    def __init__(self, group=None):
        import torch.distributed as dist

        from . import caqr

        self.caqr = caqr
        self.group = group
        self.L = caqr.lib()
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        uid = (ctypes.c_char * 128)()
        if self.rank == 0:
            caqr._check("caqr_dist_unique_id", self.L.caqr_dist_unique_id(uid))
        obj = [bytes(uid)]
        dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0) if group is not None else 0,
                                   group=group)
        uid = (ctypes.c_char * 128).from_buffer_copy(obj[0])
        h = ctypes.c_void_p()
        caqr._check("caqr_dist_create", self.L.caqr_dist_create(ctypes.byref(h), self.world, self.rank, uid))
        self.handle = h

    def factor(self, A_local, opts=None, stream=None, timeout_s: float = 600.0):
        """Factor the local column-major shard in place; returns (R, ws, gather,
        cws): the global R (identical bits on every rank), the local workspace,
        the combine's stacked tree vectors and its workspace.  All ranks first
        agree that every shard is usable (else every rank raises, none enters
        the collective); the call then waits at most timeout_s for its stream
        (caqr_dist_wait: on timeout or an NCCL error the communicator is aborted
        and CaqrError is raised instead of hanging)."""
        import torch

        c = self.caqr
        code, suf = c._dtype_code(A_local)
        m, n = A_local.shape
        agree_shards(m, n, self.group)
        pa, lda = c._colmajor(A_local, "A")
        R = c.colmajor_empty(n, n, A_local.dtype, A_local.device)
        ws = torch.empty(max(c.caqr_workspace_bytes(m, n, code, opts), 1), dtype=torch.uint8,
                         device=A_local.device)
        gather = c.colmajor_empty(self.world * n, n, A_local.dtype, A_local.device)
        cws = torch.empty(c.caqr_combine_workspace_bytes(self.world, n, code), dtype=torch.uint8,
                          device=A_local.device)
        info = getattr(self.L, f"caqr_dist_factor_{suf}")(
            self.handle, m, n, pa, lda, R.data_ptr(), n, ws.data_ptr(), ws.numel(), gather.data_ptr(),
            cws.data_ptr(), cws.numel(), c._optp(opts), c._stream(stream))
        c._check(f"caqr_dist_factor_{suf}", info)
        if timeout_s is not None:
            c._check("caqr_dist_wait", self.L.caqr_dist_wait(self.handle, c._stream(stream),
                                                             int(timeout_s * 1000)))
        return R, ws, gather, cws

    def form_q(self, A_local, ws, gather, cws, opts=None, stream=None):
        """This rank's rows of the global thin Q (after ``factor``)."""
        return local_form_q(A_local, ws, gather, cws, self.rank, self.world, opts=opts, stream=stream)

    def close(self):
        if getattr(self, "handle", None) is not None:
            self.L.caqr_dist_destroy(self.handle)
            self.handle = None

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass


class PeerTSQR:
    """Row-sharded TSQR whose R exchange is ``caqr_peer_exchange_*`` -- each rank
    stores its n x n R straight into every rank's mailbox over NVLink (CUDA IPC
    peer pointers) and raises a flag; the receive side restacks the P blocks into
    the combine's input in the same kernel -- instead of the NCCL all-gather of
    DistTSQR.  Same result bits as DistTSQR (same local factor, same combine).

    Construction maps every rank's mailbox (caqr_peer_mailbox_bytes) and flag
    array into every process (caqr_ipc_handle / caqr_ipc_open, handles swapped
    with torch.distributed.all_gather_object), so it needs one process per GPU on
    one node with peer access.  n and the dtype are fixed per instance."""

    def __init__(self, n: int, dtype=None, group=None, timeout_ms: int = 60000):
        import torch
        import torch.distributed as dist

        from . import caqr

        self.caqr = caqr
        self.group = group
        self.n = n
        self.dtype = dtype or torch.float32
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.timeout_ms = timeout_ms
        dev = torch.device("cuda", torch.cuda.current_device())
        code, _ = caqr._dtype_code(torch.empty(0, dtype=self.dtype))
        self.code = code
        self.mailbox = torch.empty(max(caqr.caqr_peer_mailbox_bytes(self.world, n, code), 16), dtype=torch.uint8,
                                   device=dev)
        self.flags = torch.zeros(max(self.world, 4), dtype=torch.int32, device=dev)
        self.status = torch.zeros(1, dtype=torch.int32, device=dev)
        torch.cuda.synchronize()
        mine = (caqr.caqr_ipc_handle(self.mailbox), caqr.caqr_ipc_handle(self.flags))
        allh = [None] * self.world
        dist.all_gather_object(allh, mine, group=group)
        self.opened = []
        mb, fl = [], []
        for q, (hm, hf) in enumerate(allh):
            if q == self.rank:
                mb.append(self.mailbox.data_ptr())
                fl.append(self.flags.data_ptr())
            else:
                pm, pf = caqr.caqr_ipc_open(hm), caqr.caqr_ipc_open(hf)
                self.opened += [pm, pf]
                mb.append(pm)
                fl.append(pf)
        self.mb_ptrs = caqr._ptr_array(mb, dev)
        self.fl_ptrs = caqr._ptr_array(fl, dev)
        self.epoch = 0
        dist.barrier(group=group)  # every rank's flags are zero before the first exchange

    def factor(self, A_local, opts=None, stream=None):
        """Factor the local column-major shard in place; returns (R, ws, gather,
        cws) exactly as DistTSQR.factor.  Raises CaqrError (CAQR_ERR_TIMEOUT)
        if some rank's block did not arrive within timeout_ms."""
        import torch

        c = self.caqr
        m, n = A_local.shape
        if n != self.n or A_local.dtype != self.dtype:
            raise ValueError(f"PeerTSQR built for n = {self.n}, {self.dtype}")
        agree_shards(m, n, self.group)
        Rl, ws = c.caqr_factor(A_local, opts=opts, stream=stream)
        self.epoch += 1
        gather = c.colmajor_empty(self.world * n, n, A_local.dtype, A_local.device)
        with torch.cuda.stream(stream or torch.cuda.current_stream()):
            self.status.zero_()  # a previous call's timeout must not fail this one
        c.caqr_peer_exchange(self.world, self.rank, Rl, self.mb_ptrs, self.fl_ptrs, gather, self.epoch,
                             status=self.status, timeout_ms=self.timeout_ms, stream=stream)
        R, cws = c.caqr_combine(gather, self.world, stream=stream)
        (stream if stream is not None else torch.cuda.current_stream()).synchronize()
        st = int(self.status.item())
        if st:
            raise c.CaqrError("caqr_peer_exchange", st)
        return R, ws, gather, cws

    def form_q(self, A_local, ws, gather, cws, opts=None, stream=None):
        return local_form_q(A_local, ws, gather, cws, self.rank, self.world, opts=opts, stream=stream)

    def close(self):
        for p in getattr(self, "opened", []):
            try:
                self.caqr.caqr_ipc_close(p)
            except Exception:
                pass
        self.opened = []
