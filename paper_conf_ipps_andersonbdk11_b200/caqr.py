"""Thin Python binding of libcaqr.so (include/caqr.h): argument marshalling only.

Every step of the factorisation runs in the CUDA kernels behind the C ABI; this
module only turns torch CUDA tensors into (pointer, leading dimension) pairs,
picks the f32/f64 entry point, and raises on a nonzero LAPACK-style info.
There is NO CPU fallback: without the built library or a GPU, calls raise.

Matrices are column-major, as in the ABI: a torch tensor of shape (m, n) with
stride (1, ld), ld >= m -- e.g. ``colmajor_empty(m, n)`` or ``x.t().contiguous().t()``.
"""
from __future__ import annotations

import ctypes
import os
import re
import threading
from typing import Optional, Tuple

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libcaqr.so")
HEADER_PATH = os.path.join(os.path.dirname(_HERE), "include", "caqr.h")

CAQR_F32, CAQR_F64 = 0, 1
_lock = threading.Lock()
_lib = None


class CaqrError(RuntimeError):
    def __init__(self, fn: str, info: int, msg: str = ""):
        super().__init__(f"{fn} returned info={info}: {msg}")
        self.info = info


class Opts(ctypes.Structure):
    """caqr_opts: leaf_rows (b), panel_cols (nb); 0 = default."""

    _fields_ = [("leaf_rows", ctypes.c_int64), ("panel_cols", ctypes.c_int64),
                ("reserved", ctypes.c_int64 * 6)]


def _i64(*xs):
    return [ctypes.c_int64] * len(xs)


def lib() -> ctypes.CDLL:
    """Load the in-tree libcaqr.so (raises if it was not built)."""
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run `python -m paper_conf_ipps_andersonbdk11_b200.build` "
                               "(no CPU fallback exists)")
        # CAQR_LIB_PATH: development A/B of alternative builds (tools/ab_time.py)
        L = ctypes.CDLL(os.environ.get("CAQR_LIB_PATH", LIB_PATH))
        i64, vp, sz, ip = ctypes.c_int64, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int
        op = ctypes.POINTER(Opts)
        L.caqr_workspace_bytes.argtypes = [i64, i64, ip, op]
        L.caqr_workspace_bytes.restype = sz
        for suf in ("f32", "f64"):
            f = getattr(L, f"caqr_factor_{suf}")
            f.argtypes = [i64, i64, vp, i64, vp, i64, vp, sz, op, vp]
            f.restype = ip
            for name in ("apply_qt", "apply_q"):
                f = getattr(L, f"caqr_{name}_{suf}")
                f.argtypes = [i64, i64, vp, i64, vp, i64, vp, i64, op, vp]
                f.restype = ip
            f = getattr(L, f"caqr_form_q_{suf}")
            f.argtypes = [i64, i64, vp, i64, vp, vp, i64, op, vp]
            f.restype = ip
            f = getattr(L, f"caqr_combine_{suf}")
            f.argtypes = [ip, i64, vp, i64, vp, i64, vp, sz, vp]
            f.restype = ip
            f = getattr(L, f"caqr_combine_apply_{suf}")
            f.argtypes = [ip, i64, vp, i64, vp, ip, i64, vp, i64, vp]
            f.restype = ip
            f = getattr(L, f"caqr_dist_factor_{suf}")
            f.argtypes = [vp, i64, i64, vp, i64, vp, i64, vp, sz, vp, vp, sz, op, vp]
            f.restype = ip
        for suf in ("f32", "f64"):
            f = getattr(L, f"caqr_factor_host_{suf}")
            f.argtypes = [i64, i64, ip, vp, i64, vp, i64, vp, i64, vp, sz, op, vp]
            f.restype = ip
        L.caqr_factor_host_workspace_bytes.argtypes = [i64, i64, ip, ip, op]
        L.caqr_factor_host_workspace_bytes.restype = sz
        L.caqr_factor_host_layout.argtypes = [i64, i64, ip, ip, op, ip, ctypes.POINTER(ctypes.c_int64)]
        L.caqr_factor_host_layout.restype = ip
        L.caqr_combine_workspace_bytes.argtypes = [ip, i64, ip]
        L.caqr_combine_workspace_bytes.restype = sz
        L.caqr_strerror.argtypes = [ip]
        L.caqr_strerror.restype = ctypes.c_char_p
        L.caqr_last_cuda_error.restype = ip
        L.caqr_build_info.restype = ctypes.c_char_p
        L.caqr_plan_info.argtypes = [i64, i64, ip, op, ctypes.POINTER(ctypes.c_int64)]
        L.caqr_plan_info.restype = ip
        L.caqr_tune.argtypes = [i64, i64, ip, vp, i64, ip, ctypes.POINTER(Opts), ctypes.POINTER(ctypes.c_float),
                                ctypes.POINTER(ctypes.c_float), ctypes.POINTER(ip), vp]
        L.caqr_tune.restype = ip
        L.caqr_trace_begin.argtypes = [ip]
        L.caqr_trace_begin.restype = ip
        L.caqr_trace_end.argtypes = [ctypes.POINTER(ip), ctypes.POINTER(ctypes.c_float),
                                     ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double), ip]
        L.caqr_trace_end.restype = ip
        L.caqr_kernel_name.argtypes = [ip]
        L.caqr_kernel_name.restype = ctypes.c_char_p
        L.caqr_dist_unique_id.argtypes = [vp]
        L.caqr_dist_unique_id.restype = ip
        L.caqr_dist_create.argtypes = [ctypes.POINTER(vp), ip, ip, vp]
        L.caqr_dist_create.restype = ip
        L.caqr_dist_destroy.argtypes = [vp]
        L.caqr_dist_destroy.restype = None
        L.caqr_dist_wait.argtypes = [vp, vp, ip]
        L.caqr_dist_wait.restype = ip
        for suf in ("f32", "f64"):
            f = getattr(L, f"caqr_dist_combine_blocks_{suf}")
            f.argtypes = [ip, i64, vp, vp, i64, vp, i64, vp, sz, vp]
            f.restype = ip
            f = getattr(L, f"caqr_peer_exchange_{suf}")
            f.argtypes = [ip, ip, i64, vp, i64, vp, vp, vp, ip, vp, ip, vp]
            f.restype = ip
            f = getattr(L, f"caqr_peer_exchange_emulate_{suf}")
            f.argtypes = [ip, i64, vp, i64, vp, vp, vp, ip, vp]
            f.restype = ip
        L.caqr_peer_mailbox_bytes.argtypes = [ip, i64, ip]
        L.caqr_peer_mailbox_bytes.restype = sz
        L.caqr_ipc_handle.argtypes = [vp, vp]
        L.caqr_ipc_handle.restype = ip
        L.caqr_ipc_open.argtypes = [vp, ctypes.POINTER(vp)]
        L.caqr_ipc_open.restype = ip
        L.caqr_ipc_close.argtypes = [vp]
        L.caqr_ipc_close.restype = ip
        fl = ctypes.c_float
        for suf in ("f32", "f64"):
            f = getattr(L, f"caqr_lstsq_{suf}")
            f.argtypes = [i64, i64, vp, i64, vp, i64, vp, i64, op, vp]
            f.restype = ip
            f = getattr(L, f"caqr_set_identity_{suf}")
            f.argtypes = [i64, i64, vp, i64, vp]
            f.restype = ip
            f = getattr(L, f"caqr_trsm_upper_{suf}")
            f.argtypes = [i64, i64, vp, i64, vp, i64, vp]
            f.restype = ip
            f = getattr(L, f"caqr_svd_small_{suf}")
            f.argtypes = [i64, vp, i64, vp, i64, vp, vp, i64, vp]
            f.restype = ip
        L.caqr_svt_core_f32.argtypes = [i64, vp, i64, vp, vp, i64, fl, vp, i64, vp]
        L.caqr_svt_core_r_f32.argtypes = [i64, vp, i64, vp, vp, i64, fl, vp, i64, vp]
        L.caqr_embed_top_f32.argtypes = [i64, i64, vp, i64, vp, i64, vp]
        L.caqr_rpca_update_f32.argtypes = [i64, i64, vp, i64, vp, i64, vp, i64, vp, i64, vp, i64, fl, fl, fl,
                                           vp, vp]
        L.caqr_rpca_init_f32.argtypes = [i64, i64, vp, i64, fl, vp, i64, vp, i64, vp, i64, fl, vp]
        L.caqr_absmax_f32.argtypes = [i64, i64, vp, i64, vp, vp]
        db = ctypes.c_double
        L.caqr_rpca_schedule_f32.argtypes = [vp, vp, db, db, db, db, vp, vp]
        L.caqr_rpca_init_sched_f32.argtypes = [i64, i64, vp, i64, vp, vp, i64, vp, i64, vp, i64, vp]
        L.caqr_svt_core_r_sched_f32.argtypes = [i64, vp, i64, vp, vp, i64, vp, vp, i64, vp]
        L.caqr_rpca_update_sched_f32.argtypes = [i64, i64, vp, i64, vp, i64, vp, i64, vp, i64, vp, i64, vp, vp,
                                                 vp]
        for name in ("svt_core", "svt_core_r", "embed_top", "rpca_update", "rpca_init", "absmax", "rpca_schedule",
                     "rpca_init_sched", "svt_core_r_sched", "rpca_update_sched"):
            getattr(L, f"caqr_{name}_f32").restype = ip
        _lib = L
        return L


def header_functions():
    """Names of every function the C header declares (for the export test)."""
    with open(HEADER_PATH) as f:
        txt = f.read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(caqr_[a-z0-9_]+)\s*\(", txt)))


def make_opts(leaf_rows: int = 0, panel_cols: int = 0) -> Optional[Opts]:
    if not leaf_rows and not panel_cols:
        return None
    return Opts(int(leaf_rows), int(panel_cols))


def _optp(opts):
    return ctypes.byref(opts) if opts is not None else None


def _check(fn: str, info: int):
    if info != 0:
        L = lib()
        msg = L.caqr_strerror(info).decode()
        if info == 1:
            msg += f" (cudaError {L.caqr_last_cuda_error()})"
        raise CaqrError(fn, info, msg)


# ---- torch plumbing ---------------------------------------------------------
def _torch():
    import torch

    return torch


def _dtype_code(t) -> Tuple[int, str]:
    torch = _torch()
    if t.dtype == torch.float32:
        return CAQR_F32, "f32"
    if t.dtype == torch.float64:
        return CAQR_F64, "f64"
    raise TypeError(f"caqr: dtype {t.dtype} not supported (float32 / float64)")


def _colmajor(t, name: str, host: bool = False):
    if not host and not t.is_cuda:
        raise ValueError(f"caqr: {name} must be a CUDA tensor (no CPU path)")
    if t.dim() != 2:
        raise ValueError(f"caqr: {name} must be 2-D")
    m, n = t.shape
    if n > 1 and t.stride(0) != 1 and m > 1:
        raise ValueError(f"caqr: {name} must be column-major (stride(0) == 1); use colmajor()")
    ld = t.stride(1) if n > 1 else max(m, 1)
    return t.data_ptr(), max(ld, m, 1)


def colmajor_empty(m: int, n: int, dtype=None, device="cuda"):
    torch = _torch()
    return torch.empty((n, m), dtype=dtype or torch.float32, device=device).t()


def colmajor(x):
    """Column-major copy of a 2-D tensor (no copy if already column-major)."""
    if x.dim() == 2 and (x.stride(0) == 1 or x.shape[1] <= 1):
        return x
    return x.t().contiguous().t()


def _stream(stream):
    torch = _torch()
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


# ---- the ABI, one Python function per C entry point (same names) ------------
def caqr_workspace_bytes(m: int, n: int, dtype: int = CAQR_F32, opts: Optional[Opts] = None) -> int:
    return int(lib().caqr_workspace_bytes(m, n, dtype, _optp(opts)))


def caqr_plan_info(m: int, n: int, dtype: int = CAQR_F32, opts: Optional[Opts] = None) -> dict:
    out = (ctypes.c_int64 * 8)()
    _check("caqr_plan_info", lib().caqr_plan_info(m, n, dtype, _optp(opts), out))
    keys = ["leaf_rows", "panel_cols", "groups", "leaves", "tree_levels", "panels", "launches", "chains"]
    return {k: int(out[i]) for i, k in enumerate(keys)}


def caqr_tune(A, reps: int = 3, stream=None):
    """Plan search on the column-major CUDA matrix A (left unchanged).  Returns
    (opts or None for the default plan, best_ms, default_ms, plans_tried)."""
    code, _ = _dtype_code(A)
    m, n = A.shape
    pa, lda = _colmajor(A, "A")
    best = Opts()
    bms, dms, nt = ctypes.c_float(), ctypes.c_float(), ctypes.c_int()
    _check("caqr_tune", lib().caqr_tune(m, n, code, pa, lda, reps, ctypes.byref(best), ctypes.byref(bms),
                                        ctypes.byref(dms), ctypes.byref(nt), _stream(stream)))
    opts = best if (best.leaf_rows or best.panel_cols) else None
    return opts, float(bms.value), float(dms.value), int(nt.value)


def caqr_factor(A, R=None, ws=None, opts: Optional[Opts] = None, stream=None):
    """Factor A in place (column-major CUDA tensor).  Returns (R, ws): R is n x n
    (strict lower zero), ws the workspace holding T; A and ws are the implicit Q."""
    torch = _torch()
    code, suf = _dtype_code(A)
    m, n = A.shape
    pa, lda = _colmajor(A, "A")
    if R is None:
        R = colmajor_empty(n, n, A.dtype, A.device)
    pr, ldr = _colmajor(R, "R")
    need = caqr_workspace_bytes(m, n, code, opts)
    if need == 0 and n > 0:
        raise CaqrError("caqr_workspace_bytes", -2, "illegal size/opts")
    if ws is None:
        ws = torch.empty(max(need, 1), dtype=torch.uint8, device=A.device)
    info = getattr(lib(), f"caqr_factor_{suf}")(m, n, pa, lda, pr, ldr, ws.data_ptr(), ws.numel(),
                                                 _optp(opts), _stream(stream))
    _check(f"caqr_factor_{suf}", info)
    return R, ws


def caqr_factor_host_workspace_bytes(m: int, n: int, chunks: int, dtype: int = CAQR_F32,
                                     opts: Optional[Opts] = None) -> int:
    return int(lib().caqr_factor_host_workspace_bytes(m, n, chunks, dtype, _optp(opts)))


def caqr_factor_host_layout(m: int, n: int, chunks: int, c: int, dtype: int = CAQR_F32,
                            opts: Optional[Opts] = None) -> Tuple[int, int, int]:
    out = (ctypes.c_int64 * 3)()
    _check("caqr_factor_host_layout", lib().caqr_factor_host_layout(m, n, chunks, dtype, _optp(opts), c, out))
    return int(out[0]), int(out[1]), int(out[2])


def caqr_factor_host(A_host, chunks: int, A=None, R=None, ws=None, opts: Optional[Opts] = None, stream=None):
    """Factor a column-major HOST matrix (pinned for overlap): chunked H2D copies
    overlapped with the chunks' factorisations, then the combine.  Returns
    (A, R, ws) on the device (A/ws: the chunked implicit Q, see caqr.h)."""
    torch = _torch()
    if A_host.is_cuda:
        raise ValueError("A_host must be a host tensor")
    code, suf = _dtype_code(A_host)
    m, n = A_host.shape
    ph, ldh = _colmajor(A_host, "A_host", host=True)
    if A is None:
        A = colmajor_empty(m, n, A_host.dtype, "cuda")
    pa, lda = _colmajor(A, "A")
    if R is None:
        R = colmajor_empty(n, n, A_host.dtype, A.device)
    pr, ldr = _colmajor(R, "R")
    need = caqr_factor_host_workspace_bytes(m, n, chunks, code, opts)
    if need == 0 and n > 0:
        raise CaqrError("caqr_factor_host_workspace_bytes", -3, "illegal size/chunks/opts")
    if ws is None:
        ws = torch.empty(max(need, 1), dtype=torch.uint8, device=A.device)
    info = getattr(lib(), f"caqr_factor_host_{suf}")(m, n, chunks, ph, ldh, pa, lda, pr, ldr, ws.data_ptr(),
                                                      ws.numel(), _optp(opts), _stream(stream))
    _check(f"caqr_factor_host_{suf}", info)
    return A, R, ws


def _apply(name, A, ws, C, n, opts, stream):
    code, suf = _dtype_code(A)
    m = A.shape[0]
    pa, lda = _colmajor(A, "A")
    pc, ldc = _colmajor(C, "C")
    if C.shape[0] != m:
        raise ValueError("C must have as many rows as A")
    info = getattr(lib(), f"caqr_{name}_{suf}")(m, n, pa, lda, ws.data_ptr(), C.shape[1], pc, ldc,
                                                 _optp(opts), _stream(stream))
    _check(f"caqr_{name}_{suf}", info)
    return C


def caqr_apply_qt(A, ws, C, n=None, opts=None, stream=None):
    """C <- Q^T C in place (A, ws as left by caqr_factor)."""
    return _apply("apply_qt", A, ws, C, A.shape[1] if n is None else n, opts, stream)


def caqr_apply_q(A, ws, C, n=None, opts=None, stream=None):
    """C <- Q C in place."""
    return _apply("apply_q", A, ws, C, A.shape[1] if n is None else n, opts, stream)


def caqr_form_q(A, ws, Q=None, n=None, opts=None, stream=None):
    """Explicit thin Q (m x n), A_original = Q R."""
    code, suf = _dtype_code(A)
    m = A.shape[0]
    n = A.shape[1] if n is None else n
    pa, lda = _colmajor(A, "A")
    if Q is None:
        Q = colmajor_empty(m, n, A.dtype, A.device)
    pq, ldq = _colmajor(Q, "Q")
    info = getattr(lib(), f"caqr_form_q_{suf}")(m, n, pa, lda, ws.data_ptr(), pq, ldq, _optp(opts),
                                                 _stream(stream))
    _check(f"caqr_form_q_{suf}", info)
    return Q


def caqr_lstsq(A, ws, B, n=None, opts=None, stream=None):
    """Least squares (xGELS): B (m x k) <- Q^T B, then B[:n] <- R^{-1} B[:n] = argmin ||A X - B||.
    Returns B; B[:n] is the solution, column norms of B[n:] the residual norms."""
    return _apply("lstsq", A, ws, B, A.shape[1] if n is None else n, opts, stream)


def caqr_set_identity(Q, stream=None):
    """Q (m x n) = [I_n; 0] on the device."""
    code, suf = _dtype_code(Q)
    pq, ldq = _colmajor(Q, "Q")
    _check(f"caqr_set_identity_{suf}", getattr(lib(), f"caqr_set_identity_{suf}")(Q.shape[0], Q.shape[1], pq, ldq,
                                                                                  _stream(stream)))
    return Q


def caqr_trsm_upper(R, B, stream=None):
    """B (n x k) <- R^{-1} B for upper-triangular R (n x n), on the device."""
    code, suf = _dtype_code(R)
    pr, ldr = _colmajor(R, "R")
    pb, ldb = _colmajor(B, "B")
    _check(f"caqr_trsm_upper_{suf}", getattr(lib(), f"caqr_trsm_upper_{suf}")(R.shape[0], B.shape[1], pr, ldr, pb,
                                                                              ldb, _stream(stream)))
    return B


def caqr_combine_workspace_bytes(P: int, n: int, dtype: int = CAQR_F32) -> int:
    return int(lib().caqr_combine_workspace_bytes(P, n, dtype))


def caqr_combine(Rstack, P: int, R=None, ws=None, stream=None):
    """Combine P stacked n x n R factors ((P*n) x n column-major, modified in
    place) into one R.  Returns (R, ws)."""
    torch = _torch()
    code, suf = _dtype_code(Rstack)
    n = Rstack.shape[1]
    ps, ld = _colmajor(Rstack, "Rstack")
    if R is None:
        R = colmajor_empty(n, n, Rstack.dtype, Rstack.device)
    pr, ldr = _colmajor(R, "R")
    need = caqr_combine_workspace_bytes(P, n, code)
    if ws is None:
        ws = torch.empty(max(need, 1), dtype=torch.uint8, device=Rstack.device)
    info = getattr(lib(), f"caqr_combine_{suf}")(P, n, ps, ld, pr, ldr, ws.data_ptr(), ws.numel(),
                                                  _stream(stream))
    _check(f"caqr_combine_{suf}", info)
    return R, ws


def caqr_combine_apply(Rstack, P: int, ws, C, trans: bool = True, stream=None):
    code, suf = _dtype_code(Rstack)
    n = Rstack.shape[1]
    ps, ld = _colmajor(Rstack, "Rstack")
    pc, ldc = _colmajor(C, "C")
    info = getattr(lib(), f"caqr_combine_apply_{suf}")(P, n, ps, ld, ws.data_ptr(), int(trans),
                                                        C.shape[1], pc, ldc, _stream(stream))
    _check(f"caqr_combine_apply_{suf}", info)
    return C


def caqr_dist_combine_blocks(blocks, P: int, n: int, gather=None, R=None, cws=None, stream=None):
    """The post-exchange half of the distributed factor (caqr_dist_combine_blocks_*):
    `blocks` holds P contiguous column-major n x n R factors (rank order, e.g. an
    all-gather's receive buffer, P*n*n elements); returns (R, gather, cws) with
    the combined R, the combine's tree vectors and its workspace."""
    torch = _torch()
    code, suf = _dtype_code(blocks)
    if blocks.numel() < P * n * n or not blocks.is_contiguous():
        raise ValueError("blocks: P*n*n contiguous elements")
    if gather is None:
        gather = colmajor_empty(P * n, n, blocks.dtype, blocks.device)
    pg, ldg = _colmajor(gather, "gather")
    if R is None:
        R = colmajor_empty(n, n, blocks.dtype, blocks.device)
    pr, ldr = _colmajor(R, "R")
    if cws is None:
        cws = torch.empty(max(caqr_combine_workspace_bytes(P, n, code), 1), dtype=torch.uint8, device=blocks.device)
    info = getattr(lib(), f"caqr_dist_combine_blocks_{suf}")(P, n, blocks.data_ptr(), pg, ldg, pr, ldr,
                                                               cws.data_ptr(), cws.numel(), _stream(stream))
    _check(f"caqr_dist_combine_blocks_{suf}", info)
    return R, gather, cws


def caqr_peer_mailbox_bytes(P: int, n: int, dtype_code: int) -> int:
    return int(lib().caqr_peer_mailbox_bytes(P, n, dtype_code))


def _ptr_array(ptrs, device):
    """Device array of raw device pointers (int64), for the pointer-array arguments."""
    torch = _torch()
    return torch.tensor([int(p) for p in ptrs], dtype=torch.int64, device=device)


def caqr_peer_exchange(P: int, rank: int, R, peer_mailbox, peer_flags, gather, epoch: int, status=None,
                       timeout_ms: int = 0, stream=None):
    """caqr_peer_exchange_*: this rank's R into every rank's mailbox (peer
    stores), flags, and the P blocks restacked into `gather` ((P n) x n).
    peer_mailbox / peer_flags: int64 device tensors of P device pointers."""
    code, suf = _dtype_code(R)
    n = R.shape[1]
    pr, ldr = _colmajor(R, "R")
    pg, _ = _colmajor(gather, "gather")
    info = getattr(lib(), f"caqr_peer_exchange_{suf}")(P, rank, n, pr, ldr, peer_mailbox.data_ptr(),
                                                        peer_flags.data_ptr(), pg, int(epoch),
                                                        status.data_ptr() if status is not None else None,
                                                        int(timeout_ms), _stream(stream))
    _check(f"caqr_peer_exchange_{suf}", info)
    return gather


def caqr_peer_exchange_emulate(Rs, mailboxes, flags, gathers, epoch: int, stream=None):
    """The exchange among len(Rs) virtual ranks on one device (tests): Rs,
    mailboxes, flags, gathers are per-rank tensors (same n, same ldr)."""
    P = len(Rs)
    code, suf = _dtype_code(Rs[0])
    n = Rs[0].shape[1]
    ldr = _colmajor(Rs[0], "R")[1]
    for r in Rs:
        if _colmajor(r, "R")[1] != ldr:
            raise ValueError("Rs: one leading dimension")
    dev = Rs[0].device
    arrs = [_ptr_array([t.data_ptr() for t in ts], dev) for ts in (Rs, mailboxes, flags, gathers)]
    info = getattr(lib(), f"caqr_peer_exchange_emulate_{suf}")(P, n, arrs[0].data_ptr(), ldr, arrs[1].data_ptr(),
                                                                arrs[2].data_ptr(), arrs[3].data_ptr(), int(epoch),
                                                                _stream(stream))
    _check(f"caqr_peer_exchange_emulate_{suf}", info)
    # the pointer arrays are temporaries: keep them alive until the launch ran
    (stream if stream is not None else _torch().cuda.current_stream(dev)).synchronize()
    return gathers


def caqr_ipc_handle(t) -> bytes:
    buf = ctypes.create_string_buffer(64)
    _check("caqr_ipc_handle", lib().caqr_ipc_handle(t.data_ptr(), buf))
    return buf.raw


def caqr_ipc_open(handle: bytes) -> int:
    p = ctypes.c_void_p()
    _check("caqr_ipc_open", lib().caqr_ipc_open(handle, ctypes.byref(p)))
    return int(p.value)


def caqr_ipc_close(ptr: int):
    _check("caqr_ipc_close", lib().caqr_ipc_close(ctypes.c_void_p(ptr)))


# ---- application layer: SVD via QR, robust PCA (include/caqr.h, Sec. VI) ----
CAQR_RPCA_RESID_LEN = 1025


def _f32(t, name):
    torch = _torch()
    if t.dtype != torch.float32:
        raise TypeError(f"caqr: {name} must be float32")
    return _colmajor(t, name)


def caqr_svd_small(R, U=None, sigma=None, V=None, stream=None, want_v: bool = True):
    """R (n x n) = U diag(sigma) V^T on the GPU (one-CTA Jacobi).  Returns (U, sigma, V);
    V is None when want_v is False (right vectors not formed)."""
    torch = _torch()
    code, suf = _dtype_code(R)
    n = R.shape[0]
    if R.shape[1] != n:
        raise ValueError("caqr_svd_small: R must be square")
    pr, ldr = _colmajor(R, "R")
    U = colmajor_empty(n, n, R.dtype, R.device) if U is None else U
    if want_v:
        V = colmajor_empty(n, n, R.dtype, R.device) if V is None else V
        pv, ldv = _colmajor(V, "V")
    else:
        V, pv, ldv = None, None, max(n, 1)
    sigma = torch.empty(n, dtype=R.dtype, device=R.device) if sigma is None else sigma
    pu, ldu = _colmajor(U, "U")
    info = getattr(lib(), f"caqr_svd_small_{suf}")(n, pr, ldr, pu, ldu, sigma.data_ptr(), pv, ldv,
                                                    _stream(stream))
    _check(f"caqr_svd_small_{suf}", info)
    return U, sigma, V


def caqr_svt_core(U, sigma, V, tau: float, W=None, stream=None):
    """W = U diag(max(sigma - tau, 0)) V^T (n x n)."""
    n = U.shape[0]
    pu, ldu = _f32(U, "U")
    pv, ldv = _f32(V, "V")
    W = colmajor_empty(n, n, U.dtype, U.device) if W is None else W
    pw, ldw = _f32(W, "W")
    _check("caqr_svt_core_f32", lib().caqr_svt_core_f32(n, pu, ldu, sigma.data_ptr(), pv, ldv, float(tau), pw,
                                                        ldw, _stream(stream)))
    return W


def caqr_svt_core_r(U, sigma, R, tau: float, W=None, stream=None):
    """W = U diag(max(sigma - tau, 0) / sigma) U^T R (= U diag(max(sigma - tau, 0)) V^T)."""
    n = U.shape[0]
    pu, ldu = _f32(U, "U")
    pr, ldr = _f32(R, "R")
    W = colmajor_empty(n, n, U.dtype, U.device) if W is None else W
    pw, ldw = _f32(W, "W")
    _check("caqr_svt_core_r_f32", lib().caqr_svt_core_r_f32(n, pu, ldu, sigma.data_ptr(), pr, ldr, float(tau), pw,
                                                            ldw, _stream(stream)))
    return W


def caqr_embed_top(W, C, stream=None):
    """C = [W; 0]."""
    pw, ldw = _f32(W, "W")
    pc, ldc = _f32(C, "C")
    _check("caqr_embed_top_f32", lib().caqr_embed_top_f32(C.shape[0], W.shape[0], pw, ldw, pc, ldc,
                                                          _stream(stream)))
    return C


def caqr_rpca_update(M, L, S, Y, X, mu: float, mu_next: float, lam: float, resid, stream=None):
    m, n = M.shape
    args = []
    for t, nm in ((M, "M"), (L, "L"), (S, "S"), (Y, "Y"), (X, "X")):
        args += list(_f32(t, nm))
    _check("caqr_rpca_update_f32", lib().caqr_rpca_update_f32(m, n, *args, float(mu), float(mu_next), float(lam),
                                                              resid.data_ptr(), _stream(stream)))


def caqr_rpca_init(M, yscale: float, S, Y, X, mu: float, stream=None):
    m, n = M.shape
    pm, ldm = _f32(M, "M")
    ps, lds = _f32(S, "S")
    py, ldy = _f32(Y, "Y")
    px, ldx = _f32(X, "X")
    _check("caqr_rpca_init_f32", lib().caqr_rpca_init_f32(m, n, pm, ldm, float(yscale), ps, lds, py, ldy, px, ldx,
                                                          float(mu), _stream(stream)))


CAQR_RPCA_SCHED_LEN = 8


def caqr_rpca_schedule(sigma, amax, lam: float, mu_factor: float, mu_max_factor: float, rho: float, sched,
                       stream=None):
    """sched (device float64[8]) <- mu, mu_max, rho, yscale, lambda from sigma[0] and amax[0]."""
    _check("caqr_rpca_schedule_f32", lib().caqr_rpca_schedule_f32(sigma.data_ptr(), amax.data_ptr(), float(lam),
                                                                  float(mu_factor), float(mu_max_factor),
                                                                  float(rho), sched.data_ptr(), _stream(stream)))
    return sched


def caqr_rpca_init_sched(M, sched, S, Y, X, stream=None):
    m, n = M.shape
    pm, ldm = _f32(M, "M")
    ps, lds = _f32(S, "S")
    py, ldy = _f32(Y, "Y")
    px, ldx = _f32(X, "X")
    _check("caqr_rpca_init_sched_f32", lib().caqr_rpca_init_sched_f32(m, n, pm, ldm, sched.data_ptr(), ps, lds, py,
                                                                      ldy, px, ldx, _stream(stream)))


def caqr_svt_core_r_sched(U, sigma, R, sched, W=None, stream=None):
    n = U.shape[0]
    pu, ldu = _f32(U, "U")
    pr, ldr = _f32(R, "R")
    W = colmajor_empty(n, n, U.dtype, U.device) if W is None else W
    pw, ldw = _f32(W, "W")
    _check("caqr_svt_core_r_sched_f32", lib().caqr_svt_core_r_sched_f32(n, pu, ldu, sigma.data_ptr(), pr, ldr,
                                                                        sched.data_ptr(), pw, ldw, _stream(stream)))
    return W


def caqr_rpca_update_sched(M, L, S, Y, X, sched, resid, stream=None):
    m, n = M.shape
    args = []
    for t, nm in ((M, "M"), (L, "L"), (S, "S"), (Y, "Y"), (X, "X")):
        args += list(_f32(t, nm))
    _check("caqr_rpca_update_sched_f32", lib().caqr_rpca_update_sched_f32(m, n, *args, sched.data_ptr(),
                                                                          resid.data_ptr(), _stream(stream)))


def caqr_absmax(M, out, stream=None):
    pm, ldm = _f32(M, "M")
    _check("caqr_absmax_f32", lib().caqr_absmax_f32(M.shape[0], M.shape[1], pm, ldm, out.data_ptr(),
                                                    _stream(stream)))
    return out


def geqrf_flops(m: int, n: int) -> float:
    """LAPACK count 2 m n^2 - 2 n^3 / 3 (the BASELINE metric's flop count)."""
    return 2.0 * m * n * n - 2.0 * n ** 3 / 3.0


# ---- launch tracing (profiling aid) -----------------------------------------
def caqr_trace_begin(capacity: int = 1 << 16) -> None:
    _check("caqr_trace_begin", lib().caqr_trace_begin(capacity))


def caqr_trace_end(capacity: int = 1 << 16):
    """Stop tracing; return a list of (kernel_name, ms, flops, bytes), one per launch."""
    L = lib()
    ids = (ctypes.c_int * capacity)()
    ms = (ctypes.c_float * capacity)()
    fl = (ctypes.c_double * capacity)()
    by = (ctypes.c_double * capacity)()
    n = L.caqr_trace_end(ids, ms, fl, by, capacity)
    n = min(n, capacity)
    return [(L.caqr_kernel_name(ids[i]).decode(), float(ms[i]), float(fl[i]), float(by[i]))
            for i in range(n)]
