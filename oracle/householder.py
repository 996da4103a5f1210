"""ctypes binding of oracle/householder.c -- TEST INFRASTRUCTURE ONLY.

Every function takes/returns float64 numpy arrays (an fp32 input converts to
float64 exactly).  ``acc`` picks the accumulation type of the C routine:
``"d"`` (double; for fp32 inputs), ``"ld"`` (x87 long double; for fp64 inputs)
or ``"f"`` (float; calibration only).  See householder.c for the paper passages
each routine follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "householder.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

# Deterministic reference build.
CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-fPIC", "-shared", "-std=c99"]


def build(force: bool = False) -> str:
    """Compile householder.c -> liboracle.so with gcc (no GPU, no CUDA)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            i64, dp, ip = ctypes.c_int64, ctypes.POINTER(ctypes.c_double), ctypes.c_int
            for suf in ("d", "ld", "f"):
                f = getattr(lib, f"oracle_geqr2_{suf}")
                f.argtypes = [i64, i64, dp, i64, dp]
                f.restype = ip
                f = getattr(lib, f"oracle_orm2r_{suf}")
                f.argtypes = [ip, i64, i64, i64, dp, i64, dp, dp, i64]
                f.restype = ip
                f = getattr(lib, f"oracle_qr_{suf}")
                f.argtypes = [i64, i64, dp, i64, dp, i64, dp, i64]
                f.restype = ip
            lib.oracle_geqrf_flops.argtypes = [i64, i64]
            lib.oracle_geqrf_flops.restype = ctypes.c_double
            _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _f64_fortran(a) -> np.ndarray:
    return np.asfortranarray(np.asarray(a, dtype=np.float64))


def geqr2(A, acc: str = "d"):
    """Householder QR in place (LAPACK xGEQR2).  Returns (VR, tau): R on and
    above the diagonal, v_j below it (unit head implicit)."""
    VR = _f64_fortran(A).copy(order="F")
    m, n = VR.shape
    tau = np.zeros(max(min(m, n), 1))
    rc = getattr(_load(), f"oracle_geqr2_{acc}")(m, n, _ptr(VR), max(m, 1), _ptr(tau))
    if rc != 0:
        raise ValueError(f"oracle_geqr2_{acc} failed: {rc}")
    return VR, tau[: min(m, n)]


def orm2r(VR, tau, C, trans: bool = True, acc: str = "d"):
    """C <- Q^T C (trans) or Q C, Q = H_0 ... H_{k-1} from geqr2's output."""
    VR = _f64_fortran(VR)
    Cw = _f64_fortran(C).copy(order="F")
    if Cw.ndim == 1:
        Cw = Cw.reshape(-1, 1, order="F")
    m = VR.shape[0]
    k = len(tau)
    nc = Cw.shape[1]
    t = np.ascontiguousarray(np.asarray(tau, dtype=np.float64))
    if k == 0:
        return Cw
    rc = getattr(_load(), f"oracle_orm2r_{acc}")(int(trans), m, nc, k, _ptr(VR), max(m, 1),
                                                   _ptr(t), _ptr(Cw), max(m, 1))
    if rc != 0:
        raise ValueError(f"oracle_orm2r_{acc} failed: {rc}")
    return Cw


def qr(A, want_q: bool = True, acc: str = "d"):
    """R (n x n, strict lower zeroed) and optionally the thin Q (m x n) of A
    (m >= n), both as the Householder process leaves them (R_jj may be < 0)."""
    Aw = _f64_fortran(A)
    m, n = Aw.shape
    if n > m:
        raise ValueError("oracle.qr needs m >= n")
    R = np.zeros((n, n), order="F")
    Q = np.zeros((m, n), order="F") if want_q else None
    rc = getattr(_load(), f"oracle_qr_{acc}")(
        m, n, _ptr(Aw), max(m, 1), _ptr(R), max(n, 1),
        _ptr(Q) if want_q else ctypes.POINTER(ctypes.c_double)(), max(m, 1))
    if rc != 0:
        raise ValueError(f"oracle_qr_{acc} failed: {rc}")
    return (R, Q) if want_q else R


def normalize_signs(R, Q=None):
    """D = diag(sign(R_jj)), sign(0) = +1; R <- D R, Q <- Q D.
    Makes R unique for full-rank A (R^T R = A^T A, positive diagonal)."""
    R = np.array(R, dtype=np.float64, copy=True)
    d = np.where(np.diag(R) < 0, -1.0, 1.0)
    R = d[:, None] * R
    if Q is None:
        return R
    Q = np.array(Q, dtype=np.float64, copy=True) * d[None, :]
    return R, Q


def geqrf_flops(m: int, n: int) -> float:
    """LAPACK xGEQRF count 2 m n^2 - 2 n^3 / 3 (BASELINE.json metric)."""
    return float(_load().oracle_geqrf_flops(int(m), int(n)))
