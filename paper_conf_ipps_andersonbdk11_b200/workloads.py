"""Seeded synthetic inputs shaped like the paper's workloads.

This module is the ONLY code shared by the oracle side (tests, bench cpu
baseline) and the CUDA side: it draws random numbers and builds the matrices
to factor, and holds none of the QR method's arithmetic.

Workloads (BASELINE.json "configs"; recipes in DESIGN.md "Inputs"):
  gaussian      N(0,1) entries (1M x 192 headline, 4096 x 16, 8192^2)
  krylov_basis  s-step Krylov basis {v, Lv, ..., L^{s-1} v} of the 2-D 5-point
                Laplacian, each column normalised ("s-step methods ...
                millions of rows by less than ten columns")
  video         Robust-PCA video matrix, one column per 288x384 frame
                (P:L1050-1054), static background x slow
                illumination, a moving elliptical foreground blob, small noise

Host generators use numpy.random.default_rng(seed) (PCG64) in float64 and
round to the target dtype.  `device_gaussian` draws on the GPU with a seeded
torch.Generator for sizes too large to build on the host every bench run.
"""
from __future__ import annotations

import numpy as np

VIDEO_H, VIDEO_W, VIDEO_FRAMES = 288, 384, 100  # 110,592 pixels x 100 frames


def _as(a: np.ndarray, dtype) -> np.ndarray:
    return np.asfortranarray(a.astype(dtype))


def gaussian(m: int, n: int, seed: int = 0, dtype=np.float32) -> np.ndarray:
    """m x n, entries N(0,1) drawn in float64 then rounded; column-major."""
    rng = np.random.default_rng(seed)
    return _as(rng.standard_normal((m, n)), dtype)


def laplacian_2d_apply(v: np.ndarray, g: int) -> np.ndarray:
    """y = L v for the 5-point Laplacian on a g x g grid, Dirichlet boundary
    (L = 4I - shifts).  Input generator only; not part of the QR method."""
    x = v.reshape(g, g)
    y = 4.0 * x
    y[1:, :] -= x[:-1, :]
    y[:-1, :] -= x[1:, :]
    y[:, 1:] -= x[:, :-1]
    y[:, :-1] -= x[:, 1:]
    return y.reshape(-1)


def krylov_basis(grid: int = 2000, s: int = 8, seed: int = 0, shifted: bool = False,
                 dtype=np.float32) -> np.ndarray:
    """(grid^2) x s matrix [v, Lv, ..., L^{s-1} v] with v ~ N(0,1) and each
    column normalised to unit 2-norm (monomial basis, kappa ~ 7e4 at s = 8), or
    with the shifted operator (L - 4I)/4 (kappa ~ 1e2).  grid = 2000 gives the
    4,000,000 x 8 configuration."""
    rng = np.random.default_rng(seed)
    m = grid * grid
    w = rng.standard_normal(m)
    out = np.empty((m, s), dtype=np.float64, order="F")
    for j in range(s):
        w = w / np.linalg.norm(w)
        out[:, j] = w
        if j + 1 < s:
            w = laplacian_2d_apply(w, grid)
            if shifted:
                w = (w - 4.0 * out[:, j]) / 4.0  # ((L - 4I)/4) applied to the unit column j
    return _as(out, dtype)


def video(frames: int = VIDEO_FRAMES, h: int = VIDEO_H, w: int = VIDEO_W, seed: int = 0,
          dtype=np.float32) -> np.ndarray:
    """(h*w) x frames video matrix for Robust PCA background subtraction.

    Background U(0.2, 0.8) times illumination 1 + 0.05 sin(3 f / 99); an
    elliptical blob (about 2-5 % of the pixels) moves across the frame and adds
    U(-0.5, 0.5) offsets; N(0, 0.01^2) noise; clipped to [0, 1]."""
    rng = np.random.default_rng(seed)
    bg = rng.uniform(0.2, 0.8, size=(h, w))
    blob_off = rng.uniform(-0.5, 0.5, size=(h, w))
    yy, xx = np.mgrid[0:h, 0:w]
    ry, rx = 0.12 * h, 0.10 * w
    out = np.empty((h * w, frames), dtype=np.float64, order="F")
    for f in range(frames):
        illum = 1.0 + 0.05 * np.sin(3.0 * f / 99.0)
        cy = h * (0.3 + 0.4 * f / max(frames - 1, 1))
        cx = w * (0.1 + 0.8 * f / max(frames - 1, 1))
        inside = ((yy - cy) / ry) ** 2 + ((xx - cx) / rx) ** 2 <= 1.0
        frame = bg * illum + np.where(inside, blob_off, 0.0)
        frame = frame + rng.normal(0.0, 0.01, size=(h, w))
        out[:, f] = np.clip(frame, 0.0, 1.0).reshape(-1)
    return _as(out, dtype)


def device_gaussian(m: int, n: int, seed: int, dtype, device):
    """Seeded N(0,1) m x n column-major matrix drawn on `device` (torch);
    returned as a torch tensor of shape (n, m) whose row c is column c of A
    (i.e. the column-major buffer of A with lda = m)."""
    import torch

    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return torch.randn((n, m), generator=g, device=device, dtype=dtype)


# BASELINE.json "configs" -> concrete synthetic workloads.
CONFIGS = {
    "c1_4096x16_f32": dict(kind="gaussian", m=4096, n=16, dtype="f32"),
    "c2_krylov_4Mx8_f32": dict(kind="krylov", m=4_000_000, n=8, dtype="f32"),
    "c3_video_110592x100_f32": dict(kind="video", m=110_592, n=100, dtype="f32", reps=100),
    "c4_1Mx192_f32": dict(kind="gaussian", m=1_000_000, n=192, dtype="f32"),
    "c4_1Mx192_f64": dict(kind="gaussian", m=1_000_000, n=192, dtype="f64"),
    "c4p_8Mx192_f32": dict(kind="gaussian", m=8_000_000, n=192, dtype="f32"),
    "c5_8192x8192_f32": dict(kind="gaussian", m=8192, n=8192, dtype="f32", nb=64),
}
