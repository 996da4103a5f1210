"""Robust PCA on the GPU through CAQR (the paper's Sec. VI application).

M (m x n, one video frame per column) = L (low rank, the
background) + S (sparse, the foreground), by the alternating-directions
iteration the paper uses (Fig. 11; its parameters: DESIGN.md
reading S19).  Every iteration:

  1. X = M - S + Y/mu is QR-factored in place by CAQR (caqr_factor_f32): X -> the
     implicit Q, R (n x n)
  2. SVD of the small R on one CTA (caqr_svd_small_f32; U, sigma only)
  3. W = U diag(max(sigma - 1/mu, 0)) V^T, formed as U diag((sigma - 1/mu)+ / sigma) U^T R
     (caqr_svt_core_r_f32)                                    (Fig. 11 threshold)
  4. L = Q [W; 0] (caqr_embed_top_f32 + caqr_apply_q_f32): the left singular
     vectors Q U of X times the thresholded spectrum
  5. S = shrink(M - L + Y/mu, lambda/mu); Y += mu (M - L - S); the next X
     (caqr_rpca_update_f32, one fused pass)

This module only allocates buffers; every arithmetic step, the scalar schedule
(mu, mu_max, rho, lambda: caqr_rpca_schedule_f32 and the *_sched_f32 kernels)
included, runs in libcaqr on the device.  There is no CPU path.
"""
from __future__ import annotations

import math

from . import caqr


class RobustPCA:
    def __init__(self, M, rho: float = 1.5, mu_factor: float = 1.25, mu_max_factor: float = 1e7, opts=None,
                 stream=None):
        import torch

        if M.dtype != torch.float32 or not M.is_cuda:
            raise TypeError("RobustPCA: M must be a float32 CUDA tensor")
        m, n = M.shape
        if n > 112 or n > m:
            raise ValueError("RobustPCA: needs n <= min(m, 112)")
        self.m, self.n, self.opts, self.stream = m, n, opts, stream
        dev = M.device
        self.M = caqr.colmajor(M)
        e = lambda r, c: caqr.colmajor_empty(r, c, torch.float32, dev)  # noqa: E731
        self.X, self.L, self.S, self.Y = e(m, n), e(m, n), e(m, n), e(m, n)
        self.R, self.U, self.W = e(n, n), e(n, n), e(n, n)
        self.sigma = torch.empty(n, dtype=torch.float32, device=dev)
        self.ws = torch.empty(max(caqr.caqr_workspace_bytes(m, n, caqr.CAQR_F32, opts), 1), dtype=torch.uint8,
                              device=dev)
        self.resid = torch.zeros(caqr.CAQR_RPCA_RESID_LEN, dtype=torch.float64, device=dev)
        self.amax = torch.zeros(1, dtype=torch.float32, device=dev)
        # the scalar schedule lives on the device (mu, mu_max, rho, yscale, lambda):
        # no step needs a host round trip
        self.sched = torch.zeros(caqr.CAQR_RPCA_SCHED_LEN, dtype=torch.float64, device=dev)
        # ||M||_2 through the same QR + small SVD, ||M||_inf by a max reduction
        self.X.copy_(self.M)
        caqr.caqr_factor(self.X, R=self.R, ws=self.ws, opts=opts, stream=stream)
        caqr.caqr_svd_small(self.R, self.U, self.sigma, stream=stream, want_v=False)
        caqr.caqr_absmax(self.M, self.amax, stream=stream)
        caqr.caqr_rpca_schedule(self.sigma, self.amax, 1.0 / math.sqrt(max(m, n)), mu_factor, mu_max_factor, rho,
                                self.sched, stream=stream)
        caqr.caqr_rpca_init_sched(self.M, self.sched, self.S, self.Y, self.X, stream=stream)
        self.iters = 0

    # schedule entries (reading them synchronises; setting them is a device write)
    def _get(self, i: int) -> float:
        import torch

        (self.stream or torch.cuda.current_stream()).synchronize()
        return float(self.sched[i].item())

    def _set(self, i: int, v: float):
        import torch

        with torch.cuda.stream(self.stream or torch.cuda.current_stream()):
            self.sched[i:i + 1].fill_(float(v))

    mu = property(lambda self: self._get(0), lambda self, v: self._set(0, v))
    mu_max = property(lambda self: self._get(1), lambda self, v: self._set(1, v))
    rho = property(lambda self: self._get(2), lambda self, v: self._set(2, v))
    lam = property(lambda self: self._get(4), lambda self, v: self._set(4, v))

    def load_state(self, S, Y, X, mu: float):
        """Set the iteration state (S, Y, the SVT input X = M - S + Y/mu, mu):
        tests start the GPU path and the oracle from the same state."""
        self.S.copy_(S)
        self.Y.copy_(Y)
        self.X.copy_(X)
        self.mu = mu

    def step(self):
        """One iteration; returns nothing (no host synchronisation, no host scalar)."""
        s, o = self.stream, self.opts
        caqr.caqr_factor(self.X, R=self.R, ws=self.ws, opts=o, stream=s)
        caqr.caqr_svd_small(self.R, self.U, self.sigma, stream=s, want_v=False)
        caqr.caqr_svt_core_r_sched(self.U, self.sigma, self.R, self.sched, self.W, stream=s)
        caqr.caqr_embed_top(self.W, self.L, stream=s)
        caqr.caqr_apply_q(self.X, self.ws, self.L, opts=o, stream=s)
        caqr.caqr_rpca_update_sched(self.M, self.L, self.S, self.Y, self.X, self.sched, self.resid, stream=s)
        self.iters += 1

    def residual(self) -> float:
        """||M - L - S||_F after the last step (synchronises)."""
        return math.sqrt(float(self.resid[0].item()))
