"""C-ABI checks that need no GPU: the library builds, loads, exports every
symbol include/caqr.h declares, and its host-side planner / argument checks
behave as documented (LAPACK info codes, workspace sizes)."""
import ctypes

import pytest

from paper_conf_ipps_andersonbdk11_b200 import build as cbuild
from paper_conf_ipps_andersonbdk11_b200 import caqr


@pytest.fixture(scope="module")
def L():
    cbuild.build()
    return caqr.lib()


def test_exports_every_header_symbol(L):
    names = caqr.header_functions()
    assert len(names) >= 20
    missing = [n for n in names if not hasattr(L, n)]
    assert not missing, missing


def test_build_info(L):
    assert b"sm_100a" in L.caqr_build_info()


def test_sass_is_sm100a():
    import subprocess

    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", caqr.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_workspace_bytes(L):
    # one T block (32x32) per (tile, panel) and per (merge, panel), the merges indexed
    # by their right member's slot (< P chains): (L + P)*npan*1024 elems, plus the
    # fused kernel's ticket + (slot, panel) flags: (32 + L*npan) ints, 256-B rounded
    def ws(L, npan, es, P=None):
        P = L if P is None else P
        return (L + P) * npan * 1024 * es + -(-(32 + L * npan) * 4 // 256) * 256
    # default tile height 224 (n <= 224): 4096 rows -> 19 tiles, 1M rows -> 4465 tiles;
    # skinny fp32 (n <= 16, m >= 1024: the warp-per-chain streaming kernel) uses
    # 256 (n <= 8) / 128-row tiles and a cross-CTA exchange area in the flag
    # area: 64 ints + one n x n R per CTA of 8 chains (32-int aligned) + 16
    # counters per CTA: 4096 x 16 -> 32 tiles, 4 CTAs
    nct = 4
    sync = max(32 + 32, 64 + ((nct * 16 * 16 + 31) & ~31) + 16 * nct)
    assert caqr.caqr_workspace_bytes(4096, 16) == 2 * 32 * 1024 * 4 + -(-sync * 4 // 256) * 256
    assert caqr.caqr_workspace_bytes(4096, 16, caqr.CAQR_F64) == ws(19, 1, 8)
    assert caqr.caqr_workspace_bytes(1_000_000, 192) == ws(4465, 6, 4, P=280)  # chains of 16 tiles
    assert caqr.caqr_workspace_bytes(4096, 16, 0, caqr.make_opts(leaf_rows=256)) == ws(16, 1, 4)
    assert caqr.caqr_workspace_bytes(10, 11) == 0  # n > m
    assert caqr.caqr_workspace_bytes(-1, 1) == 0
    assert caqr.caqr_workspace_bytes(10, 2, 7) == 0  # bad dtype
    assert caqr.caqr_workspace_bytes(100, 8, 0, caqr.make_opts(leaf_rows=100)) == 0  # not /32


def test_plan_info(L):
    p = caqr.caqr_plan_info(1_000_000, 192)
    assert p["leaf_rows"] == 224 and p["panel_cols"] == 192 and p["groups"] == 1
    # 4465 tiles in chains of K = ceil(4465/296) = 16 -> 280 chains -> 9 tree levels
    assert p["leaves"] == 4465 and p["chains"] == 280 and p["tree_levels"] == 9 and p["panels"] == 6
    assert p["launches"] == 2  # one fused TSQR kernel + extract_r
    p = caqr.caqr_plan_info(8192, 8192)
    assert p["panel_cols"] == 128 and p["groups"] == 64 and p["leaf_rows"] == 256  # wide: (b, nb) = (256, 128)
    p = caqr.caqr_plan_info(4096, 16, 0, caqr.make_opts(leaf_rows=128))
    assert p["leaf_rows"] == 128 and p["leaves"] == 32 and p["tree_levels"] == 5
    p = caqr.caqr_plan_info(4_000_000, 8)  # skinny: 256-row tiles, ~2368 chains (16 warps x 148 SMs)
    assert p["leaf_rows"] == 256 and p["leaves"] == 15625 and p["chains"] == 2233 and p["launches"] == 2


def test_info_codes_without_gpu(L):
    """Illegal arguments are rejected before any CUDA call (LAPACK info)."""
    vp = ctypes.c_void_p
    f = L.caqr_factor_f32
    null = None
    assert f(-1, 1, vp(8), 1, vp(8), 1, vp(8), 1 << 20, null, null) == -1
    assert f(4, 5, vp(8), 4, vp(8), 5, vp(8), 1 << 20, null, null) == -2
    assert f(4, 2, null, 4, vp(8), 2, vp(8), 1 << 20, null, null) == -3
    assert f(4, 2, vp(8), 3, vp(8), 2, vp(8), 1 << 20, null, null) == -4
    assert f(4, 2, vp(8), 4, null, 2, vp(8), 1 << 20, null, null) == -5
    assert f(4, 2, vp(8), 4, vp(8), 1, vp(8), 1 << 20, null, null) == -6
    assert f(4, 2, vp(8), 4, vp(8), 2, null, 1 << 20, null, null) == -7
    assert f(4, 2, vp(8), 4, vp(8), 2, vp(8), 1, null, null) == -8
    bad = caqr.Opts(100, 0)
    assert f(4, 2, vp(8), 4, vp(8), 2, vp(8), 1 << 20, ctypes.byref(bad), null) == -9
    # quick return
    assert f(0, 0, vp(8), 1, vp(8), 1, null, 0, null, null) == 0
    g = L.caqr_apply_qt_f32
    assert g(4, 2, vp(8), 4, vp(8), -1, vp(8), 4, null, null) == -6
    assert g(4, 2, vp(8), 4, vp(8), 3, vp(8), 2, null, null) == -8
    h = L.caqr_form_q_f64
    assert h(4, 2, vp(8), 4, vp(8), vp(8), 3, null, null) == -7
    c = L.caqr_combine_f32
    assert c(0, 4, vp(8), 4, vp(8), 4, vp(8), 1 << 20, null) == -1
    assert c(2, 300, vp(8), 600, vp(8), 300, vp(8), 1 << 30, null) == -2
    assert L.caqr_strerror(-3) and L.caqr_strerror(1)
    # peer-memory R exchange (alternative to the NCCL all-gather)
    assert L.caqr_peer_mailbox_bytes(8, 192, caqr.CAQR_F32) == 2 * 8 * 192 * 192 * 4
    assert L.caqr_peer_mailbox_bytes(0, 192, caqr.CAQR_F32) == 0
    pe = L.caqr_peer_exchange_f32
    assert pe(0, 0, 8, vp(8), 8, vp(8), vp(8), vp(8), 1, null, 0, null) == -1
    assert pe(2, 2, 8, vp(8), 8, vp(8), vp(8), vp(8), 1, null, 0, null) == -2
    assert pe(2, 0, 300, vp(8), 300, vp(8), vp(8), vp(8), 1, null, 0, null) == -3
    assert pe(2, 0, 8, null, 8, vp(8), vp(8), vp(8), 1, null, 0, null) == -4
    assert pe(2, 0, 8, vp(8), 4, vp(8), vp(8), vp(8), 1, null, 0, null) == -5
    assert pe(2, 0, 8, vp(8), 8, null, vp(8), vp(8), 1, null, 0, null) == -6
    assert pe(2, 0, 8, vp(8), 8, vp(8), null, vp(8), 1, null, 0, null) == -7
    assert pe(2, 0, 8, vp(8), 8, vp(8), vp(8), null, 1, null, 0, null) == -8
    assert pe(2, 0, 8, vp(8), 8, vp(8), vp(8), vp(8), 0, null, 0, null) == -9
    assert pe(2, 0, 0, vp(8), 8, vp(8), vp(8), vp(8), 1, null, 0, null) == 0
    assert L.caqr_ipc_handle(null, vp(8)) == -1 and L.caqr_ipc_open(null, ctypes.byref(vp())) == -1


def test_info_codes_application_layer_without_gpu(L):
    """The f1 / f4 entry points validate their arguments (LAPACK info) before any
    CUDA call: robust-PCA kernels, small SVD, least squares, triangular solve."""
    vp = ctypes.c_void_p
    null = None
    one = vp(8)
    # caqr_svd_small_f32(n, R, ldr, U, ldu, sigma, V, ldv, stream)
    s = L.caqr_svd_small_f32
    assert s(113, one, 113, one, 113, one, one, 113, null) == -1  # n > 112
    assert s(-1, one, 1, one, 1, one, one, 1, null) == -1
    assert s(8, one, 7, one, 8, one, one, 8, null) == -3
    assert s(8, one, 8, one, 7, one, one, 8, null) == -5
    assert s(8, one, 8, one, 8, one, one, 7, null) == -8
    assert s(8, null, 8, one, 8, one, one, 8, null) == -2
    assert s(8, one, 8, one, 8, null, one, 8, null) == -6
    assert s(0, null, 1, null, 1, null, null, 1, null) == 0  # quick return
    # caqr_svt_core_f32(n, U, ldu, sigma, V, ldv, tau, W, ldw, stream)
    t = L.caqr_svt_core_f32
    assert t(4, one, 4, one, one, 4, 1.0, one, 3, null) == -9
    assert t(4, one, 4, null, one, 4, 1.0, one, 4, null) == -4
    # caqr_rpca_update_f32(m, n, M, ldm, L, ldl, S, lds, Y, ldy, X, ldx, mu, mu_next, lambda, resid, stream)
    u = L.caqr_rpca_update_f32
    assert u(4, 2, one, 4, one, 4, one, 4, one, 4, one, 4, 0.0, 1.0, 0.1, one, null) == -13
    assert u(4, 2, one, 4, one, 4, one, 4, one, 4, one, 4, 1.0, -1.0, 0.1, one, null) == -14
    assert u(4, 2, one, 4, one, 4, one, 4, one, 4, one, 4, 1.0, 1.0, -0.1, one, null) == -15
    assert u(4, 2, one, 4, one, 4, one, 4, one, 4, one, 4, 1.0, 1.0, 0.1, null, null) == -16
    assert u(4, 2, one, 4, one, 3, one, 4, one, 4, one, 4, 1.0, 1.0, 0.1, one, null) == -6
    assert u(4, 2, one, 4, null, 4, one, 4, one, 4, one, 4, 1.0, 1.0, 0.1, one, null) == -5
    # caqr_embed_top_f32(m, n, W, ldw, C, ldc, stream)
    e = L.caqr_embed_top_f32
    assert e(4, 5, one, 5, one, 4, null) == -2 and e(4, 2, one, 2, one, 3, null) == -6
    # caqr_trsm_upper_f32(n, k, R, ldr, B, ldb, stream)
    r = L.caqr_trsm_upper_f32
    assert r(-1, 1, one, 1, one, 1, null) == -1 and r(4, -1, one, 4, one, 4, null) == -2
    assert r(4, 1, one, 3, one, 4, null) == -4 and r(4, 1, one, 4, one, 3, null) == -6
    assert r(4, 1, null, 4, one, 4, null) == -3 and r(0, 3, null, 1, null, 1, null) == 0
    # caqr_lstsq_f32(m, n, A, lda, ws, k, B, ldb, opts, stream): apply_qt's numbering
    q = L.caqr_lstsq_f32
    assert q(4, 5, one, 4, one, 1, one, 4, null, null) == -2
    assert q(4, 2, one, 4, one, -1, one, 4, null, null) == -6
    assert q(4, 2, one, 4, one, 1, one, 3, null, null) == -8
    # caqr_set_identity_f32(m, n, Q, ldq, stream)
    i = L.caqr_set_identity_f32
    assert i(4, 5, one, 4, null) == -2 and i(4, 2, one, 3, null) == -4 and i(4, 2, null, 4, null) == -3


def test_factor_host_layout(L):
    """caqr_factor_host_*: chunk rows m*c/S, 256-B aligned chunk workspaces,
    then the R stack and the combine workspace (include/caqr.h)."""
    a256 = lambda x: -(-x // 256) * 256
    m, n, S = 1_000_003, 192, 8
    off = 0
    for c in range(S):
        r0, mc, o = caqr.caqr_factor_host_layout(m, n, S, c)
        assert (r0, mc, o) == (m * c // S, m * (c + 1) // S - m * c // S, off)
        off += a256(caqr.caqr_workspace_bytes(mc, n))
    assert caqr.caqr_factor_host_layout(m, n, S, S) == (0, S * n, off)
    off += a256(S * n * n * 4)
    assert caqr.caqr_factor_host_layout(m, n, S, S + 1) == (0, 0, off)
    total = off + a256(caqr.caqr_combine_workspace_bytes(S, n))
    assert caqr.caqr_factor_host_workspace_bytes(m, n, S) == total
    # S = 1: one chunk = the whole matrix
    assert caqr.caqr_factor_host_layout(5000, 16, 1, 0) == (0, 5000, 0)
    # illegal: m/S < n, n > 256 with S > 1, S out of range, bad dtype
    assert caqr.caqr_factor_host_workspace_bytes(100, 64, 4) == 0
    assert caqr.caqr_factor_host_workspace_bytes(100_000, 300, 2) == 0
    assert caqr.caqr_factor_host_workspace_bytes(100_000, 30, 0) == 0
    assert caqr.caqr_factor_host_workspace_bytes(100_000, 30, 1025) == 0
    assert caqr.caqr_factor_host_workspace_bytes(100_000, 30, 2, 7) == 0
    with pytest.raises(caqr.CaqrError):
        caqr.caqr_factor_host_layout(m, n, S, S + 2)
    # info codes that need no device: bad m, n, chunks, lda_host, lda, ldr
    fn = L.caqr_factor_host_f32
    assert fn(-1, 4, 2, None, 10, None, 10, None, 4, None, 0, None, None) == -1
    assert fn(10, 11, 2, None, 10, None, 10, None, 11, None, 0, None, None) == -2
    assert fn(100, 64, 4, None, 100, None, 100, None, 64, None, 0, None, None) == -3
    assert fn(100, 4, 2, None, 99, None, 100, None, 4, None, 0, None, None) == -5
    assert fn(100, 4, 2, None, 100, None, 99, None, 4, None, 0, None, None) == -7
    assert fn(100, 4, 2, None, 100, None, 100, None, 3, None, 0, None, None) == -9
    assert fn(0, 0, 1, None, 1, None, 1, None, 1, None, 0, None, None) == 0
