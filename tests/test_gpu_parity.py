"""GPU parity: the CUDA path through the C ABI against the CPU oracle.

Bounds (BASELINE.json north_star):
    fp32: ||A-QR||/||A|| <= 1e-5, ||Q^T Q - I|| <= 1e-5, ||R - R_oracle||/||R|| <= 1e-4
    fp64: 1e-13, 1e-13, 1e-12
R and Q are compared after sign normalisation (several correct answers:
DESIGN.md reading S17); rows n.. of Q^T C only through column norms.
"""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_andersonbdk11_b200 import workloads

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

BOUNDS = {
    np.float32: dict(res=1e-5, orth=1e-5, r=1e-4, acc="d"),
    np.float64: dict(res=1e-13, orth=1e-13, r=1e-12, acc="ld"),
}


@pytest.fixture(scope="module")
def caqr():
    from paper_conf_ipps_andersonbdk11_b200 import build as cbuild
    from paper_conf_ipps_andersonbdk11_b200 import caqr as c

    cbuild.build()
    c.lib()
    return c


def to_dev(c, A):
    t = c.colmajor_empty(A.shape[0], A.shape[1], torch.float32 if A.dtype == np.float32 else torch.float64)
    t.copy_(torch.from_numpy(np.ascontiguousarray(A)))
    return t


def gpu_qr(c, A, opts=None, want_q=True):
    Ad = to_dev(c, A)
    R, ws = c.caqr_factor(Ad, opts=opts)
    Q = c.caqr_form_q(Ad, ws, opts=opts) if want_q else None
    torch.cuda.synchronize()
    return R.cpu().numpy().astype(np.float64), (None if Q is None else Q.cpu().numpy().astype(np.float64)), Ad, ws


def oracle_f_orth(A64):
    """||Q^T Q - I||_F of the oracle's plain fp32 Householder QR (accumulation in
    float, acc="f"): what an fp32 Householder QR of this matrix reaches."""
    _, Qf = oracle.qr(A64, want_q=True, acc="f")
    n = A64.shape[1]
    return np.linalg.norm(Qf.T @ Qf - np.eye(n))


def orth_bound(A64, bd, dt):
    """north_star's 1e-5 (fp32) / 1e-13 (fp64) orthogonality bound.  SURVEY 9.1:
    for fp32 and n > 192 an fp32 Householder QR itself exceeds 1e-5 (LAPACK
    sgeqrf+sorgqr: 1.5e-5 at n = 512 ... 8.4e-5 at 8192), so there the bound is
    3x the oracle's own fp32 value on the same matrix."""
    n = A64.shape[1]
    if dt == np.float32 and n > 192:
        return max(bd["orth"], 3.0 * oracle_f_orth(A64))
    return bd["orth"]


def check_against_oracle(c, A, opts=None, C_cols=3):
    dt = A.dtype.type
    bd = BOUNDS[dt]
    m, n = A.shape
    R, Q, Ad, ws = gpu_qr(c, A, opts)
    A64 = A.astype(np.float64)
    # R is upper triangular, exactly zero below the diagonal
    assert np.all(np.tril(R, -1) == 0)
    Ro = oracle.qr(A64, want_q=False, acc=bd["acc"])
    Rn, Qn = oracle.normalize_signs(R, Q)
    Ron = oracle.normalize_signs(Ro)
    nr = max(np.linalg.norm(Ron), 1e-300)
    assert np.linalg.norm(Rn - Ron) / nr <= bd["r"], "R vs oracle"
    assert np.linalg.norm(A64 - Q @ R) / max(np.linalg.norm(A64), 1e-300) <= bd["res"], "residual"
    assert np.linalg.norm(Q.T @ Q - np.eye(n)) <= orth_bound(A64, bd, dt), "orthogonality"
    # Q^T C: top n rows equal Q_thin^T C (sign-normalised); column norms preserved
    if C_cols:
        rng = np.random.default_rng(m + n)
        C = rng.standard_normal((m, C_cols)).astype(A.dtype)
        Cd = to_dev(c, C)
        c.caqr_apply_qt(Ad, ws, Cd, opts=opts)
        QtC = Cd.cpu().numpy().astype(np.float64)
        VR, tau = oracle.geqr2(A64, acc=bd["acc"])
        QtC_o = oracle.orm2r(VR, tau, C.astype(np.float64), trans=True, acc=bd["acc"])
        d_gpu = np.where(np.diag(R) < 0, -1.0, 1.0)
        d_orc = np.where(np.diag(Ro) < 0, -1.0, 1.0)
        top_gpu = d_gpu[:, None] * QtC[:n]
        top_orc = d_orc[:, None] * QtC_o[:n]
        scale = np.linalg.norm(C.astype(np.float64))
        assert np.linalg.norm(top_gpu - top_orc) / scale <= bd["r"], "Q^T C top rows"
        np.testing.assert_allclose(np.linalg.norm(QtC, axis=0), np.linalg.norm(C.astype(np.float64), axis=0),
                                   rtol=10 * bd["res"])
        # round trip Q (Q^T C) = C
        c.caqr_apply_q(Ad, ws, Cd, opts=opts)
        back = Cd.cpu().numpy().astype(np.float64)
        assert np.linalg.norm(back - C) / scale <= 10 * bd["res"]
    return R, Q


SHAPES = [
    (4096, 16),    # config C1
    (1, 1), (2, 2), (7, 7), (33, 1), (100, 5), (257, 32), (300, 33),
    (1000, 7), (777, 100), (2049, 192), (600, 192), (5000, 64), (266, 32),  # 266: last leaf 10 rows < n
    (256, 256), (513, 256),
]


@pytest.mark.parametrize("dtype", [np.float32, np.float64], ids=["f32", "f64"])
@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: f"{s[0]}x{s[1]}")
def test_factor_parity(caqr, shape, dtype):
    A = workloads.gaussian(*shape, seed=shape[0] * 7 + shape[1], dtype=dtype)
    check_against_oracle(caqr, A)


@pytest.mark.parametrize("shape", [(90000, 256), (80000, 232)], ids=lambda s: f"{s[0]}x{s[1]}")
def test_tall_wide_groups_parity(caqr, shape):
    """Tall matrices with 224 < n <= 256: two 128-column panel groups of
    224-row tiles in chains (the fused kernel for both groups' TSQRs, the
    tree-replayed trailing update between them), against the oracle at the
    unrelaxed bounds of check_against_oracle."""
    info = caqr.caqr_plan_info(*shape)
    assert info["groups"] == 2 and info["leaf_rows"] == 224 and info["leaves"] > info["chains"]
    A = workloads.gaussian(*shape, seed=shape[1] + 11)
    check_against_oracle(caqr, A)


@pytest.mark.parametrize("leaf_rows", [32, 64, 128, 256])
def test_leaf_size_sweep(caqr, leaf_rows):
    """Uniqueness of R: every leaf size / tree gives the oracle's R (S5, S6)."""
    A = workloads.gaussian(3000, 24, seed=5)
    check_against_oracle(caqr, A, opts=caqr.make_opts(leaf_rows=leaf_rows))


@pytest.mark.parametrize("shape,nb", [((512, 512), 64), ((1000, 300), 0), ((2000, 130), 32),
                                       ((700, 200), 96), ((3000, 256), 0), ((1024, 1024), 64)])
@pytest.mark.parametrize("dtype", [np.float32, np.float64], ids=["f32", "f64"])
def test_caqr_panel_loop(caqr, shape, nb, dtype):
    """CAQR: TSQR panel groups + trailing update (Fig. 4), square-ish
    shapes, at north_star's unrelaxed R and residual bounds (fp32 LAPACK reaches
    4.6-5.9e-7 on R and <= 7.1e-7 residual for square n <= 8192);
    orthogonality per orth_bound."""
    A = workloads.gaussian(*shape, seed=11, dtype=dtype)
    opts = caqr.make_opts(panel_cols=nb) if nb else None
    m, n = shape
    R, Q, Ad, ws = gpu_qr(caqr, A, opts)
    bd = BOUNDS[dtype]
    A64 = A.astype(np.float64)
    Ro = oracle.qr(A64, want_q=False, acc=bd["acc"])
    Rn = oracle.normalize_signs(R)
    Ron = oracle.normalize_signs(Ro)
    assert np.linalg.norm(Rn - Ron) / np.linalg.norm(Ron) <= bd["r"]
    assert np.linalg.norm(A64 - Q @ R) / np.linalg.norm(A64) <= bd["res"]
    assert np.linalg.norm(Q.T @ Q - np.eye(n)) <= orth_bound(A64, bd, dtype)


def test_caqr_2048_square_vs_oracle(caqr):
    """Square CAQR (the C5 path: 64-wide panel groups, trailing update on the
    tensor cores) at 2048 x 2048 against the oracle, unrelaxed R bound 1e-4."""
    A = workloads.gaussian(2048, 2048, seed=3)
    R, Q, Ad, ws = gpu_qr(caqr, A, caqr.make_opts(panel_cols=64))
    A64 = A.astype(np.float64)
    Ron = oracle.normalize_signs(oracle.qr(A64, want_q=False))
    assert np.linalg.norm(oracle.normalize_signs(R) - Ron) / np.linalg.norm(Ron) <= 1e-4
    assert np.linalg.norm(A64 - Q @ R) / np.linalg.norm(A64) <= 1e-5
    assert np.linalg.norm(Q.T @ Q - np.eye(2048)) <= 3.0 * oracle_f_orth(A64)


def test_c5_square_8192_properties(caqr):
    """Config C5 (8192 x 8192 fp32, panel width 64) in its default plan: checks
    that hold at any size, in fp64 on the device -- R^T R = A^T A and A = QR at
    north_star's 1e-5, and ||Q^T Q - I||_F <= 3x the oracle's own fp32
    Householder QR on an 8192^2 Gaussian (tests/golden/oracle_f_orth.json,
    tools/make_golden_orth.py; the 1e-5 of north_star is infeasible
    for any fp32 Householder QR at this n -- fp32 LAPACK: 8.4e-5)."""
    import json
    import os
    with open(os.path.join(os.path.dirname(__file__), "golden", "oracle_f_orth.json")) as f:
        orth_f = float(json.load(f)["8192"])
    n = 8192
    A = workloads.device_gaussian(n, n, seed=7, dtype=torch.float32, device="cuda").t()
    A0 = A.clone()
    R, ws = caqr.caqr_factor(A)
    Q = caqr.caqr_form_q(A, ws)
    torch.cuda.synchronize()
    A64 = A0.double()
    del A0
    R64 = R.double()
    G = A64.t() @ A64
    assert (torch.linalg.norm(R64.t() @ R64 - G) / torch.linalg.norm(G)).item() <= 1e-5
    del G
    Q64 = Q.double()
    del Q
    assert (torch.linalg.norm(A64 - Q64 @ R64) / torch.linalg.norm(A64)).item() <= 1e-5
    I = torch.eye(n, dtype=torch.float64, device="cuda")
    assert torch.linalg.norm(Q64.t() @ Q64 - I).item() <= 3.0 * orth_f


@pytest.mark.parametrize("name,dtype,tol", [("r_1000000x192_f32_seed0", np.float32, 1e-4),
                                            ("r_200000x192_f64_seed1", np.float64, 1e-12)],
                         ids=["C4-f32-1Mx192", "C4-f64-200kx192"])
def test_full_size_r_vs_oracle_golden(caqr, name, dtype, tol):
    """Config C4 at full size: the whole R (every element) against the oracle's R,
    computed on the CPU by tools/make_golden.py (oracle only) from the same seeded
    host input, in the bench's launch configuration (default plan).  fp32: oracle
    in double; fp64: oracle in long double."""
    import os
    g = np.load(os.path.join(os.path.dirname(__file__), "golden", name + ".npz"))
    m, n, seed = int(g["m"]), int(g["n"]), int(g["seed"])
    A = workloads.gaussian(m, n, seed=seed, dtype=dtype)
    R, _, Ad, ws = gpu_qr(caqr, A, want_q=False)
    Ro = g["R"]
    assert np.all(np.tril(R, -1) == 0)
    err = np.linalg.norm(oracle.normalize_signs(R) - Ro) / np.linalg.norm(Ro)
    assert err <= tol, err
    # Q^T A = [R; 0]: top rows equal R, bottom rows vanish (relative to ||A||)
    Cd = to_dev(caqr, A[:, :4])
    caqr.caqr_apply_qt(Ad, ws, Cd)
    QtA = Cd.cpu().numpy().astype(np.float64)
    res = 1e-5 if dtype == np.float32 else 1e-13
    assert np.linalg.norm(QtA[:n] - R[:, :4]) / np.linalg.norm(R[:, :4]) <= 10 * res
    assert np.linalg.norm(QtA[n:]) / np.linalg.norm(A[:, :4].astype(np.float64)) <= 10 * res


def test_deterministic(caqr):
    """Run-to-run bitwise determinism (S15: no float atomics)."""
    A = workloads.gaussian(20000, 64, seed=2)
    R1, Q1, _, _ = gpu_qr(caqr, A)
    R2, Q2, _, _ = gpu_qr(caqr, A)
    assert np.array_equal(R1, R2) and np.array_equal(Q1, Q2)


def test_power_of_two_column_scaling_bitwise(caqr):
    """R(A diag(2^e)) == R(A) diag(2^e) bitwise: every Householder step is
    scale-covariant and the reductions are deterministic."""
    A = workloads.gaussian(5000, 48, seed=9)
    e = np.random.default_rng(1).integers(-20, 20, size=48)
    s = np.ldexp(np.float32(1), e).astype(np.float32)
    As = (A * s[None, :]).astype(np.float32)
    assert As.dtype == np.float32
    R, _, _, _ = gpu_qr(caqr, A, want_q=False)
    Rs, _, _, _ = gpu_qr(caqr, As, want_q=False)
    assert np.array_equal(Rs, (R.astype(np.float32) * s[None, :]).astype(np.float64))


def test_zero_row_padding_bitwise(caqr):
    """R([A; 0]) == R(A) bitwise when the padding fills whole leaves: zero
    leaves merge with tau = 0 (reading S2)."""
    opts = caqr.make_opts(leaf_rows=256)
    A = workloads.gaussian(256 * 5, 40, seed=4)
    Z = np.vstack([A, np.zeros((256 * 3, 40), np.float32)])
    R, _, _, _ = gpu_qr(caqr, A, opts, want_q=False)
    Rz, _, _, _ = gpu_qr(caqr, Z, opts, want_q=False)
    assert np.array_equal(R, Rz)


def test_row_permutation_of_leaves(caqr):
    """Permuting whole leaves changes the tree's inputs, not R (uniqueness)."""
    b = 256
    A = workloads.gaussian(b * 8, 32, seed=6)
    perm = np.random.default_rng(0).permutation(8)
    Ap = np.vstack([A[i * b:(i + 1) * b] for i in perm])
    opts = caqr.make_opts(leaf_rows=b)
    R, _, _, _ = gpu_qr(caqr, A, opts, want_q=False)
    Rp, _, _, _ = gpu_qr(caqr, Ap, opts, want_q=False)
    Rn, Rpn = oracle.normalize_signs(R), oracle.normalize_signs(Rp)
    assert np.linalg.norm(Rn - Rpn) / np.linalg.norm(Rn) <= 1e-5


@pytest.mark.parametrize("dtype", [np.float32, np.float64], ids=["f32", "f64"])
@pytest.mark.parametrize("P,n", [(2, 16), (3, 100), (8, 192), (5, 33)])
def test_combine_matches_single_shot(caqr, P, n, dtype):
    """Multi-GPU combine emulated on one GPU: factor P row slices separately,
    stack their R's, combine -> the R of the whole matrix."""
    m_local = 1000
    A = workloads.gaussian(P * m_local, n, seed=P * 100 + n, dtype=dtype)
    stack = np.zeros((P * n, n), dtype=dtype)
    for r in range(P):
        Rr, _, _, _ = gpu_qr(caqr, A[r * m_local:(r + 1) * m_local], want_q=False)
        stack[r * n:(r + 1) * n] = Rr.astype(dtype)
    Sd = to_dev(caqr, stack)
    R, ws = caqr.caqr_combine(Sd, P)
    torch.cuda.synchronize()
    R = R.cpu().numpy().astype(np.float64)
    bd = BOUNDS[dtype]
    Ro = oracle.normalize_signs(oracle.qr(A.astype(np.float64), want_q=False, acc=bd["acc"]))
    assert np.linalg.norm(oracle.normalize_signs(R) - Ro) / np.linalg.norm(Ro) <= bd["r"]
    # the combine's Q maps the stack to [R; 0]
    C = to_dev(caqr, stack)
    caqr.caqr_combine_apply(Sd, P, ws, C, trans=True)
    top = C.cpu().numpy().astype(np.float64)
    np.testing.assert_allclose(top[:n], R, atol=50 * bd["res"] * np.abs(R).max())
    assert np.abs(top[n:]).max() <= 50 * bd["res"] * np.abs(R).max()


@pytest.mark.parametrize("shifted", [False, True])
def test_krylov_basis_config(caqr, shifted):
    """s-step Krylov basis (config C2 recipe, smaller grid): kappa up to ~7e4."""
    A = workloads.krylov_basis(grid=500, s=8, seed=0, shifted=shifted)
    R, Q = check_against_oracle(caqr, A, C_cols=0)


def test_video_config(caqr):
    """Robust-PCA video matrix (config C3 shape 110,592 x 100)."""
    A = workloads.video(seed=0)
    check_against_oracle(caqr, A, C_cols=2)


def test_krylov_full_size(caqr):
    """Config C2 at full size (4,000,000 x 8) against the oracle."""
    A = workloads.krylov_basis(grid=2000, s=8, seed=0, shifted=True)
    R, _, _, _ = gpu_qr(caqr, A, want_q=False)
    Ro = oracle.normalize_signs(oracle.qr(A.astype(np.float64), want_q=False))
    assert np.linalg.norm(oracle.normalize_signs(R) - Ro) / np.linalg.norm(Ro) <= 1e-4


@pytest.mark.parametrize("dtype", [torch.float32, torch.float64], ids=["f32", "f64"])
def test_headline_full_size_properties(caqr, dtype):
    """Config C4 (1,000,000 x 192) in the bench's launch configuration: checks
    that hold at any size, computed in fp64 on the device -- R^T R = A^T A,
    column norms of R = column norms of A, Q^T Q = I, A = QR."""
    m, n = 1_000_000, 192
    A = workloads.device_gaussian(m, n, seed=0, dtype=dtype, device="cuda").t()  # column-major
    A0 = A.clone()
    R, ws = caqr.caqr_factor(A)
    Q = caqr.caqr_form_q(A, ws)
    torch.cuda.synchronize()
    A64, R64, Q64 = A0.double(), R.double(), Q.double()
    G = A64.t() @ A64
    eps = 1e-4 if dtype == torch.float32 else 1e-12
    assert (torch.linalg.norm(R64.t() @ R64 - G) / torch.linalg.norm(G)).item() <= 2 * eps
    cn = torch.linalg.norm(A64, dim=0)
    assert (torch.abs(torch.linalg.norm(R64, dim=0) - cn) / cn).max().item() <= eps
    I = torch.eye(n, dtype=torch.float64, device="cuda")
    tol = 1e-5 if dtype == torch.float32 else 1e-13
    assert torch.linalg.norm(Q64.t() @ Q64 - I).item() <= tol
    assert (torch.linalg.norm(A64 - Q64 @ R64) / torch.linalg.norm(A64)).item() <= tol
    # sampled oracle check: a few leading columns' R entries against the oracle on A[:, :8]
    R8o = oracle.normalize_signs(oracle.qr(A0[:, :8].double().cpu().numpy(), want_q=False))
    R8 = oracle.normalize_signs(R64[:8, :8].cpu().numpy())
    assert np.linalg.norm(R8 - R8o) / np.linalg.norm(R8o) <= eps


def test_errors_raise(caqr):
    A = caqr.colmajor_empty(10, 4)
    with pytest.raises(caqr.CaqrError):
        caqr.caqr_factor(A, opts=caqr.Opts(48, 0))
    with pytest.raises(ValueError):
        caqr.caqr_factor(torch.zeros(10, 4, device="cuda"))  # row-major


def test_dist_single_rank_nccl(caqr):
    """caqr_dist_* through a real NCCL communicator with one rank (the only
    configuration one GPU allows): local TSQR + all-gather + combine must give
    exactly the single-GPU R."""
    import os
    import socket

    import torch.distributed as dist

    from paper_conf_ipps_andersonbdk11_b200 import dist as cdist

    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        A = workloads.gaussian(20000, 96, seed=8)
        R_ref, _, _, _ = gpu_qr(caqr, A, want_q=False)
        d = cdist.DistTSQR()
        Ad = to_dev(caqr, A)
        R, ws, gather, cws = d.factor(Ad)
        torch.cuda.synchronize()
        assert np.array_equal(R.cpu().numpy().astype(np.float64), R_ref)
        d.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("m,n,leaf", [(20000, 24, 32), (40000, 48, 64), (70000, 100, 128), (70000, 192, 224)])
@pytest.mark.parametrize("path", ["fused", "split"])
def test_chains(caqr, m, n, leaf, path, monkeypatch):
    """More tiles than the chain target (296): tiles form flat-tree chains of
    K > 1 tiles ([chain R; tile] steps), then the binary tree over chains.
    Both the one-launch dataflow kernel and the split path."""
    if path == "split":
        monkeypatch.setenv("CAQR_FUSED", "0")
    opts = caqr.make_opts(leaf_rows=leaf)
    info = caqr.caqr_plan_info(m, n, 0, opts)
    assert info["leaves"] > 296 and info["chains"] < info["leaves"]
    A = workloads.gaussian(m, n, seed=m + n)
    check_against_oracle(caqr, A, opts=opts, C_cols=2)


def test_fused_and_split_agree(caqr, monkeypatch):
    """The two execution paths run the same plan: results agree to rounding
    (different reduction orders inside the panel factorization)."""
    A = workloads.gaussian(70000, 64, seed=1)
    opts = caqr.make_opts(leaf_rows=64)
    R1, _, _, _ = gpu_qr(caqr, A, opts, want_q=False)
    monkeypatch.setenv("CAQR_FUSED", "0")
    R2, _, _, _ = gpu_qr(caqr, A, opts, want_q=False)
    assert np.linalg.norm(R1 - R2) / np.linalg.norm(R1) <= 1e-5


@pytest.mark.parametrize("m,n", [(600_000, 16), (2_100_000, 8), (700_000, 3)])
def test_skinny_chains(caqr, m, n):
    """Skinny fp32 panels (n <= 16) go to the streaming warp-per-chain kernel;
    with more tiles than its chain target (1184 chains for n <= 16, 2368 for
    n <= 8) the tiles form chains."""
    info = caqr.caqr_plan_info(m, n)
    assert info["chains"] < info["leaves"]
    A = workloads.gaussian(m, n, seed=n)
    check_against_oracle(caqr, A, C_cols=2)


def test_skinny_vs_block_kernel(caqr, monkeypatch):
    """Warp-per-task and block kernels on the same plan agree to rounding."""
    A = workloads.gaussian(300_000, 12, seed=3)
    R1, _, _, _ = gpu_qr(caqr, A, want_q=False)
    monkeypatch.setenv("CAQR_SKINNY", "0")
    R2, _, _, _ = gpu_qr(caqr, A, want_q=False)
    assert np.linalg.norm(R1 - R2) / np.linalg.norm(R1) <= 1e-5


@pytest.mark.parametrize("m,n,pad", [(300_001, 5, 1), (262_147, 9, 3), (400_000, 1, 0), (1_000_003, 16, 0),
                                     (524_288, 8, 4)])
def test_stream_kernel_layouts(caqr, m, n, pad):
    """Streaming skinny kernel (tsqr_stream.cuh): ragged last tile, n = 1 / 5 /
    8 / 9 / 16, lda = m + pad (pad % 4 != 0 -> 4-byte cp.async path) -- R
    against the oracle, Q^T Q = I, A = QR, Q^T A = [R; 0] through apply_qt."""
    bd = BOUNDS[np.float32]
    A = workloads.gaussian(m, n, seed=m % 97 + n)
    big = caqr.colmajor_empty(m + pad, n, torch.float32)
    Av = big[:m]
    Av.copy_(torch.from_numpy(A))
    R, ws = caqr.caqr_factor(Av)
    Q = caqr.caqr_form_q(Av, ws)
    C = caqr.colmajor_empty(m, n, torch.float32)
    C.copy_(torch.from_numpy(A))
    caqr.caqr_apply_qt(Av, ws, C)
    torch.cuda.synchronize()
    R64, Q64 = R.cpu().double().numpy(), Q.cpu().double().numpy()
    A64 = A.astype(np.float64)
    Ro = oracle.normalize_signs(oracle.qr(A64, want_q=False))
    assert np.linalg.norm(oracle.normalize_signs(R64) - Ro) / np.linalg.norm(Ro) <= bd["r"]
    assert np.linalg.norm(A64 - Q64 @ R64) / np.linalg.norm(A64) <= bd["res"]
    assert np.linalg.norm(Q64.T @ Q64 - np.eye(n)) <= bd["orth"]
    top = C.cpu().double().numpy()
    assert np.linalg.norm(top[:n] - R64) / np.linalg.norm(R64) <= bd["res"]
    assert np.linalg.norm(top[n:]) / np.linalg.norm(R64) <= 10 * bd["res"]


def test_stream_vs_warp_task_kernel(caqr, monkeypatch):
    """Streaming kernel and the older flag-waiting warp-per-task kernel run the
    same plan: R agrees to rounding, both against the oracle."""
    A = workloads.gaussian(2_000_000, 8, seed=4)
    R1, _, _, _ = gpu_qr(caqr, A, want_q=False)
    monkeypatch.setenv("CAQR_SKINNY", "2")
    R2, _, _, _ = gpu_qr(caqr, A, want_q=False)
    assert np.linalg.norm(R1 - R2) / np.linalg.norm(R1) <= 1e-5
    Ro = oracle.normalize_signs(oracle.qr(A.astype(np.float64), want_q=False))
    assert np.linalg.norm(oracle.normalize_signs(R1) - Ro) / np.linalg.norm(Ro) <= 1e-4


@pytest.mark.parametrize("dtype", [np.float32, np.float64], ids=["f32", "f64"])
def test_leading_dimensions(caqr, dtype):
    """lda > m (A is a row-slice view of a taller buffer) and ldc > m for Q^T C."""
    m, n, pad = 5000, 40, 77
    tdt = torch.float32 if dtype == np.float32 else torch.float64
    A = workloads.gaussian(m, n, seed=21, dtype=dtype)
    big = caqr.colmajor_empty(m + pad, n, tdt)
    big.zero_()
    Av = big[:m]  # column-major view, stride (1, m + pad)
    assert Av.stride(1) == m + pad
    Av.copy_(torch.from_numpy(A))
    R, ws = caqr.caqr_factor(Av)
    Q = caqr.caqr_form_q(Av, ws)
    Cbig = caqr.colmajor_empty(m + 13, 3, tdt)
    C0 = workloads.gaussian(m, 3, seed=22, dtype=dtype)
    Cv = Cbig[:m]
    Cv.copy_(torch.from_numpy(C0))
    caqr.caqr_apply_qt(Av, ws, Cv)
    torch.cuda.synchronize()
    bd = BOUNDS[dtype]
    R64, Q64 = R.cpu().double().numpy(), Q.cpu().double().numpy()
    assert np.linalg.norm(A - Q64 @ R64) / np.linalg.norm(A) <= bd["res"]
    np.testing.assert_allclose(Cv.cpu().double().numpy()[:n], Q64.T @ C0, atol=50 * bd["res"] * np.abs(C0).max())
    # rows below m of the padded buffer are untouched
    assert torch.count_nonzero(big[m:]).item() == 0


def test_empty_and_degenerate_shapes(caqr):
    """m = n = 0 and n = 0 are quick returns; a zero matrix gives R = 0, tau = 0."""
    A = caqr.colmajor_empty(10, 0)
    R, ws = caqr.caqr_factor(A)
    assert R.shape == (0, 0)
    A = caqr.colmajor_empty(0, 0)
    R, ws = caqr.caqr_factor(A)
    Z = np.zeros((3000, 24), np.float32)
    R, Q, _, _ = gpu_qr(caqr, Z)
    assert np.all(R == 0)
    # Q of a zero matrix is [I; 0] (every reflector is the identity)
    assert np.array_equal(Q, np.eye(3000, 24))


def test_chains_fp64(caqr):
    A = workloads.gaussian(70000, 96, seed=31, dtype=np.float64)
    opts = caqr.make_opts(leaf_rows=128)
    assert caqr.caqr_plan_info(70000, 96, 1, opts)["chains"] < 547
    check_against_oracle(caqr, A, opts=opts, C_cols=2)


def test_max_single_gpu_size_properties(caqr):
    """Config C4' (8,000,000 x 192 fp32, 6.1 GB) factored on one GPU: column
    norms of R equal those of A and R^T R = A^T A (computed in fp64)."""
    m, n = 8_000_000, 192
    A = workloads.device_gaussian(m, n, seed=5, dtype=torch.float32, device="cuda").t()
    G = torch.zeros((n, n), dtype=torch.float64, device="cuda")
    cn = torch.zeros(n, dtype=torch.float64, device="cuda")
    for s0 in range(0, m, 1_000_000):
        blk = A[s0:s0 + 1_000_000].double()
        G += blk.t() @ blk
        cn += (blk * blk).sum(0)
        del blk
    R, ws = caqr.caqr_factor(A)
    torch.cuda.synchronize()
    R64 = R.double()
    assert (torch.abs(torch.linalg.norm(R64, dim=0) - cn.sqrt()) / cn.sqrt()).max().item() <= 1e-4
    assert (torch.linalg.norm(R64.t() @ R64 - G) / torch.linalg.norm(G)).item() <= 2e-4


@pytest.mark.parametrize("m,n", [(2_000_000, 8), (600_000, 16)])
def test_stream_kernel_deterministic(caqr, m, n):
    """The skinny kernel's cross-CTA tree is merged by whichever CTA arrives
    second at each pair; the merge is the same arithmetic on any SM, so R, the
    stored vectors and Q are bitwise identical run to run (S15)."""
    A = workloads.gaussian(m, n, seed=m % 13)
    outs = []
    for _ in range(2):
        Ad = caqr.colmajor_empty(m, n)
        Ad.copy_(torch.from_numpy(A))
        R, ws = caqr.caqr_factor(Ad)
        Q = caqr.caqr_form_q(Ad, ws)
        torch.cuda.synchronize()
        outs.append((R.cpu().numpy(), Ad.cpu().numpy(), Q.cpu().numpy()))  # (ws: partly never written)
    for a, b in zip(*outs):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("m,n,dtype", [(70_000, 192, np.float32), (110_592, 100, np.float32),
                                       (30_000, 40, np.float64), (600_000, 8, np.float32)])
def test_node_update_matches_per_panel_launches(caqr, m, n, dtype, monkeypatch):
    """Q^T C / Q C / form_q with one launch per tree level (+ one for all chains)
    equal the per-(tile or level, panel) launches BITWISE: each node runs the
    same device routine in the same order; only the launch grouping differs."""
    monkeypatch.setenv("CAQR_STREAM_APPLY", "0")  # (the warp-per-chain skinny apply sums in another order)
    tdt = torch.float32 if dtype == np.float32 else torch.float64
    A = workloads.gaussian(m, n, seed=5, dtype=dtype)
    C0 = workloads.gaussian(m, 3, seed=6, dtype=dtype)
    Ad = caqr.colmajor_empty(m, n, tdt)
    Ad.copy_(torch.from_numpy(A))
    R, ws = caqr.caqr_factor(Ad)

    def run():
        Q = caqr.caqr_form_q(Ad, ws)
        C = caqr.colmajor_empty(m, 3, tdt)
        C.copy_(torch.from_numpy(C0))
        caqr.caqr_apply_qt(Ad, ws, C)
        D = caqr.colmajor_empty(m, 3, tdt)
        D.copy_(torch.from_numpy(C0))
        caqr.caqr_apply_q(Ad, ws, D)
        torch.cuda.synchronize()
        return Q.cpu().numpy(), C.cpu().numpy(), D.cpu().numpy()

    new = run()
    monkeypatch.setenv("CAQR_APPLY_ALL", "0")
    per_level = run()
    monkeypatch.setenv("CAQR_CHAIN_APPLY", "0")
    old = run()
    for a, b, c in zip(new, per_level, old):
        assert np.array_equal(a, b)
        assert np.array_equal(b, c)


@pytest.mark.parametrize("m,n,dtype", [(1_000_000, 192, np.float32), (200_000, 100, np.float64)])
def test_apply_one_launch_per_group(caqr, m, n, dtype):
    """Q^T C and form_q of a one-group plan are ONE apply
    launch (node_update_all_kernel schedules the chains and every tree level
    on the device) -- counted from the launch trace."""
    tdt = torch.float32 if dtype == np.float32 else torch.float64
    Ad = workloads.device_gaussian(m, n, seed=3, dtype=tdt, device="cuda").t()
    A = caqr.colmajor_empty(m, n, tdt)
    A.copy_(Ad)
    R, ws = caqr.caqr_factor(A)
    info = caqr.caqr_plan_info(m, n, 0 if dtype == np.float32 else 1)
    assert info["groups"] == 1 and info["tree_levels"] >= 5
    C = caqr.colmajor(Ad[:, :4].clone())
    torch.cuda.synchronize()
    caqr.caqr_trace_begin(1 << 12)
    caqr.caqr_apply_qt(A, ws, C)
    Q = caqr.caqr_form_q(A, ws)
    torch.cuda.synchronize()
    names = [t[0] for t in caqr.caqr_trace_end(1 << 12)]
    assert names.count("node_update_all") == 2, names
    assert "node_update" not in names and "panel_update" not in names, names
    # and the result is Q: Q^T Q = I, Q^T A = [R; 0] on the top rows
    bd = BOUNDS[dtype]
    Q64 = Q.double()
    eye = torch.eye(n, dtype=torch.float64, device="cuda")
    assert (Q64.t() @ Q64 - eye).norm().item() <= bd["orth"]
    top = (Q64.t() @ Ad[:, :4].double() - C[:n].double()).norm() / Ad[:, :4].double().norm()
    assert top.item() <= bd["res"]


@pytest.mark.parametrize("m,n,k", [(4_000_000, 8, 8), (600_001, 5, 11), (1_000_003, 16, 16), (262_147, 12, 3)])
def test_stream_apply_vs_node_update(caqr, m, n, k, monkeypatch):
    """Skinny plans: the warp-per-chain leaf apply (tsqr_stream_apply.cuh) and
    the CTA-per-node apply agree to rounding for Q^T C, Q C and form_q, and
    Q^T Q = I, Q^T A = [R; 0] hold (C4-style bounds, BASELINE fp32)."""
    bd = BOUNDS[np.float32]
    A = workloads.gaussian(m, n, seed=k)
    C0 = workloads.gaussian(m, k, seed=k + 1)
    Ad = caqr.colmajor_empty(m, n)
    Ad.copy_(torch.from_numpy(A))
    R, ws = caqr.caqr_factor(Ad)

    def run():
        Q = caqr.caqr_form_q(Ad, ws)
        C = caqr.colmajor_empty(m, k)
        C.copy_(torch.from_numpy(C0))
        caqr.caqr_apply_qt(Ad, ws, C)
        D = caqr.colmajor_empty(m, k)
        D.copy_(torch.from_numpy(C0))
        caqr.caqr_apply_q(Ad, ws, D)
        torch.cuda.synchronize()
        return [t.cpu().double().numpy() for t in (Q, C, D)]

    new = run()
    monkeypatch.setenv("CAQR_STREAM_APPLY", "0")
    old = run()
    for a, b in zip(new, old):
        assert np.linalg.norm(a - b) <= 1e-6 * np.linalg.norm(b)
    Q = new[0]
    R64 = R.cpu().double().numpy()
    assert np.linalg.norm(Q.T @ Q - np.eye(n)) <= bd["orth"]
    assert np.linalg.norm(A.astype(np.float64) - Q @ R64) / np.linalg.norm(A) <= bd["res"]
    QtC = new[1]
    Qt_ref = Q.T @ C0.astype(np.float64)
    assert np.linalg.norm(QtC[:n] - Qt_ref) / np.linalg.norm(C0) <= bd["res"]


@pytest.mark.parametrize("m,n,P,dtype", [(4_000_000, 8, 4, np.float32), (200_000, 48, 3, np.float32),
                                         (60_000, 40, 8, np.float64)])
def test_sharded_form_q_emulated(caqr, m, n, P, dtype):
    """The row-sharded explicit Q (dist.local_form_q: e.g. the
    s-step Krylov basis across GPUs), emulated on one GPU: each shard factored
    on its own, the stacked R's combined, then every shard's rows of Q formed
    from the combine's Q_c and the local Q.  Stacked, they are the thin Q of
    the whole matrix: Q^T Q = I, A = Q R, R against the oracle."""
    from paper_conf_ipps_andersonbdk11_b200 import dist as cdist

    tdt = torch.float32 if dtype == np.float32 else torch.float64
    bd = BOUNDS[dtype]
    A = workloads.gaussian(m, n, seed=P, dtype=dtype)
    gather = caqr.colmajor_empty(P * n, n, tdt)
    shards = []
    for p in range(P):
        s0, rows = cdist.shard_rows(m, P, p)
        Ap = caqr.colmajor_empty(rows, n, tdt)
        Ap.copy_(torch.from_numpy(A[s0:s0 + rows]))
        Rp, wsp = caqr.caqr_factor(Ap)
        gather[p * n:(p + 1) * n].copy_(Rp)
        shards.append((Ap, wsp))
    R, cws = caqr.caqr_combine(gather, P)
    Q = np.concatenate([cdist.local_form_q(Ap, wsp, gather, cws, p, P).cpu().double().numpy()
                        for p, (Ap, wsp) in enumerate(shards)])
    R = R.cpu().double().numpy()
    A64 = A.astype(np.float64)
    assert np.linalg.norm(Q.T @ Q - np.eye(n)) <= bd["orth"]
    assert np.linalg.norm(A64 - Q @ R) / np.linalg.norm(A64) <= bd["res"]
    rows = min(m, 300_000)
    if rows == m:
        Ro = oracle.normalize_signs(oracle.qr(A64, want_q=False, acc=bd["acc"]))
        assert np.linalg.norm(oracle.normalize_signs(R) - Ro) / np.linalg.norm(Ro) <= bd["r"]


@pytest.mark.parametrize("dtype", [np.float32, np.float64], ids=["f32", "f64"])
@pytest.mark.parametrize("m,n,S", [(5000, 16, 1), (20011, 64, 4), (30000, 192, 7), (4099, 33, 3)])
def test_factor_host_matches_oracle(caqr, m, n, S, dtype):
    """caqr_factor_host: chunked H2D + per-chunk TSQR + combine (the distributed
    TSQR tree of P:L181-188 over row blocks of one GPU).  R against the oracle;
    Q^T A = [R; 0] through the chunk layout (apply_qt per chunk, then the
    combine's Q^T on the chunks' top n rows)."""
    A = workloads.gaussian(m, n, seed=m + n + S, dtype=dtype)
    tdt = torch.float32 if dtype == np.float32 else torch.float64
    Ah = torch.empty((n, m), dtype=tdt, pin_memory=True).t()
    Ah.copy_(torch.from_numpy(A))
    Ad, R, ws = caqr.caqr_factor_host(Ah, S)
    torch.cuda.synchronize()
    R = R.cpu().numpy().astype(np.float64)
    bd = BOUNDS[dtype]
    assert np.all(np.tril(R, -1) == 0)
    Ro = oracle.normalize_signs(oracle.qr(A.astype(np.float64), want_q=False, acc=bd["acc"]))
    assert np.linalg.norm(oracle.normalize_signs(R) - Ro) / np.linalg.norm(Ro) <= bd["r"]
    code = caqr.CAQR_F32 if dtype == np.float32 else caqr.CAQR_F64
    C = to_dev(caqr, A)
    tops = []
    for c in range(S):
        r0, mc, off = caqr.caqr_factor_host_layout(m, n, S, c, code)
        assert mc >= n and r0 == (m * c) // S
        wb = caqr.caqr_workspace_bytes(mc, n, code)
        caqr.caqr_apply_qt(Ad[r0:r0 + mc], ws[off:off + wb], C[r0:r0 + mc], n=n)
        tops.append(C[r0:r0 + n].clone())
    if S > 1:
        _, rows, rs_off = caqr.caqr_factor_host_layout(m, n, S, S, code)
        _, _, cw_off = caqr.caqr_factor_host_layout(m, n, S, S + 1, code)
        esz = 4 if dtype == np.float32 else 8
        Rs = ws[rs_off:rs_off + rows * n * esz].view(tdt).view(n, rows).t()
        st = caqr.colmajor(torch.cat(tops, 0))
        caqr.caqr_combine_apply(Rs, S, ws[cw_off:], st, trans=True)
        top = st.cpu().numpy().astype(np.float64)
    else:
        top = C.cpu().numpy().astype(np.float64)
    tol = 50 * bd["res"] * np.abs(R).max()
    np.testing.assert_allclose(top[:n], R, atol=tol)
    assert np.abs(top[n:]).max() <= tol
    # the host factorization's R equals the single-shot device factorization's R up to rounding
    R1, _, _, _ = gpu_qr(caqr, A, want_q=False)
    assert np.linalg.norm(oracle.normalize_signs(R1) - oracle.normalize_signs(R)) / np.linalg.norm(R1) <= bd["r"]


def test_factor_host_errors(caqr):
    with pytest.raises(caqr.CaqrError):
        caqr.caqr_factor_host(torch.zeros(64, 100).t(), 4)  # 100 x 64 in 4 chunks: m/S < n
    with pytest.raises(ValueError):
        caqr.caqr_factor_host(torch.zeros(100, 4, device="cuda").t().contiguous().t(), 2)


@pytest.mark.parametrize("dtype", [np.float32, np.float64], ids=["f32", "f64"])
@pytest.mark.parametrize("P,m,n", [(2, 4000, 64), (3, 10001, 96), (8, 40000, 192), (8, 1600, 192)])
def test_dist_combine_blocks_P_ranks(caqr, P, m, n, dtype):
    """The post-all-gather half of caqr_dist_factor (caqr_dist_combine_blocks,
    the code caqr_dist_factor runs after ncclAllGather) at P > 1, emulating P
    ranks on one GPU: each row shard factored on its own, the local R's laid out
    exactly as the all-gather leaves them (P contiguous n x n column-major
    blocks in rank order, some with ldr != n copies), restacked + combined.  The
    result must be the oracle's R of the whole matrix (uniqueness of R, S17),
    and Q^T A through the local Q's and the combine's Q_c must be [R; 0]."""
    from paper_conf_ipps_andersonbdk11_b200 import dist as cdist

    tdt = torch.float32 if dtype == np.float32 else torch.float64
    bd = BOUNDS[dtype]
    A = workloads.gaussian(m, n, seed=100 + P, dtype=dtype)
    blocks = torch.empty(P * n * n, dtype=tdt, device="cuda")
    shards = []
    for p in range(P):
        s0, rows = cdist.shard_rows(m, P, p)
        Ap = caqr.colmajor_empty(rows, n, tdt)
        Ap.copy_(torch.from_numpy(A[s0:s0 + rows]))
        Rp, wsp = caqr.caqr_factor(Ap)
        # the send slot of rank p: its R as a contiguous column-major n x n block
        blocks[p * n * n:(p + 1) * n * n].copy_(Rp.t().contiguous().reshape(-1))
        shards.append((s0, rows, Ap, wsp))
    R, gather, cws = caqr.caqr_dist_combine_blocks(blocks, P, n)
    torch.cuda.synchronize()
    Rn = R.cpu().double().numpy()
    assert np.all(np.tril(Rn, -1) == 0)
    A64 = A.astype(np.float64)
    Ro = oracle.normalize_signs(oracle.qr(A64, want_q=False, acc=bd["acc"]))
    assert np.linalg.norm(oracle.normalize_signs(Rn) - Ro) / np.linalg.norm(Ro) <= bd["r"]
    # Q^T A: local Q_p^T A_p, top n rows of every shard stacked, then Q_c^T
    k = 3
    top = caqr.colmajor_empty(P * n, k, tdt)
    bottom_sq = 0.0
    for p, (s0, rows, Ap, wsp) in enumerate(shards):
        Cp = to_dev(caqr, A[s0:s0 + rows, :k])
        caqr.caqr_apply_qt(Ap, wsp, Cp)
        top[p * n:(p + 1) * n].copy_(Cp[:n])
        bottom_sq += float((Cp[n:].double() ** 2).sum())
    caqr.caqr_combine_apply(gather, P, cws, top, trans=True)
    T = top.cpu().double().numpy()
    scale = np.linalg.norm(A64[:, :k])
    assert np.linalg.norm(T[:n] - Rn[:, :k]) / scale <= 10 * bd["res"]
    assert np.sqrt(bottom_sq + np.linalg.norm(T[n:]) ** 2) / scale <= 10 * bd["res"]


def test_dist_combine_blocks_errors(caqr):
    blocks = torch.zeros(2 * 4 * 4, device="cuda")
    with pytest.raises(caqr.CaqrError):
        caqr.caqr_dist_combine_blocks(blocks, 0, 4)          # P < 1
    with pytest.raises(caqr.CaqrError):
        caqr.caqr_dist_combine_blocks(blocks, 2, 4, cws=torch.empty(8, dtype=torch.uint8, device="cuda"))


@pytest.mark.parametrize("dual", ["0", "1"])
@pytest.mark.parametrize("m,n,S,nb", [(30000, 192, 6, 0), (20000, 130, 4, 64), (9000, 96, 3, 32)])
def test_factor_host_dual_and_panel_groups(caqr, m, n, S, nb, dual, monkeypatch):
    """caqr_factor_host with both stream policies (CAQR_HOST_DUAL: odd chunks on
    the library's second stream or all on the caller's) and with chunks that run
    the CAQR panel loop (panel_cols < n: the shared early-start side stream):
    R against the oracle and bitwise identical between the two policies."""
    monkeypatch.setenv("CAQR_HOST_DUAL", dual)
    A = workloads.gaussian(m, n, seed=m + S, dtype=np.float32)
    Ah = torch.empty((n, m), dtype=torch.float32, pin_memory=True).t()
    Ah.copy_(torch.from_numpy(A))
    opts = caqr.make_opts(panel_cols=nb) if nb else None
    Ad, R, ws = caqr.caqr_factor_host(Ah, S, opts=opts)
    torch.cuda.synchronize()
    R = R.cpu().numpy().astype(np.float64)
    Ro = oracle.normalize_signs(oracle.qr(A.astype(np.float64), want_q=False))
    assert np.linalg.norm(oracle.normalize_signs(R) - Ro) / np.linalg.norm(Ro) <= 1e-4
    monkeypatch.setenv("CAQR_HOST_DUAL", "1" if dual == "0" else "0")
    _, R2, _ = caqr.caqr_factor_host(Ah, S, opts=opts)
    torch.cuda.synchronize()
    assert np.array_equal(R, R2.cpu().numpy().astype(np.float64))


def test_concurrent_caqr_calls_two_threads(caqr):
    """Two host threads factoring different matrices through the CAQR panel loop
    (n > 256: early-start overlap on the per-device side stream) at once, each
    on its own stream: both R's match their single-threaded results bitwise."""
    import threading

    mats = [workloads.gaussian(3000, 300, seed=s) for s in (1, 2)]
    ref = [gpu_qr(caqr, M, want_q=False)[0] for M in mats]
    out = [None, None]

    def work(i):
        st = torch.cuda.Stream()
        with torch.cuda.stream(st):
            for _ in range(5):
                Ad = to_dev(caqr, mats[i])
                R, _ = caqr.caqr_factor(Ad, stream=st)
            st.synchronize()
            out[i] = R.cpu().numpy().astype(np.float64)

    th = [threading.Thread(target=work, args=(i,)) for i in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    for i in range(2):
        assert np.array_equal(out[i], ref[i])


@pytest.mark.parametrize("m,n", [(100_000, 192), (3000, 300)])
def test_cuda_graph_capture(caqr, m, n):
    """The header's claim that every call only enqueues work on its stream:
    factor + apply_qt + form_q captured into one CUDA graph (for n = 300 the
    CAQR loop with its early-start fork to the library's side stream and the
    join back), replayed twice on a freshly restored A: R, Q^T C and Q bitwise
    equal to the eager calls."""
    A = workloads.gaussian(m, n, seed=9)
    Ad = to_dev(caqr, A)
    A0 = Ad.clone()
    C0 = to_dev(caqr, A[:, :3])
    R, ws = caqr.caqr_factor(Ad)
    C = C0.clone()
    caqr.caqr_apply_qt(Ad, ws, C)
    Q = caqr.caqr_form_q(Ad, ws)
    torch.cuda.synchronize()
    R_e, C_e, Q_e = R.clone(), C.clone(), Q.clone()
    st = torch.cuda.Stream()
    st.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(st):
        Ad.copy_(A0)
        C.copy_(C0)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=st):
            caqr.caqr_factor(Ad, R=R, ws=ws, stream=st)
            caqr.caqr_apply_qt(Ad, ws, C, stream=st)
            caqr.caqr_form_q(Ad, ws, Q=Q, stream=st)
    for _ in range(2):
        Ad.copy_(A0)
        C.copy_(C0)
        R.zero_()
        Q.zero_()
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        assert torch.equal(R, R_e) and torch.equal(C, C_e) and torch.equal(Q, Q_e)


@pytest.mark.parametrize("m,n,dtype", [(20_000, 100, np.float32), (4096, 640, np.float32), (30_000, 24, np.float64)])
def test_tune_plan_search(caqr, m, n, dtype):
    """caqr_tune: times several distinct plans on
    a scratch copy, leaves A unchanged, returns a plan no slower than the
    default (the default is a candidate), and that plan factors A correctly
    (R^T R = A^T A)."""
    tdt = torch.float32 if dtype == np.float32 else torch.float64
    A0 = workloads.device_gaussian(m, n, seed=11, dtype=tdt, device="cuda").t()
    A = caqr.colmajor_empty(m, n, tdt)
    A.copy_(A0)
    opts, best_ms, default_ms, tried = caqr.caqr_tune(A, reps=2)
    torch.cuda.synchronize()
    assert torch.equal(A, A0)
    assert tried >= 3 and 0 < best_ms <= default_ms
    R, _ = caqr.caqr_factor(A, opts=opts)
    A64 = A0.double()
    G = A64.t() @ A64
    R64 = R.double()
    err = (R64.t() @ R64 - G).norm() / G.norm()
    assert err.item() <= BOUNDS[dtype]["res"]  # backward error of a Householder QR (the residual bound)
    assert torch.tril(R, -1).abs().max().item() == 0.0


def test_tune_info_codes(caqr):
    L = caqr.lib()
    import ctypes

    best = caqr.Opts()
    f = ctypes.c_float()
    assert L.caqr_tune(-1, 4, 0, None, 1, 1, ctypes.byref(best), ctypes.byref(f), None, None, None) == -1
    assert L.caqr_tune(4, 5, 0, None, 4, 1, ctypes.byref(best), ctypes.byref(f), None, None, None) == -2
    assert L.caqr_tune(8, 4, 7, None, 8, 1, ctypes.byref(best), ctypes.byref(f), None, None, None) == -3
    assert L.caqr_tune(8, 4, 0, None, 8, 1, ctypes.byref(best), ctypes.byref(f), None, None, None) == -4
    assert L.caqr_tune(8, 4, 0, None, 8, 1, None, ctypes.byref(f), None, None, None) == -7


@pytest.mark.gpu
@pytest.mark.parametrize("P,m,n,dtype", [(2, 4000, 64, np.float32), (3, 9000, 100, np.float32),
                                         (8, 16000, 192, np.float32), (3, 6000, 50, np.float64)])
def test_peer_exchange_emulated_ranks(caqr, P, m, n, dtype):
    """caqr_peer_exchange (the NVLink peer-store exchange, alternative to the NCCL
    all-gather) with P virtual ranks on one device (one cooperative launch, the
    kernel code of the per-rank call): every rank's stack must hold all P local
    R's in rank order bit for bit, for two consecutive epochs (both mailbox
    buffers), and the combine of any rank's stack must give the oracle's R of
    the whole matrix (DistTSQR's result)."""
    from paper_conf_ipps_andersonbdk11_b200 import dist as cdist

    tdt = torch.float32 if dtype == np.float32 else torch.float64
    code = caqr.CAQR_F32 if dtype == np.float32 else caqr.CAQR_F64
    bd = BOUNDS[dtype]
    mb_bytes = caqr.caqr_peer_mailbox_bytes(P, n, code)
    assert mb_bytes == 2 * P * n * n * np.dtype(dtype).itemsize
    mailboxes = [torch.full((mb_bytes // np.dtype(dtype).itemsize,), float("nan"), dtype=tdt, device="cuda")
                 for _ in range(P)]
    flags = [torch.zeros(P, dtype=torch.int32, device="cuda") for _ in range(P)]
    for epoch, seed in ((1, 200 + P), (2, 300 + P)):
        A = workloads.gaussian(m, n, seed=seed, dtype=dtype)
        Rs = []
        for p in range(P):
            s0, rows = cdist.shard_rows(m, P, p)
            Ap = caqr.colmajor_empty(rows, n, tdt)
            Ap.copy_(torch.from_numpy(A[s0:s0 + rows]))
            Rp, _ = caqr.caqr_factor(Ap)
            Rs.append(Rp)
        gathers = [caqr.colmajor_empty(P * n, n, tdt) for _ in range(P)]
        caqr.caqr_peer_exchange_emulate(Rs, mailboxes, flags, gathers, epoch)
        torch.cuda.synchronize()
        want = torch.cat([r for r in Rs], dim=0)  # (P n) x n stack in rank order
        for p in range(P):
            assert torch.equal(gathers[p], want), (epoch, p)
            assert torch.all(flags[p] == epoch)
        R, _ = caqr.caqr_combine(gathers[P - 1], P)
        torch.cuda.synchronize()
        Rn = R.cpu().double().numpy()
        Ro = oracle.normalize_signs(oracle.qr(A.astype(np.float64), want_q=False, acc=bd["acc"]))
        assert np.linalg.norm(oracle.normalize_signs(Rn) - Ro) / np.linalg.norm(Ro) <= bd["r"]


@pytest.mark.gpu
def test_peer_exchange_arguments(caqr):
    """Argument checks of the per-rank call (no launch on a bad argument)."""
    R = caqr.colmajor_empty(8, 8, torch.float32)
    g = caqr.colmajor_empty(16, 8, torch.float32)
    ptrs = torch.zeros(2, dtype=torch.int64, device="cuda")
    L = caqr.lib()
    assert L.caqr_peer_exchange_f32(0, 0, 8, R.data_ptr(), 8, ptrs.data_ptr(), ptrs.data_ptr(), g.data_ptr(),
                                    1, None, 0, None) == -1
    assert L.caqr_peer_exchange_f32(2, 2, 8, R.data_ptr(), 8, ptrs.data_ptr(), ptrs.data_ptr(), g.data_ptr(),
                                    1, None, 0, None) == -2
    assert L.caqr_peer_exchange_f32(2, 0, 8, R.data_ptr(), 4, ptrs.data_ptr(), ptrs.data_ptr(), g.data_ptr(),
                                    1, None, 0, None) == -5
    assert L.caqr_peer_exchange_f32(2, 0, 8, R.data_ptr(), 8, ptrs.data_ptr(), ptrs.data_ptr(), g.data_ptr(),
                                    0, None, 0, None) == -9
    assert L.caqr_peer_exchange_f32(2, 0, 0, R.data_ptr(), 8, ptrs.data_ptr(), ptrs.data_ptr(), g.data_ptr(),
                                    1, None, 0, None) == 0
