"""GPU parity of least squares through CAQR (caqr_lstsq_*, caqr_trsm_upper_*;
SURVEY 8(f) f4, xGELS semantics) against the oracle
(oracle/lstsq.py: its own Householder QR + back substitution)."""
import numpy as np
import pytest

from oracle import lstsq as ol
from paper_conf_ipps_andersonbdk11_b200 import workloads

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def caqr():
    from paper_conf_ipps_andersonbdk11_b200 import build
    from paper_conf_ipps_andersonbdk11_b200 import caqr as c

    build.build()
    return c


def _dev(c, A, dt):
    t = c.colmajor_empty(A.shape[0], A.shape[1], dt)
    t.copy_(torch.from_numpy(np.ascontiguousarray(A)))
    return t


@pytest.mark.parametrize("n,k", [(1, 1), (7, 3), (192, 5), (1000, 2)])
@pytest.mark.parametrize("dtype", [np.float32, np.float64], ids=["f32", "f64"])
def test_trsm_upper(caqr, n, k, dtype):
    rng = np.random.default_rng(n)
    R = np.triu(rng.standard_normal((n, n))) + np.diag(np.sign(rng.standard_normal(n)) * (2.0 + n ** 0.5))
    R = R.astype(dtype)
    X0 = rng.standard_normal((n, k))
    B = (R.astype(np.float64) @ X0).astype(dtype)
    tdt = torch.float32 if dtype == np.float32 else torch.float64
    Bd = _dev(caqr, B, tdt)
    caqr.caqr_trsm_upper(_dev(caqr, R, tdt), Bd)
    X = Bd.cpu().double().numpy()
    Xo = ol.back_substitute(R.astype(np.float64), B.astype(np.float64))
    tol = 1e-4 if dtype == np.float32 else 1e-12
    assert np.linalg.norm(X - Xo) <= tol * np.linalg.norm(Xo)


@pytest.mark.parametrize("m,n,k,dtype", [(20_000, 48, 3, np.float32), (110_592, 100, 2, np.float32),
                                         (4_000_000, 8, 1, np.float32), (30_000, 40, 2, np.float64)])
def test_lstsq_vs_oracle(caqr, m, n, k, dtype):
    tdt = torch.float32 if dtype == np.float32 else torch.float64
    A = workloads.gaussian(m, n, seed=m % 11, dtype=dtype)
    B = workloads.gaussian(m, k, seed=m % 7 + 1, dtype=dtype)
    if m > 1_000_000:  # oracle on a size it finishes in seconds: same plan family, sampled rows
        A, B = A[:300_000], B[:300_000]
        m = A.shape[0]
    Ad = _dev(caqr, A, tdt)
    R, ws = caqr.caqr_factor(Ad)
    Bd = _dev(caqr, B, tdt)
    caqr.caqr_lstsq(Ad, ws, Bd)
    out = Bd.cpu().double().numpy()
    X, res = out[:n], np.linalg.norm(out[n:], axis=0)
    Xo, reso = ol.lstsq(A.astype(np.float64), B.astype(np.float64), acc="d" if dtype == np.float32 else "ld")
    tol = 1e-4 if dtype == np.float32 else 1e-11
    assert np.linalg.norm(X - Xo) <= tol * np.linalg.norm(Xo)
    assert np.abs(res - reso).max() <= tol * reso.max()
    # normal equations of the GPU solution, in float64: A^T (A x - b) ~ 0
    g = A.astype(np.float64).T @ (A.astype(np.float64) @ X - B.astype(np.float64))
    assert np.abs(g).max() <= (1e-3 if dtype == np.float32 else 1e-9) * np.linalg.norm(A) * np.linalg.norm(B)


def test_lstsq_consistent_system(caqr):
    """b = A x0 exactly (in fp64): the solution is x0, the residual 0."""
    rng = np.random.default_rng(2)
    m, n = 50_000, 24
    A = rng.standard_normal((m, n))
    x0 = rng.standard_normal((n, 2))
    Ad = _dev(caqr, A, torch.float64)
    R, ws = caqr.caqr_factor(Ad)
    Bd = _dev(caqr, A @ x0, torch.float64)
    caqr.caqr_lstsq(Ad, ws, Bd)
    out = Bd.cpu().numpy()
    assert np.abs(out[:n] - x0).max() <= 1e-12
    assert np.linalg.norm(out[n:]) <= 1e-11 * np.linalg.norm(A @ x0)
