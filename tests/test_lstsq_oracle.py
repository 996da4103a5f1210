"""Pins for the least-squares oracle (oracle/lstsq.py), -m "not gpu"."""
import numpy as np

from oracle import lstsq as ol
from paper_conf_ipps_andersonbdk11_b200 import workloads


def test_closed_form_3x2():
    # A = [[1,0],[0,1],[1,1]], b = [1,2,4]: A^T A = [[2,1],[1,2]], A^T b = [5,6]
    # -> x = [4/3, 7/3]; residual b - A x = [-1/3, -1/3, 1/3], norm 1/sqrt(3)
    A = np.array([[1.0, 0.0], [0.0, 1.0], [1.0, 1.0]])
    b = np.array([1.0, 2.0, 4.0])
    X, res = ol.lstsq(A, b)
    assert np.abs(X[:, 0] - [4 / 3, 7 / 3]).max() <= 1e-15
    assert abs(res[0] - 1 / np.sqrt(3)) <= 1e-15


def test_against_numpy_gelsd():
    A = workloads.gaussian(500, 12, seed=3).astype(np.float64)
    B = workloads.gaussian(500, 3, seed=4).astype(np.float64)
    X, res = ol.lstsq(A, B)
    Xn, rn, _, _ = np.linalg.lstsq(A, B, rcond=None)
    assert np.abs(X - Xn).max() <= 1e-13
    assert np.abs(res ** 2 - rn).max() <= 1e-11 * rn.max()


def test_consistent_system_and_normal_equations():
    rng = np.random.default_rng(0)
    A = rng.standard_normal((300, 20))
    x0 = rng.standard_normal((20, 2))
    X, res = ol.lstsq(A, A @ x0)
    assert np.abs(X - x0).max() <= 1e-13 and res.max() <= 1e-12
    b = rng.standard_normal((300, 1))
    X, _ = ol.lstsq(A, b)
    assert np.abs(A.T @ (A @ X - b)).max() <= 1e-11


def test_back_substitution():
    R = np.array([[2.0, 1.0, -1.0], [0.0, 4.0, 2.0], [0.0, 0.0, 5.0]])
    x = np.array([1.0, -2.0, 3.0])
    assert np.array_equal(ol.back_substitute(R, R @ x)[:, 0], x)
