"""Pins for the oracle's SIRT.

* the first iterate in closed form, x_1 = C A^T R y, from a dense brute-force A;
* the fixed point: the weighted least-squares solution argmin ||R^(1/2) (y - A x)|| (numpy
  lstsq on the dense matrix) -- the stationary point of x += C A^T R (y - A x);
* residual norms reported for k = 0 (= ||y||) and consistency with the iterate.
"""
import numpy as np

from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
from test_oracle_siddon import dense_bruteforce


def test_sirt_first_iterate_closed_form(orc):
    n, m, c = 8, 7, 8
    rows, cols, vals = orc.trace_all(n, m, c)
    A = dense_bruteforce(n, m, c)
    y = np.random.default_rng(9).random(m * c)
    R = np.where(A.sum(1) > 0, 1.0 / np.maximum(A.sum(1), 1e-300), 0.0)
    C = np.where(A.sum(0) > 0, 1.0 / np.maximum(A.sum(0), 1e-300), 0.0)
    x1 = C * (A.T @ (R * y))
    x, res = orc.sirt(rows, cols, vals, y, m * c, n * n, 1)
    assert np.allclose(x, x1, rtol=0, atol=1e-12 * np.abs(x1).max())
    assert res[0] == np.linalg.norm(y) or abs(res[0] - np.linalg.norm(y)) <= 1e-14 * np.linalg.norm(y)
    assert abs(res[1] - np.linalg.norm(y - A @ x1)) <= 1e-12 * res[0]


def test_sirt_iterates_match_closed_form_around_weighted_lsq(orc):
    """x_k = (I - (I - G)^k) x*, G = C A^T R A, x* = argmin ||R^(1/2)(y - A x)|| (full rank)."""
    n, m, c = 8, 12, 8
    rows, cols, vals = orc.trace_all(n, m, c)
    A = dense_bruteforce(n, m, c)
    y = np.random.default_rng(10).random(m * c)
    r, cc = 1.0 / A.sum(1), 1.0 / A.sum(0)
    xs = np.linalg.lstsq(np.sqrt(r)[:, None] * A, np.sqrt(r) * y, rcond=None)[0]
    G = cc[:, None] * (A.T @ (r[:, None] * A))
    for k in (1, 7, 45, 400):
        xk = (np.eye(n * n) - np.linalg.matrix_power(np.eye(n * n) - G, k)) @ xs
        x, res = orc.sirt(rows, cols, vals, y, m * c, n * n, k)
        assert np.linalg.norm(x - xk) <= 1e-9 * np.linalg.norm(xk), k
    # the weighted normal equations hold at x*
    assert np.linalg.norm(A.T @ (r * (y - A @ xs))) <= 1e-10 * np.linalg.norm(A.T @ (r * y))


def test_sirt_reduces_residual_on_phantom(orc, coo_cache):
    n, m, c = 64, 90, 64
    rows, cols, vals = coo_cache(n, m, c)
    xt = inputs.shepp_logan(n)
    y = orc.spmv_coo(rows, cols, vals, xt, m * c)
    x, res = orc.sirt(rows, cols, vals, y, m * c, n * n, 45)
    assert res[-1] < 0.1 * res[0]
    assert np.linalg.norm(x - xt) < np.linalg.norm(xt)
