"""Pins for the oracle's CGLS (sec. 3.5.2; readings R13-R16) and canonical sums.

* against the least-squares solution from a dense brute-force A (normal equations, numpy lstsq);
* the first iterate in closed form (exact line search along A^T y);
* monotone ||r_k|| and ||x_k - x_true|| on a consistent noiseless system (Shepp-Logan);
* recovery error to the phantom after 30 / 300 iterations (SURVEY 8(c) C.4 thresholds);
* canonical dots against math.fsum; canonical and plain CGLS agree early (order-only difference).
"""
import math

import numpy as np
import pytest

from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
from test_oracle_siddon import dense_bruteforce


def test_cgls_converges_to_lstsq_solution(orc):
    n, m, c = 8, 12, 8                    # 96 rays >= 64 pixels: full column rank
    rows, cols, vals = orc.trace_all(n, m, c)
    A = dense_bruteforce(n, m, c)
    y = np.random.default_rng(5).standard_normal(m * c)   # inconsistent: true least squares
    xs = np.linalg.lstsq(A, y, rcond=None)[0]
    x, res, tres, done = orc.cgls(rows, cols, vals, y, m * c, n * n, 200)
    assert np.linalg.norm(x - xs) <= 1e-8 * np.linalg.norm(xs)
    # normal-equation residual vanishes
    assert np.linalg.norm(A.T @ (y - A @ x)) <= 1e-8 * np.linalg.norm(A.T @ y)


def test_cgls_first_iterate_closed_form(orc):
    n, m, c = 8, 7, 8
    rows, cols, vals = orc.trace_all(n, m, c)
    A = dense_bruteforce(n, m, c)
    y = np.random.default_rng(6).standard_normal(m * c)
    g = A.T @ y
    x1 = (g @ g) / np.sum((A @ g) ** 2) * g
    x, res, tres, done = orc.cgls(rows, cols, vals, y, m * c, n * n, 1)
    assert np.allclose(x, x1, rtol=0, atol=1e-12 * np.abs(x1).max())
    assert res[0] == pytest.approx(np.linalg.norm(y), rel=1e-14)
    assert res[1] == pytest.approx(np.linalg.norm(y - A @ x1), rel=1e-10)


def test_cgls_zero_rhs_and_zero_iters(orc):
    n, m, c = 8, 8, 8
    rows, cols, vals = orc.trace_all(n, m, c)
    x, res, tres, done = orc.cgls(rows, cols, vals, np.zeros(m * c), m * c, n * n, 5)
    assert done == 0 and np.all(x == 0)
    x, res, tres, done = orc.cgls(rows, cols, vals, np.ones(m * c), m * c, n * n, 0)
    assert done == 0 and np.all(x == 0)


def _phantom_problem(orc, coo_cache, n, m, c):
    rows, cols, vals = coo_cache(n, m, c)
    xt = inputs.shepp_logan(n)
    y = orc.spmv_coo(rows, cols, vals, xt, m * c).astype(np.float32).astype(np.float64)
    return rows, cols, vals, xt, y


def test_cgls_monotone_and_recovers_phantom_cfg1(orc, coo_cache):
    n, m, c = 64, 90, 64
    rows, cols, vals, xt, y = _phantom_problem(orc, coo_cache, n, m, c)
    x, res, tres, done = orc.cgls(rows, cols, vals, y, m * c, n * n, 30)
    assert done == 30
    assert np.all(np.diff(res) <= 1e-12 * res[0])
    assert np.all(np.diff(tres) <= 1e-12 * tres[0])
    err = np.linalg.norm(x - xt) / np.linalg.norm(xt)
    assert err <= 0.12
    # ||x_k - x_true|| non-increasing (consistent system, A full column rank)
    errs = []
    for k in range(0, 31, 3):
        xk = orc.cgls(rows, cols, vals, y, m * c, n * n, k)[0]
        errs.append(np.linalg.norm(xk - xt))
    assert np.all(np.diff(errs) <= 1e-9)
    x300 = orc.cgls(rows, cols, vals, y, m * c, n * n, 300)[0]
    assert np.linalg.norm(x300 - xt) / np.linalg.norm(xt) <= 5e-3


@pytest.mark.slow
def test_cgls_recovers_phantom_cfg2(orc, coo_cache):
    n, m, c = 256, 360, 256
    rows, cols, vals, xt, y = _phantom_problem(orc, coo_cache, n, m, c)
    x, res, tres, done = orc.cgls(rows, cols, vals, y, m * c, n * n, 30)
    assert np.all(np.diff(res) <= 1e-12 * res[0])
    assert np.linalg.norm(x - xt) / np.linalg.norm(xt) <= 0.10


def test_dot_canonical_against_fsum(orc):
    rng = np.random.default_rng(7)
    a = rng.standard_normal(10001)
    b = rng.standard_normal(10001)
    key = rng.permutation(10001).astype(np.int64)
    exact = math.fsum((a * b).tolist())  # products rounded, then exactly summed
    for chunk in (1, 7, 512, 10001, 20000):
        d = orc.dot_canonical(a, b, key, chunk)
        assert abs(d - exact) <= 1e-12 * np.abs(a * b).sum()
    # chunk = 1: every partial is RN(a*b), partials added sequentially in key order
    acc = 0.0
    for i in np.argsort(key):
        acc = acc + float(a[i] * b[i])
    assert orc.dot_canonical(a, b, key, 1) == acc


def test_canonical_and_plain_cgls_agree_early(orc, coo_cache):
    n, m, c = 64, 90, 64
    rows, cols, vals, xt, y = _phantom_problem(orc, coo_cache, n, m, c)
    rk = orc.hilbert_rank(m, c, 8)
    ck = orc.hilbert_rank(n, n, 8)
    vals32 = vals.astype(np.float32).astype(np.float64)
    xa = orc.cgls(rows, cols, vals32, y, m * c, n * n, 10)[0]
    xb = orc.cgls(rows, cols, vals32, y, m * c, n * n, 10, canonical=True, row_key=rk,
                  col_key=ck, chunk_rows=256, chunk_cols=256)[0]
    assert np.linalg.norm(xa - xb) <= 1e-6 * np.linalg.norm(xa)
    # canonical mode is deterministic: identical on a second run
    xc = orc.cgls(rows, cols, vals32, y, m * c, n * n, 10, canonical=True, row_key=rk,
                  col_key=ck, chunk_rows=256, chunk_cols=256)[0]
    assert np.array_equal(xb, xc)
