"""Pins for the oracle's Siddon tracer (sec. 2.3; readings R1-R5 in DESIGN.md).

Each pin is independent of the tracer's own arithmetic:
* closed-form chord of a line through the square grid (row sums of A);
* a brute-force dense A by Liang-Barsky clipping of each ray against every pixel square;
* Table 3's printed "regular data" footprints;
* the adjoint identity with an A^T built by a separate sort-based transpose.
"""
import math

import numpy as np
import pytest

from conftest import read_golden


def chord(theta, t, L):
    """Length of the line {p : p.(cos th, sin th) = t} inside [-L, L]^2 (closed form)."""
    cp, sp = abs(math.cos(theta)), abs(math.sin(theta))
    c1, s1 = max(cp, sp), min(cp, sp)
    tau = abs(t)
    if s1 == 0.0:
        return 2 * L if tau < L else 0.0
    if tau <= L * (c1 - s1):
        return 2 * L / c1
    if tau < L * (c1 + s1):
        return (L * (c1 + s1) - tau) / (c1 * s1)
    return 0.0


GEOMS = [(64, 90, 64), (8, 8, 8), (8, 7, 8), (16, 12, 16), (33, 17, 33), (16, 5, 23),
         (1, 3, 1), (12, 1, 12), (15, 9, 14)]


@pytest.mark.parametrize("n,m,c", GEOMS)
def test_row_sums_equal_closed_form_chord(orc, n, m, c):
    L = n / 2.0
    worst = 0.0
    for ray in range(m * c):
        mm, k = divmod(ray, c)
        th = mm * math.pi / m
        t = (k + 0.5) - c / 2.0
        _, ln = orc.trace_ray(n, m, c, ray)
        ch = chord(th, t, L)
        err = abs(ln.sum() - ch) / max(1.0, ch)
        worst = max(worst, err)
        assert np.all(ln > 1e-9)
    assert worst <= 1e-12, worst


def dense_bruteforce(n, m, c):
    """Dense A by clipping each ray against each pixel square (independent of Siddon's traversal)."""
    L = n / 2.0
    A = np.zeros((m * c, n * n))
    jj, ii = np.meshgrid(np.arange(n), np.arange(n))
    x0 = (jj - L).ravel().astype(np.float64)
    y0 = (ii - L).ravel().astype(np.float64)
    for ray in range(m * c):
        mm, k = divmod(ray, c)
        th = mm * math.pi / m
        cs, sn = math.cos(th), math.sin(th)
        t = (k + 0.5) - c / 2.0
        px, py = t * cs, t * sn
        dx, dy = -sn, cs
        lo = np.full(n * n, -np.inf)
        hi = np.full(n * n, np.inf)
        for p, d, b0 in ((px, dx, x0), (py, dy, y0)):
            if abs(d) < 1e-15:
                inside = (b0 < p) & (p < b0 + 1)
                lo = np.where(inside, lo, np.inf)
            else:
                t1 = (b0 - p) / d
                t2 = (b0 + 1 - p) / d
                lo = np.maximum(lo, np.minimum(t1, t2))
                hi = np.minimum(hi, np.maximum(t1, t2))
        ln = np.where(hi > lo, hi - lo, 0.0)
        A[ray] = np.where(ln > 1e-9, ln, 0.0)
    return A


@pytest.mark.parametrize("n,m,c", [(8, 8, 8), (8, 7, 8), (16, 12, 16), (9, 6, 11)])
def test_matches_bruteforce_dense(orc, n, m, c):
    rows, cols, vals = orc.trace_all(n, m, c)
    A = np.zeros((m * c, n * n))
    A[rows, cols] = vals
    # each (ray, pixel) at most once: a line meets a convex pixel in one interval
    assert len(set(zip(rows.tolist(), cols.tolist()))) == len(rows)
    B = dense_bruteforce(n, m, c)
    assert np.array_equal(A != 0, B != 0)
    assert np.max(np.abs(A - B)) <= 1e-12


def _table3():
    out = {}
    for name, m, n, val, unit in read_golden("table3_footprints.txt"):
        out[name] = (int(m), int(n), val, unit)
    return out


def _rounds_to_printed(nbytes, printed, unit):
    scale = {"MiB": 2 ** 20, "GiB": 2 ** 30}[unit]
    decimals = len(printed.split(".")[1]) if "." in printed else 0
    return round(nbytes / scale, decimals) == float(printed)


def test_table3_ads1_footprint(orc):
    m, n, printed, unit = _table3()["ADS1"]
    nnz = orc.count_nnz(n, m, n)
    assert _rounds_to_printed(8 * nnz, printed, unit)
    assert nnz == 28_200_696  # regression value of this reading


@pytest.mark.slow
def test_table3_ads2_footprint(orc):
    m, n, printed, unit = _table3()["ADS2"]
    nnz = orc.count_nnz(n, m, n)
    assert _rounds_to_printed(8 * nnz, printed, unit)
    assert nnz == 235_014_288


def test_nnz_ratio_and_row_length_bounds(orc):
    n, m, c = 64, 90, 64
    rl = orc.row_lengths(n, m, c)
    assert rl.max() <= 2 * n - 1
    assert rl.min() > 0            # C = N: every ray crosses the grid
    ratio = rl.sum() / (m * n * n)
    assert 1.18 < ratio < 1.20


def test_adjoint_identity(orc, coo_cache):
    n, m, c = 64, 90, 64
    rows, cols, vals = coo_cache(n, m, c)
    rng = np.random.default_rng(0)
    x = rng.standard_normal(n * n)
    y = rng.standard_normal(m * c)
    Ax = orc.spmv_coo(rows, cols, vals, x, m * c)
    # A^T through the sort-based transpose + canonical row sums (a different code path)
    key = np.arange(m * c, dtype=np.int64)
    ATy = orc.spmv_canonical(cols, rows, vals, key, y, n * n)
    lhs, rhs = float(Ax @ y), float(x @ ATy)
    assert abs(lhs - rhs) <= 1e-12 * max(abs(lhs), 1.0)


def test_spmv_matches_dense_product(orc):
    n, m, c = 16, 12, 16
    rows, cols, vals = orc.trace_all(n, m, c)
    B = dense_bruteforce(n, m, c)
    x = np.random.default_rng(1).standard_normal(n * n)
    y = orc.spmv_coo(rows, cols, vals, x, m * c)
    assert np.allclose(y, B @ x, rtol=0, atol=1e-11)
    yt = np.random.default_rng(2).standard_normal(m * c)
    xt = orc.spmv_coo(cols, rows, vals, yt, n * n)
    assert np.allclose(xt, B.T @ yt, rtol=0, atol=1e-11)
    key = np.random.default_rng(3).permutation(n * n).astype(np.int64)
    yc = orc.spmv_canonical(rows, cols, vals, key, x, m * c)
    assert np.allclose(yc, B @ x, rtol=0, atol=1e-11)


def test_degenerate_geometries(orc):
    # C > N: outer rays miss the grid -> empty rows (all-zero rows are legal, C.3)
    rl = orc.row_lengths(8, 4, 14)
    assert (rl == 0).any() and (rl > 0).any()
    # N = 1: one pixel; every crossing ray has a single entry
    rows, cols, vals = orc.trace_all(1, 3, 1)
    assert set(cols.tolist()) == {0}
    # M = 1 (theta = 0 only): vertical rays, each crosses N pixels with length 1
    rows, cols, vals = orc.trace_all(6, 1, 6)
    assert len(rows) == 36 and np.allclose(vals, 1.0)
