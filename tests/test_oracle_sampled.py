"""Pins for the oracle's sampled rows / columns, closed-form chord and threaded CPU-baseline SpMV
(SURVEY 8(c) C.4 "Large configs": the full-size parity checks compare sampled rows of A x and of
A^T y, and chord sums on every row, because the oracle cannot hold all of A at configs 3-5).

Each pin compares against something other than the function itself:
* orc_sample_columns (rows of A^T) against the columns of the full transpose of orc_trace_all --
  for >= 500 pixels on configs 1 and 2 and on odd / C > N geometries -- so a candidate-window
  rule that is too narrow (a missed ray) or a wrong ray index fails;
* orc_sample_rows against orc_trace_all's rows;
* orc_chord against Liang-Barsky clipping of the line against the square [-L, L]^2 (an
  independent computation) and against the tracer's row sums;
* orc_spmv_csr_threaded bit-identical to orc_spmv_coo (the plain Listing 2 product).
"""
import math

import numpy as np
import pytest
import scipy.sparse as sp

GEOMS = [(64, 90, 64), (33, 17, 33), (15, 9, 14), (8, 4, 14), (16, 5, 23), (1, 3, 1), (12, 1, 12)]


def _transpose(rows, cols, vals, n, m, c):
    return sp.csr_matrix((vals, (cols.astype(np.int64), rows.astype(np.int64))), shape=(n * n, m * c))


def _check_columns(orc, n, m, c, pixels, AT):
    ptr, rays, ln = orc.sample_columns(n, m, c, pixels, threads=4)
    assert len(ptr) == len(pixels) + 1
    for q, p in enumerate(pixels):
        row = AT.getrow(int(p))
        o = np.argsort(row.indices)
        assert np.array_equal(rays[ptr[q]:ptr[q + 1]], row.indices[o]), (n, m, c, p)
        assert np.array_equal(ln[ptr[q]:ptr[q + 1]], row.data[o]), (n, m, c, p)   # identical values


@pytest.mark.parametrize("n,m,c", GEOMS)
def test_sampled_columns_equal_full_transpose(orc, coo_cache, n, m, c):
    rows, cols, vals = coo_cache(n, m, c)
    AT = _transpose(rows, cols, vals, n, m, c)
    rng = np.random.default_rng(n * 1000 + m)
    pixels = rng.permutation(n * n)[:max(500, 0)]          # all pixels when n*n <= 500
    _check_columns(orc, n, m, c, pixels, AT)


def test_sampled_columns_cfg2(orc, coo_cache):
    """Config 2 (ADS1 shape, 256^2, 360 x 256): 600 random pixels plus two 8 x 8 blocks and the
    four corners (pixels the extreme rays graze)."""
    n, m, c = 256, 360, 256
    rows, cols, vals = coo_cache(n, m, c)
    AT = _transpose(rows, cols, vals, n, m, c)
    rng = np.random.default_rng(2)
    pix = set(rng.choice(n * n, 600, replace=False).tolist())
    for (i0, j0) in [(0, 0), (120, 64)]:
        pix |= {(i0 + a) * n + j0 + b for a in range(8) for b in range(8)}
    pix |= {0, n - 1, n * (n - 1), n * n - 1}
    _check_columns(orc, n, m, c, np.array(sorted(pix), np.int64), AT)


def test_sampled_columns_reject_repeats(orc):
    with pytest.raises(ValueError):
        orc.sample_columns(8, 4, 8, [3, 5, 3])


@pytest.mark.parametrize("n,m,c", [(64, 90, 64), (33, 17, 33), (8, 4, 14)])
def test_sampled_rows_equal_trace_all(orc, coo_cache, n, m, c):
    rows, cols, vals = coo_cache(n, m, c)
    rng = np.random.default_rng(7)
    rays = rng.choice(m * c, min(500, m * c), replace=False)
    ptr, pix, ln = orc.sample_rows(n, m, c, rays, threads=3)
    starts = np.searchsorted(rows, np.arange(m * c + 1))
    for i, r in enumerate(rays):
        a, b = starts[r], starts[r + 1]
        assert np.array_equal(pix[ptr[i]:ptr[i + 1]], cols[a:b])
        assert np.array_equal(ln[ptr[i]:ptr[i + 1]], vals[a:b])


def _clip_chord(theta, t, L):
    """Liang-Barsky: length of the line p(a) = t (cos, sin) + a (-sin, cos) inside [-L, L]^2."""
    cs, sn = math.cos(theta), math.sin(theta)
    p0, d = (t * cs, t * sn), (-sn, cs)
    lo, hi = -math.inf, math.inf
    for a in range(2):
        if abs(d[a]) < 1e-15:
            if not (-L < p0[a] < L):
                return 0.0
            continue
        t1, t2 = (-L - p0[a]) / d[a], (L - p0[a]) / d[a]
        lo, hi = max(lo, min(t1, t2)), min(hi, max(t1, t2))
    return max(0.0, hi - lo)


@pytest.mark.parametrize("n,m,c", [(64, 90, 64), (33, 17, 33), (8, 4, 14), (12, 1, 12), (1024, 1500, 1024)])
def test_chord_closed_form_against_clipping(orc, n, m, c):
    L = n / 2.0
    rng = np.random.default_rng(c)
    rays = rng.choice(m * c, min(3000, m * c), replace=False)
    ch = orc.chords(n, m, c)
    for r in rays:
        mm, k = divmod(int(r), c)
        ref = _clip_chord(mm * math.pi / m, (k + 0.5) - c / 2.0, L)
        assert abs(ch[r] - ref) <= 1e-12 * max(1.0, ref), (r, ch[r], ref)
        assert orc.chord(n, m, c, int(r)) == ch[r]


@pytest.mark.parametrize("n,m,c", [(64, 90, 64), (33, 17, 33), (8, 4, 14)])
def test_chord_equals_tracer_row_sums(orc, coo_cache, n, m, c):
    rows, cols, vals = coo_cache(n, m, c)
    sums = np.bincount(rows, vals, minlength=m * c)
    ch = orc.chords(n, m, c)
    assert np.all(np.abs(sums - ch) <= 1e-12 * np.maximum(1.0, ch))


@pytest.mark.parametrize("threads", [1, 3, 8])
def test_threaded_spmv_bit_identical_to_coo(orc, coo_cache, threads):
    n, m, c = 64, 90, 64
    rows, cols, vals = coo_cache(n, m, c)             # ray-major: rows ascending, trace order
    x = np.random.default_rng(1).standard_normal(n * n)
    ptr = np.searchsorted(rows, np.arange(m * c + 1)).astype(np.int64)
    y, nt = orc.spmv_csr_threaded(ptr, cols, vals, x, threads)
    assert nt == threads
    assert np.array_equal(y, orc.spmv_coo(rows, cols, vals, x, m * c))
    # the transposed product through a stable CSR of A^T equals the COO scatter order too
    tp, tc, tv = orc.coo_to_csr(cols, rows, vals, n * n)
    yt = np.random.default_rng(2).standard_normal(m * c)
    xb, _ = orc.spmv_csr_threaded(tp, tc, tv, yt, threads)
    assert np.array_equal(xb, orc.spmv_coo(cols, rows, vals, yt, n * n))


def test_csr_transpose_equals_sort_based(orc, coo_cache):
    n, m, c = 33, 17, 33
    rows, cols, vals = coo_cache(n, m, c)
    ptr = np.searchsorted(rows, np.arange(m * c + 1)).astype(np.int64)
    tp, tc, tv = orc.csr_transpose(ptr, cols, vals, n * n)
    rp, rc, rv = orc.coo_to_csr(cols, rows, vals, n * n)
    assert np.array_equal(tp, rp) and np.array_equal(tc, rc) and np.array_equal(tv, rv)
