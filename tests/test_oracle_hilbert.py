"""Pins for the oracle's two-level pseudo-Hilbert ordering (sec. 3.2; readings R6-R10).

* Fig. 4(a)'s printed tile-order fragments on the 13x11 / 4x4-tile example;
* the textbook 4x4 Hilbert curve (special case H = W = T = 2^k);
* bijection and edge-connectivity on many shapes;
* Fig. 6's data reuse and stage counts through Hilbert partitions;
* locality: Hilbert partitions touch far fewer distinct inputs than row-major ones.
"""
import numpy as np
import pytest

from conftest import read_golden


def order_from_rank(rank, h, w):
    """(row, col) visiting sequence from rank[i*w + j]."""
    seq = np.empty(h * w, np.int64)
    seq[rank] = np.arange(h * w)
    return np.stack([seq // w, seq % w], axis=1)


def test_fig4a_tile_order_fragments(orc):
    rows = read_golden("fig4a_tile_order.txt")
    frags = [list(map(int, r[1:])) for r in rows if r[0] == "fragment"]
    # 13 x 11 domain, 4 x 4 tiles -> 4 tile rows x 3 tile cols = 12 tiles
    xs, ys = orc.gilbert2d(3, 4)
    grid = np.full((4, 3), -1)
    grid[ys, xs] = np.arange(12)
    assert sorted(grid.ravel().tolist()) == list(range(12))
    tile_rows = [grid[r].tolist() for r in range(4)]
    for f in frags:
        assert f in tile_rows, (f, tile_rows)
    # consecutive tiles are edge neighbours (connectivity of subdomains)
    assert np.all(np.abs(np.diff(xs)) + np.abs(np.diff(ys)) == 1)
    # "subdomain 0 consists of tiles 0-2" is a connected set
    r = orc.hilbert_rank(13, 11, 4)
    assert sorted(r.tolist()) == list(range(143))


def test_textbook_hilbert_4x4(orc):
    pts = [tuple(map(int, r)) for r in read_golden("hilbert_4x4_textbook.txt")]
    assert [orc.d2xy(4, d) for d in range(16)] == pts
    # two-level ordering with a single 4x4 tile reduces to the textbook curve
    rank = orc.hilbert_rank(4, 4, 4)
    seq = order_from_rank(rank, 4, 4)
    assert [(int(c), int(r)) for r, c in seq] == pts
    # gilbert2d on a 2^k square is the textbook curve as well
    xs, ys = orc.gilbert2d(4, 4)
    assert list(zip(xs.tolist(), ys.tolist())) == pts


@pytest.mark.parametrize("k", [1, 2, 3, 4, 5])
def test_textbook_curve_properties(orc, k):
    n = 2 ** k
    pts = np.array([orc.d2xy(n, d) for d in range(n * n)])
    assert tuple(pts[0]) == (0, 0) and tuple(pts[-1]) == (n - 1, 0)
    assert len({tuple(p) for p in pts.tolist()}) == n * n
    assert np.all(np.abs(np.diff(pts, axis=0)).sum(1) == 1)
    # recursive structure: each quadrant is visited contiguously
    q = (pts[:, 0] >= n // 2).astype(int) * 2 + (pts[:, 1] >= n // 2)
    if n > 1:
        assert np.count_nonzero(np.diff(q)) == 3


@pytest.mark.parametrize("h,w,t", [(13, 11, 4), (90, 64, 8), (64, 64, 8), (256, 256, 32),
                                   (360, 256, 32), (7, 3, 4), (1, 1, 4), (5, 17, 2), (33, 31, 8)])
def test_two_level_bijection_and_connectivity(orc, h, w, t):
    rank = orc.hilbert_rank(h, w, t)
    assert np.array_equal(np.sort(rank), np.arange(h * w))
    seq = order_from_rank(rank, h, w)
    steps = np.abs(np.diff(seq, axis=0)).sum(1)
    full = (h % t == 0) and (w % t == 0)
    # full tiling by 2^k tiles: a fully edge-connected curve
    if full and ((h // t) & (h // t - 1)) == 0 and h == w:
        assert np.all(steps == 1)
    # jumps can only occur where a tile is clipped by the domain
    bad = np.nonzero(steps != 1)[0]
    for b in bad:
        r, c = seq[b]
        r2, c2 = seq[b + 1]
        clipped = lambda rr, cc: ((rr // t + 1) * t > h) or ((cc // t + 1) * t > w)
        assert clipped(r, c) or clipped(r2, c2)
    # tiles are contiguous ranges of the order
    tile = (seq[:, 0] // t) * ((w + t - 1) // t) + seq[:, 1] // t
    assert np.count_nonzero(np.diff(tile)) == len(np.unique(tile)) - 1


def test_many_small_shapes_bijective(orc):
    for h in range(1, 23, 3):
        for w in range(1, 23, 2):
            for t in (1, 2, 4):
                rank = orc.hilbert_rank(h, w, t)
                assert np.array_equal(np.sort(rank), np.arange(h * w))


def _partition_stats(rows_h, cols_h, nnz_rows, part_rows, nparts):
    """Per partition of `part_rows` consecutive Hilbert rows: (nnz, distinct inputs)."""
    pid = rows_h // part_rows
    key = pid.astype(np.int64) * (cols_h.max() + 1) + cols_h
    distinct = np.bincount(np.unique(key) // (cols_h.max() + 1), minlength=nparts)
    nnz = np.bincount(pid, minlength=nparts)
    return nnz, distinct


def test_fig6_data_reuse_and_stages(orc):
    g = {r[0]: float(r[1]) for r in read_golden("fig6_reuse.txt")}
    n, m, c, t = 256, 256, 256, 64
    rows, cols, vals = orc.trace_all(n, m, c)
    sino_rank = orc.hilbert_rank(m, c, t)      # rows of A: rays, sinogram (M x C) Hilbert order
    tomo_rank = orc.hilbert_rank(n, n, t)      # cols of A: pixels, tomogram Hilbert order
    rh = sino_rank[rows]
    ch = tomo_rank[cols]
    part = t * t                               # one 64 x 64 tile per partition (Fig. 6)
    B = int(g["buffer_entries"])
    # forward: sinogram partitions read the tomogram
    nnz_f, dist_f = _partition_stats(rh, ch, None, part, m * c // part)
    reuse_f = (nnz_f / dist_f).mean()
    # back: tomogram partitions read the sinogram
    nnz_b, dist_b = _partition_stats(ch, rh, None, part, n * n // part)
    reuse_b = (nnz_b / dist_b).mean()
    assert abs(reuse_f / g["forward_reuse"] - 1) < 0.05, reuse_f
    assert abs(reuse_b / g["back_reuse"] - 1) < 0.05, reuse_b
    st_f = -(-dist_f // B)
    st_b = -(-dist_b // B)
    assert set(st_f.tolist()) <= {3, 4} and g["forward_stages"] in st_f
    assert set(st_b.tolist()) <= {2, 3} and g["back_stages"] in st_b


def test_hilbert_partitions_touch_fewer_inputs(orc, coo_cache):
    n, m, c = 256, 360, 256
    rows, cols, vals = coo_cache(n, m, c)
    sino_rank = orc.hilbert_rank(m, c, 32)
    tomo_rank = orc.hilbert_rank(n, n, 32)
    R = 512
    nparts = -(-m * c // R)
    _, d_h = _partition_stats(sino_rank[rows], tomo_rank[cols], None, R, nparts)
    _, d_r = _partition_stats(rows.astype(np.int64), cols.astype(np.int64), None, R, nparts)
    assert d_r.mean() / d_h.mean() > 3.0
