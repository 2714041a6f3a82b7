"""Full-size parity helpers ("Large configs (3-5), where the oracle cannot hold
A"): sampled rows of y = A x and of x = A^T y against the oracle's own traces
(orc_sample_rows / orc_sample_columns, pinned in tests/test_oracle_sampled.py), and row sums
against the closed-form chord (orc_chords).  Expected values come only from oracle/."""
import numpy as np

from conftest import rel_l2

N_RAYS = 10_000      # C.4: 1e4 random rays
N_PIXELS = 1024      # C.4: 1e3 random pixels, drawn as 16 random 8 x 8 blocks (8-aligned, so a
BLOCK = 8            # block lies in one Hilbert tile and hence on one rank)


def pick_pixels(rng, n, anchors=None, count=N_PIXELS, block=BLOCK):
    """`count` distinct natural pixel indices as count / block^2 random aligned blocks; anchors
    (natural indices, optional) restricts the block origins to blocks containing those pixels."""
    nb = count // (block * block)
    out = set()
    while len(out) < nb * block * block:
        if anchors is None:
            i0, j0 = (rng.integers(0, max(1, n // block), 2) * block).tolist()
        else:
            a = int(anchors[rng.integers(0, len(anchors))])
            i0, j0 = (a // n) // block * block, (a % n) // block * block
        blk = {(i0 + di) * n + (j0 + dj) for di in range(block) for dj in range(block)
               if i0 + di < n and j0 + dj < n}
        out |= blk
    return np.array(sorted(out), np.int64)[: nb * block * block]


def sampled_forward_error(orc, n, m, c, rays, y_gpu_rows, x_nat, pixel_mask=None):
    """rel L2 of the GPU's rows `y_gpu_rows` (one per ray in `rays`) against sum(len * x) over
    the oracle's trace of each ray (only pixels with pixel_mask True, if given)."""
    ptr, pix, ln = orc.sample_rows(n, m, c, rays)
    contrib = ln * x_nat[pix]
    if pixel_mask is not None:
        keep = pixel_mask(pix)
        # a footprint ray crosses at least one local pixel
        assert np.all(np.add.reduceat(keep.astype(np.int64), ptr[:-1]) > 0)
        contrib = np.where(keep, contrib, 0.0)
    exp = np.add.reduceat(contrib, ptr[:-1]) if len(contrib) else np.zeros(len(rays))
    exp[ptr[:-1] == ptr[1:]] = 0.0
    return rel_l2(np.asarray(y_gpu_rows, np.float64), exp)


def sampled_back_error(orc, n, m, c, pixels, x_gpu_pix, y_of_ray):
    """rel L2 of the GPU's pixel values against sum(len * y[ray]) over the oracle's column of
    each pixel; y_of_ray maps natural ray indices to input values (NaN = not available, which
    must not be reached)."""
    ptr, rays, ln = orc.sample_columns(n, m, c, pixels)
    vals = y_of_ray(rays.astype(np.int64))
    assert np.all(np.isfinite(vals)), "a ray crossing a sampled pixel has no input value"
    exp = np.add.reduceat(ln * vals, ptr[:-1])
    exp[ptr[:-1] == ptr[1:]] = 0.0
    return rel_l2(np.asarray(x_gpu_pix, np.float64), exp)


def chord_errors(orc, n, m, c, row_sums_nat):
    """(rel L2 over all rays, max per-ray |sum - chord| / max(1, chord)) of the row sums of the
    GPU-built A (forward of a vector of ones) against the closed-form chord of every ray."""
    ch = orc.chords(n, m, c)
    s = np.asarray(row_sums_nat, np.float64)
    per = np.abs(s - ch) / np.maximum(1.0, ch)
    return rel_l2(s, ch), float(per.max())
