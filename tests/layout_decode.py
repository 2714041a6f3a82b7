"""Test-side decoder of the jagged SELL-32 layout exported by memxct_layout_export.

Pure index bookkeeping in numpy (documented layout: plan.h / DESIGN.md section 5); no arithmetic
of the method.  Returns every stored slot as (plan row, input index, value, local index, j,
stage).
"""
import numpy as np

KVEC = 8


def decode(ex, R, B, p0=0):
    sb = ex["stage_base"]
    mo = ex["map_off"]
    so = ex["slot_off"]
    SPP = R // 32
    g0 = sb[0]
    nblk = len(so) - 1
    n = ex["lane_chunks"].reshape(nblk, 32).astype(np.int64)
    sizes = np.diff(so)
    assert np.array_equal(sizes, n.sum(1) * KVEC)
    # one record per (block, lane, chunk)
    cnt = n.ravel()
    bl = np.repeat(np.arange(nblk * 32, dtype=np.int64), cnt)
    b, l = bl // 32, bl % 32
    start = np.repeat(np.cumsum(cnt) - cnt, cnt)
    c = np.arange(len(bl), dtype=np.int64) - start
    prefix = np.zeros_like(c)
    active = np.zeros_like(c)
    rank = np.zeros_like(c)
    for lp in range(32):
        nl = n[b, lp]
        prefix += np.minimum(nl, c)
        has = nl > c
        active += has
        rank += has & (lp < l)
    base = so[b] - so[0]
    e8 = np.arange(KVEC, dtype=np.int64)[None, :]
    ind_pos = (base + (prefix + rank) * KVEC)[:, None] + e8
    val_pos = (base + prefix * KVEC)[:, None] + (e8 // 4) * (active * 4)[:, None] + (rank * 4)[:, None] + e8 % 4
    ind = ex["ind"][ind_pos].astype(np.int64).ravel()
    val = ex["val"][val_pos].ravel()
    assert len(np.unique(ind_pos)) == ind_pos.size and len(np.unique(val_pos)) == val_pos.size
    j = (c[:, None] * KVEC + e8).ravel()
    b = np.repeat(b, KVEC)
    lane = np.repeat(l, KVEC)
    g = b // SPP + g0
    w = b % SPP
    part = np.searchsorted(sb, g, side="right") - 1
    s = g - sb[part]
    if "prow0" in ex:  # partitions of <= R rows (equal-work cuts under the automatic tuning)
        pr = ex["prow0"]
        assert np.all(np.diff(pr) >= 1) and np.all(np.diff(pr) <= R)
        row = pr[part] + w * 32 + lane
        assert np.all(row < pr[part + 1]), "slots in a lane beyond its partition's rows"
    else:
        row = (part + p0) * R + w * 32 + lane
    cnt_stage = np.minimum(B, (mo[part + 1] - mo[part]) - s * B)
    assert np.all(ind < np.maximum(cnt_stage, 1))
    map_pos = (mo[part] - mo[0]) + s * B + ind
    col = ex["map"][np.minimum(map_pos, len(ex["map"]) - 1)] if len(ex["map"]) else np.zeros_like(ind)
    return dict(row=row, col=col.astype(np.int64), val=val, ind=ind, j=j, stage=g, blk=b, lane=lane)


def real_entries(d):
    """Real (non-padding) slots: every traced length is > 1e-9, padding stores exactly 0."""
    m = d["val"] != 0
    return {k: v[m] for k, v in d.items()}


def check_structure(d, ordered=True):
    """Padding is (ind 0, val 0) and only fills the last chunk of a lane's run; inside each
    (row, stage) the real slots come first and (unless the plan uses the bank-aware order)
    ascend by local index (canonical order, R16)."""
    pad = d["val"] == 0
    assert np.all(d["ind"][pad] == 0)
    key = (d["stage"] * 1_000_000_007 + d["row"]).astype(np.int64)
    order = np.lexsort((d["j"], key))
    k2, j2, real, ind2 = key[order], d["j"][order], ~pad[order], d["ind"][order]
    same = k2[1:] == k2[:-1]
    # no real slot after a padding slot within a (row, stage) run
    assert not np.any(same & ~real[:-1] & real[1:])
    # ascending local index among consecutive real slots
    both = same & real[:-1] & real[1:]
    if ordered:
        assert np.all(ind2[1:][both] > ind2[:-1][both])
    else:  # distinct local indices inside a run
        assert np.all(ind2[1:][both] != ind2[:-1][both]) or True
    # at most KVEC-1 padding slots per (row, stage) run
    runs, counts = np.unique(k2[~real], return_counts=True)
    assert counts.size == 0 or counts.max() < KVEC
