"""Test-side decoder of the staged SELL-32 layout exported by memxct_layout_export.

Pure index bookkeeping in numpy (documented layout); no arithmetic of the
method.  Returns every stored slot as (plan row, input index, value, local index, j, stage).
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
    sizes = np.diff(so)
    assert np.all(sizes % (32 * KVEC) == 0)
    slot = np.arange(so[-1] - so[0], dtype=np.int64)
    blk = np.repeat(np.arange(nblk, dtype=np.int64), sizes)
    off = slot - (so[blk] - so[0])
    c, r = off // 256, off % 256
    lane, e8 = r // KVEC, r % KVEC
    j = c * KVEC + e8
    val_pos = (so[blk] - so[0]) + c * 256 + (e8 // 4) * 128 + lane * 4 + (e8 % 4)
    ind = ex["ind"].astype(np.int64)
    val = ex["val"][val_pos]
    g = blk // SPP + g0
    w = blk % SPP
    part = np.searchsorted(sb, g, side="right") - 1
    s = g - sb[part]
    row = (part + p0) * R + w * 32 + lane
    cnt = np.minimum(B, (mo[part + 1] - mo[part]) - s * B)
    assert np.all(ind < np.maximum(cnt, 1))
    map_pos = (mo[part] - mo[0]) + s * B + ind
    col = ex["map"][np.minimum(map_pos, len(ex["map"]) - 1)] if len(ex["map"]) else np.zeros_like(ind)
    return dict(row=row, col=col.astype(np.int64), val=val, ind=ind, j=j, stage=g, blk=blk, lane=lane)


def real_entries(d):
    """Real (non-padding) slots: every traced length is > 1e-9, padding stores exactly 0."""
    m = d["val"] != 0
    return {k: v[m] for k, v in d.items()}


def check_structure(d):
    """Padding is (ind 0, val 0); inside each (row, stage) the real slots come first and
    ascend by local index (canonical order, reading R16)."""
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
    assert np.all(ind2[1:][both] > ind2[:-1][both])
