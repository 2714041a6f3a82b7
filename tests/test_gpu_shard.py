"""Shard probe (memxct_plan_set_shard): one rank's part of a P-way decomposition A = R C A_p
 built alone on one device.

* At small sizes every rank's shard is checked against the same rank of a virtual-rank group
  (the build a real P-rank job runs): identical tile ranges, footprint rays, exchange counts and
  maps, layouts, and bit-identical A_p / A_p^T products.
* A_p alone is checked against the fp64 oracle: footprint ray i's partial is the oracle row of
  that ray restricted to the rank's pixels (its Hilbert range, from the oracle's own ordering).
* At config 5 (11293^2, 360 x 11293, BASELINE configs[4]; A_p of one of 8 ranks holds ~6.9e9
  nonzeros), where no single GPU holds A: the tomogram and sinogram Hilbert permutations in full
  against the oracle, and sampled footprint rows / local pixels of A_p and A_p^T against the
  oracle's own traces ("large configs")."""
import numpy as np
import pytest

from conftest import rel_l2
from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
from test_gpu_multirank import build_group, run_ranks

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_hidayetoglubgrg19_b200 import build_ext
    build_ext.build()


def shard(n, m, c, rank, nranks, **kw):
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    return MemXCT(n, m, c, rank=rank, nranks=nranks, shard=True, vector_order="plan", **kw).build()


def local_hilbert_range(orc_rank, lo, hi):
    """Natural indices whose oracle Hilbert position lies in [lo, hi), in Hilbert order."""
    sel = np.nonzero((orc_rank >= lo) & (orc_rank < hi))[0]
    return sel[np.argsort(orc_rank[sel], kind="stable")]


@pytest.mark.parametrize("geom,nranks", [((64, 90, 64), 3), ((256, 360, 256), 4), ((33, 17, 33), 2)])
def test_shard_equals_virtual_rank(geom, nranks):
    n, m, c = geom
    g, plans = build_group(n, m, c, nranks)
    x = inputs.uniform(n * n, 11)
    y = inputs.uniform(m * c, 12)
    for r, vp in enumerate(plans):
        sp = shard(n, m, c, r, nranks)
        for d in (0, 1):
            assert np.array_equal(sp.domain_ranges(d), vp.domain_ranges(d))
            assert np.array_equal(sp.local_indices(d), vp.local_indices(d))
        assert sp.exchange_info() == vp.exchange_info()
        cs, cv = sp.exchange_counts(), vp.exchange_counts()
        assert np.array_equal(cs["send"], cv["send"]) and np.array_equal(cs["recv"], cv["recv"])
        assert np.array_equal(sp.footprint_rays(), vp.footprint_rays())
        for d in (0, 1):
            assert sp.layout_info(d) == vp.layout_info(d)
        xl = torch.from_numpy(x[vp.local_indices(0)]).cuda()
        yf = torch.from_numpy(y[vp.footprint_rays()]).cuda()
        assert torch.equal(sp.footprint_forward(xl), vp.footprint_forward(xl))
        assert torch.equal(sp.footprint_back(yf), vp.footprint_back(yf))
        sp.close()
    # the footprint partials are exactly what the exchange sums: their reduction is A x
    xs = [torch.from_numpy(x[p.local_indices(0)]).cuda() for p in plans]
    parts = [p.footprint_forward(xs[r]) for r, p in enumerate(plans)]
    full = np.zeros(m * c)
    for p, v in zip(plans, parts):
        np.add.at(full, p.footprint_rays(), v.cpu().numpy().astype(np.float64))
    ys = run_ranks(nranks, lambda r: plans[r].forward(xs[r]))
    yg = np.zeros(m * c)
    for p, v in zip(plans, ys):
        yg[p.local_indices(1)] = v.cpu().numpy()
    assert rel_l2(yg, full) <= 1e-6


@pytest.mark.parametrize("nranks", [2, 4])
def test_shard_footprint_operators_vs_oracle(orc, coo_cache, nranks):
    n, m, c = 64, 90, 64
    rows, cols, vals = coo_cache(n, m, c)
    hr = orc.hilbert_rank(n, n, 8)
    x = inputs.uniform(n * n, 21).astype(np.float64)
    tot_nnz = 0
    for r in range(nranks):
        sp = shard(n, m, c, r, nranks)
        b = sp.domain_ranges(0)
        loc = local_hilbert_range(hr, b[r], b[r + 1])
        assert np.array_equal(sp.local_indices(0), loc)
        inside = (hr[cols] >= b[r]) & (hr[cols] < b[r + 1])
        tot_nnz += sp.layout_info(0)["nnz"]
        assert sp.layout_info(0)["nnz"] == int(inside.sum())
        fp = sp.footprint_rays()
        assert np.array_equal(np.sort(fp), np.unique(rows[inside]))   # rays crossing the local pixels
        xl = np.zeros(n * n)
        xl[loc] = x[loc]
        y_orc = orc.spmv_coo(rows, cols, vals, xl, m * c)[fp]
        y = sp.footprint_forward(torch.from_numpy(x[loc].astype(np.float32)).cuda()).cpu().numpy()
        assert rel_l2(y, y_orc) <= 1e-5
        yf = inputs.uniform(len(fp), 22 + r).astype(np.float64)
        yfull = np.zeros(m * c)
        yfull[fp] = yf
        x_orc = orc.spmv_coo(cols, rows, vals * inside, yfull, n * n)[loc]
        xb = sp.footprint_back(torch.from_numpy(yf.astype(np.float32)).cuda()).cpu().numpy()
        assert rel_l2(xb, x_orc) <= 1e-5
        sp.close()
    assert tot_nnz == len(rows)


def test_shard_rejects_whole_operators():
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, MemXCTError
    n, m, c = 32, 20, 32
    sp = shard(n, m, c, 1, 2)
    x = torch.zeros(sp.local_size(0), device="cuda")
    y = torch.zeros(sp.local_size(1), device="cuda")
    for call in (lambda: sp.forward(x), lambda: sp.back(y), lambda: sp.cg(y, 3), lambda: sp.exchange_time(2)):
        with pytest.raises(MemXCTError, match="UNSUPPORTED"):
            call()
    t = sp.spmv_time(3)
    assert t["fwd_us"] > 0 and t["back_us"] > 0
    with pytest.raises(MemXCTError, match="UNSUPPORTED"):
        MemXCT(n, m, c, rank=0, nranks=2, shard=True, vector_order="plan", exchange="peer").build()
    plain = MemXCT(n, m, c).build()
    with pytest.raises(MemXCTError, match="INVALID_ARG"):
        plain.footprint_rays()


@pytest.mark.slow
def test_cfg5_shards_full_size(orc):
    """Config 5 (BASELINE configs[4], 11293^2, 360 x 11293): A never fits one GPU, so every one
    of the 8 ranks' shards is built in turn on this GPU (the A_p each GPU of the 8-GPU job
    holds, ~6.9e9 nonzeros each).  SURVEY C.4 "large configs":
      * chord sums on EVERY ray: the footprint partials of a forward of ones, summed over the 8
        ranks' MIXED shards (fp64 sums of the stored fp32 lengths), equal the closed-form chord
        to <= 2e-7 per ray -- only the fp32 rounding of the lengths (<= 2^-24 relative), so the 8
        shards together hold every entry of A exactly once with its value.  (Sums of ~2.2e4
        positive terms in fp32 drift by ~1e-5 relative, which would hide a missing entry; the
        FP32 operator is gated by the sampled rows below, as at configs 3-4);
      * rank 3 (FP32, the default plan): the tomogram and sinogram Hilbert permutations in full
        against the oracle, 1e4 random footprint rows of A_p x and 1024 local pixels (16 8 x 8
        blocks) of A_p^T y against the oracle's own traces restricted to the rank's pixels
        (<= 1e-5 relative L2)."""
    import gc
    from fullsize import N_RAYS, chord_errors, pick_pixels, sampled_back_error, sampled_forward_error
    n, m, c = inputs.CONFIGS[5]
    nranks, r = 8, 3

    def fresh():
        gc.collect()
        torch.cuda.empty_cache()

    fresh()
    sp = shard(n, m, c, r, nranks)
    assert sp.get_option("ray_block") == 16        # 2 a* = 10.7 (a* = sqrt(1024 / (4100 pi / 360)))
    info = sp.layout_info(0)
    assert 0.9 < info["nnz"] * nranks / (1.1953 * m * c * n) < 1.1      # about 1/P of nnz(A)
    fp = sp.footprint_rays()
    tb, sb = sp.domain_ranges(0), sp.domain_ranges(1)
    hr_t = orc.hilbert_rank(n, n, sp.get_option("tile_tomo") or 64)
    loc = local_hilbert_range(hr_t, tb[r], tb[r + 1])
    assert np.array_equal(sp.local_indices(0), loc)
    hr_s = orc.hilbert_rank(m, c, sp.get_option("tile_sino") or 32)
    assert np.array_equal(sp.local_indices(1), local_hilbert_range(hr_s, sb[r], sb[r + 1]))
    del hr_s
    x = inputs.uniform(n * n, inputs.seed_for(5)).astype(np.float64)
    y = sp.footprint_forward(torch.from_numpy(x[loc].astype(np.float32)).cuda()).cpu().numpy()
    rng = np.random.default_rng(5)
    pick = rng.choice(len(fp), N_RAYS, replace=False)
    lo, hi = tb[r], tb[r + 1]
    e_fwd = sampled_forward_error(orc, n, m, c, fp[pick], y[pick], x,
                                  pixel_mask=lambda pix: (hr_t[pix] >= lo) & (hr_t[pix] < hi))
    yf = inputs.uniform(len(fp), inputs.seed_for(5) + 1).astype(np.float64)
    xb = sp.footprint_back(torch.from_numpy(yf.astype(np.float32)).cuda()).cpu().numpy()
    y_nat = np.full(m * c, np.nan)                 # rays outside the footprint: NaN
    y_nat[fp] = yf.astype(np.float32).astype(np.float64)
    pixels = pick_pixels(rng, n, anchors=loc)
    assert np.all((hr_t[pixels] >= lo) & (hr_t[pixels] < hi))
    pos = np.empty(n * n, np.int64)
    pos[loc] = np.arange(len(loc))
    e_back = sampled_back_error(orc, n, m, c, pixels, xb[pos[pixels]], lambda q: y_nat[q])
    print(f"cfg5 rank 3: {len(pick)} footprint rows {e_fwd:.2e}, {len(pixels)} pixels {e_back:.2e}")
    assert e_fwd <= 1e-5 and e_back <= 1e-5, (e_fwd, e_back)
    del hr_t, pos, x, y_nat
    sp.close()
    del sp

    row_sums = np.zeros(m * c, np.float64)
    nnz = 0
    for q in range(nranks):
        fresh()
        sq = shard(n, m, c, q, nranks, precision="mixed")
        nnz += sq.layout_info(0)["nnz"]
        part = sq.footprint_forward(torch.ones(sq.local_size(0), device="cuda", dtype=torch.float64))
        row_sums[sq.footprint_rays()] += part.cpu().numpy()
        sq.close()
        del sq
    assert abs(nnz / (m * c * n) - 1.1953) < 2e-3
    l2, per = chord_errors(orc, n, m, c, row_sums)
    print(f"cfg5 chord sums over 8 MIXED shards: rel L2 {l2:.2e}, worst ray {per:.2e}")
    assert per <= 2e-7, (l2, per)
