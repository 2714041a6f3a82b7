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
def test_cfg5_shard_sampled_rows(orc):
    """Config 5 (BASELINE configs[4]), rank 3 of 8, the shard a GPU of the 8-GPU job holds."""
    n, m, c = inputs.CONFIGS[5]
    nranks, r = 8, 3
    sp = shard(n, m, c, r, nranks)
    # Hilbert permutations of both domains, in full, against the oracle (bit-exact)
    tb, sb = sp.domain_ranges(0), sp.domain_ranges(1)
    hr_t = orc.hilbert_rank(n, n, sp.get_option("tile_tomo") or 64)
    loc = local_hilbert_range(hr_t, tb[r], tb[r + 1])
    assert np.array_equal(sp.local_indices(0), loc)
    hr_s = orc.hilbert_rank(m, c, sp.get_option("tile_sino") or 32)
    assert np.array_equal(sp.local_indices(1), local_hilbert_range(hr_s, sb[r], sb[r + 1]))
    del hr_s
    assert sp.get_option("ray_block") == 16        # 2 a* = 10.7 (a* = sqrt(1024 / (4100 pi / 360)))
    info = sp.layout_info(0)
    assert 0.9 < info["nnz"] * nranks / (1.1953 * m * c * n) < 1.1      # about 1/P of nnz(A)
    fp = sp.footprint_rays()
    x = inputs.uniform(n * n, inputs.seed_for(5)).astype(np.float64)
    y = sp.footprint_forward(torch.from_numpy(x[loc].astype(np.float32)).cuda()).cpu().numpy()
    rng = np.random.default_rng(5)
    pick = rng.choice(len(fp), 2000, replace=False)
    got, exp = [], []
    for i in pick:
        pix, ln = orc.trace_ray(n, m, c, int(fp[i]))
        keep = (hr_t[pix] >= tb[r]) & (hr_t[pix] < tb[r + 1])
        assert keep.any()                                  # a footprint ray crosses a local pixel
        got.append(y[i])
        exp.append(float(ln[keep] @ x[pix[keep]]))
    assert rel_l2(np.array(got), np.array(exp)) <= 1e-5
    yf = inputs.uniform(len(fp), inputs.seed_for(5) + 1).astype(np.float64)
    xb = sp.footprint_back(torch.from_numpy(yf.astype(np.float32)).cuda()).cpu().numpy()
    pos = {int(v): i for i, v in enumerate(fp)}
    li = rng.choice(len(loc), 6, replace=False)
    got, exp = [], []
    for k, (rr, ll) in zip(li, orc.sampled_back_rows(n, m, c, loc[li])):
        got.append(xb[k])
        exp.append(float(sum(l * yf[pos[int(q)]] for q, l in zip(rr, ll))))   # every ray of a local pixel is in the footprint
    assert rel_l2(np.array(got), np.array(exp)) <= 1e-5
    sp.close()
