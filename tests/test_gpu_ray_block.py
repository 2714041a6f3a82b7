"""Forward partitions over projection x channel blocks (MEMXCT_OPT_RAY_BLOCK).

The paper cuts A into partitions of R consecutive Hilbert rows.  With few
projections and a wide detector (config 5) such a ~square block of rays fans out across the
tomogram and shares few pixels, so the forward stage buffers are refilled for almost every
nonzero; blocks of `a` projections x R/a channels keep the fan narrow.  Only the grouping of rows
into partitions changes: every row still accumulates its entries in ascending Hilbert input order,
so FP32 projections are bit-identical to the Hilbert-row layout, and the vector layouts (natural,
plan, footprint) are unchanged."""
import numpy as np
import pytest

from conftest import rel_l2
from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
from test_gpu_multirank import build_group, gather, run_ranks, scatter

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_hidayetoglubgrg19_b200 import build_ext
    build_ext.build()


@pytest.mark.parametrize("geom", [(64, 90, 64), (256, 360, 256), (40, 7, 97)])
@pytest.mark.parametrize("order", ["natural", "plan"])
def test_blocked_rows_bit_identical(orc, coo_cache, geom, order):
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    n, m, c = geom
    ref = MemXCT(n, m, c, vector_order=order, ray_block=-1, stage_order=-1).build()
    assert ref.get_option("ray_block") == -1
    x = inputs.uniform(n * n, 31)
    xi = x if order == "natural" else x[ref.local_indices(0)]
    xt = torch.from_numpy(np.ascontiguousarray(xi)).cuda()
    y_ref = ref.forward(xt)
    rows, cols, vals = coo_cache(n, m, c)
    y_orc = orc.spmv_coo(rows, cols, vals, x.astype(np.float64), m * c)
    yo = y_ref.cpu().numpy() if order == "natural" else np.zeros(m * c)
    if order == "plan":
        yo[ref.local_indices(1)] = y_ref.cpu().numpy()
    assert rel_l2(yo, y_orc) <= 1e-5
    for a in (1, 2, 4, 8):
        p = MemXCT(n, m, c, vector_order=order, ray_block=a, stage_order=-1).build()
        assert p.get_option("ray_block") == min(a, p.layout_info(0)["part_rows"] // 32)
        assert p.layout_info(0)["nnz"] == ref.layout_info(0)["nnz"]
        assert torch.equal(p.forward(xt), y_ref), a
        yb = torch.from_numpy(inputs.uniform(m * c, 32)).cuda()
        if order == "plan":
            yb = yb[torch.from_numpy(ref.local_indices(1)).cuda()].contiguous()
        assert torch.equal(p.back(yb), ref.back(yb))
        # the fused CG dot sums the same rows in other CTAs: same solve up to dot rounding
        ys = torch.from_numpy(np.ascontiguousarray(
            (y_orc if order == "natural" else y_orc[ref.local_indices(1)]).astype(np.float32))).cuda()
        assert rel_l2(p.cg(ys, 10).cpu().numpy(), ref.cg(ys, 10).cpu().numpy()) <= 1e-4
        p.close()


def test_blocked_rows_batched_and_mixed():
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    n, m, c = 64, 90, 64
    x = inputs.uniform(n * n, 41)
    ref = MemXCT(n, m, c, ray_block=-1, slices=4).build()
    blk = MemXCT(n, m, c, ray_block=4, slices=4).build()        # slab stages (auto with blocks)
    assert blk.get_option("stage_order") == 1
    X = torch.from_numpy(np.stack([x, 2 * x, x[::-1].copy()])).cuda()
    assert rel_l2(blk.forward_batch(X).cpu().numpy(), ref.forward_batch(X).cpu().numpy()) <= 1e-6
    mref = MemXCT(n, m, c, ray_block=-1, precision="mixed", stage_order=-1).build()
    mblk = MemXCT(n, m, c, ray_block=4, precision="mixed", stage_order=-1).build()
    xd = torch.from_numpy(x.astype(np.float64)).cuda()
    assert torch.equal(mblk.forward(xd), mref.forward(xd))   # one fp64 chain per row, same order
    can = MemXCT(n, m, c, ray_block=4, precision="mixed", canonical=True).build()
    assert can.get_option("ray_block") == -1                    # canonical keeps the Hilbert rows
    assert can.get_option("stage_order") == -1                  # ... and the Hilbert stages
    assert MemXCT(n, m, c, precision="mixed").build().get_option("stage_order") == -1
    slab = MemXCT(n, m, c, ray_block=4, precision="mixed", stage_order=1).build()
    assert rel_l2(slab.forward(xd).cpu().numpy(), mref.forward(xd).cpu().numpy()) <= 1e-14


def test_auto_rule():
    """Auto: Hilbert rows where the paper's square blocks are near the reuse optimum (configs 1-2;
    L pi / M ~ 2), projection blocks where they are far from it (few projections, wide grid)."""
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    assert MemXCT(256, 360, 256).build().get_option("ray_block") == -1
    assert MemXCT(256, 360, 256).build().get_option("stage_order") == 1      # slab stages by default
    assert MemXCT(64, 90, 64).build().get_option("ray_block") == -1
    wide = MemXCT(2048, 60, 2048).build()          # L pi / M = 107: a* = sqrt(R / 107) ~ 3
    assert wide.get_option("ray_block") == 8       # smallest power of two >= 2 a*
    assert wide.get_option("stage_order") == 1


@pytest.mark.parametrize("nranks", [2, 4])
def test_blocked_rows_virtual_ranks_and_shard(nranks):
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    n, m, c = 256, 360, 256
    g0, ref = build_group(n, m, c, nranks, ray_block=-1, stage_order=-1)
    g1, blk = build_group(n, m, c, nranks, ray_block=4, stage_order=-1)
    x = inputs.uniform(n * n, 51)
    xs = scatter(ref, x, 0, np.float32)
    y0 = run_ranks(nranks, lambda r: ref[r].forward(xs[r]))
    y1 = run_ranks(nranks, lambda r: blk[r].forward(xs[r]))
    for a, b in zip(y0, y1):
        assert torch.equal(a, b)
    for r in range(nranks):
        sp = MemXCT(n, m, c, rank=r, nranks=nranks, shard=True, vector_order="plan", ray_block=4,
                    stage_order=-1).build()
        assert torch.equal(sp.footprint_forward(xs[r]), ref[r].footprint_forward(xs[r]))
        sp.close()
    assert rel_l2(gather(blk, y1, 1, m * c), gather(ref, y0, 1, m * c)) == 0.0


def test_slab_stages_virtual_ranks_peer_and_shard():
    """Slab stages (STAGE_ORDER = 1) on the decomposed path: same sums up to fp32 rounding order,
    in the collective and the shard builds alike (identical layouts, bit-identical A_p)."""
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    n, m, c, nranks = 256, 360, 256, 3
    g0, ref = build_group(n, m, c, nranks, ray_block=-1, stage_order=-1)
    g1, slab = build_group(n, m, c, nranks, ray_block=4, stage_order=1)
    x = inputs.uniform(n * n, 61)
    xs = scatter(ref, x, 0, np.float32)
    y0 = gather(ref, run_ranks(nranks, lambda r: ref[r].forward(xs[r])), 1, m * c)
    y1 = gather(slab, run_ranks(nranks, lambda r: slab[r].forward(xs[r])), 1, m * c)
    assert rel_l2(y1, y0) <= 1e-6
    for r in range(nranks):
        sp = MemXCT(n, m, c, rank=r, nranks=nranks, shard=True, vector_order="plan", ray_block=4,
                    stage_order=1).build()
        assert torch.equal(sp.footprint_forward(xs[r]), slab[r].footprint_forward(xs[r]))
        sp.close()
