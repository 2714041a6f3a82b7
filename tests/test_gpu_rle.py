"""Run-length stage maps (Layout::rle, rle.cu, MEMXCT_RLE): the stage gather reads one 16 B record
of up to 4 runs per 32 slots instead of 32 int32 map entries (blocks with more runs keep their
entries in an overflow array).  The gathered stage buffer is the same, so every product must be
bit-identical to the plain map's, for every kernel that gathers from a single-slice map: the
plain FP32 SpMV, the drifting-stage kernel, the fp64 (MIXED / CANONICAL) kernel, the fused-dot
epilogues, CG, and decomposed plans (virtual ranks, the fused peer exchange's remote epilogue)."""
import numpy as np
import pytest

from paper_conf_sc_hidayetoglubgrg19_b200 import inputs

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_hidayetoglubgrg19_b200 import build_ext
    build_ext.build()


def _pair(monkeypatch, n, m, c, **kw):
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    monkeypatch.setenv("MEMXCT_RLE", "0")
    a = MemXCT(n, m, c, **kw).build()
    monkeypatch.setenv("MEMXCT_RLE", "1")
    b = MemXCT(n, m, c, **kw).build()
    monkeypatch.delenv("MEMXCT_RLE")
    return a, b


CASES = [
    ((64, 90, 64), {}),
    ((256, 360, 256), {}),
    ((33, 17, 33), {"buffer_entries": 256}),                   # many stages, partial blocks
    ((256, 360, 256), {"buffer_entries": 1024}),
    ((256, 36, 256), {"ray_block": 8}),                        # projection blocks: drifting kernel
    ((64, 90, 64), {"precision": "mixed", "canonical": True}),
    ((256, 360, 256), {"precision": "mixed"}),
    ((40, 7, 97), {"vector_order": "plan"}),
]


@pytest.mark.parametrize("geom,kw", CASES)
def test_rle_bit_identical(monkeypatch, geom, kw):
    n, m, c = geom
    plain, rle = _pair(monkeypatch, n, m, c, **kw)
    dt = np.float64 if kw.get("precision") == "mixed" else np.float32
    rng = np.random.default_rng(n + m)
    x = torch.from_numpy(rng.random(n * n).astype(dt)).cuda()
    y = torch.from_numpy(rng.random(m * c).astype(dt)).cuda()
    assert torch.equal(plain.forward(x), rle.forward(x))
    assert torch.equal(plain.back(y), rle.back(y))
    x0, r0 = plain.cg(y, 8, residuals=True)
    x1, r1 = rle.cg(y, 8, residuals=True)
    assert torch.equal(x0, x1) and np.array_equal(r0, r1)


def test_rle_virtual_ranks_all_exchanges(monkeypatch):
    from test_gpu_multirank import build_group, gather, run_ranks, scatter
    n, m, c = 256, 360, 256
    x = inputs.uniform(n * n, 5)
    y = inputs.uniform(m * c, 6)
    out = []
    for val in ("0", "1"):
        monkeypatch.setenv("MEMXCT_RLE", val)
        _, plans = build_group(n, m, c, 3, exchange="dense")
        xs, ys = scatter(plans, x, 0, np.float32), scatter(plans, y, 1, np.float32)
        fw = gather(plans, run_ranks(3, lambda r: plans[r].forward(xs[r])), 1, m * c)
        bk = gather(plans, run_ranks(3, lambda r: plans[r].back(ys[r])), 0, n * n)
        out.append((fw, bk))
    monkeypatch.delenv("MEMXCT_RLE")
    assert np.array_equal(out[0][0], out[1][0]) and np.array_equal(out[0][1], out[1][1])
