"""The chunked device build (layout.cu) produces the same layout whatever the chunk budget:
forcing tiny chunks (MEMXCT_BUILD_CHUNK, entries per chunk) must give bit-identical layouts and
projections, single GPU and virtual ranks.  This is the path configs 4-5 take for real."""
import os

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


def _build(n, m, c, chunk=None, **kw):
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    old = os.environ.pop("MEMXCT_BUILD_CHUNK", None)
    if chunk is not None:
        os.environ["MEMXCT_BUILD_CHUNK"] = str(chunk)
    try:
        return MemXCT(n, m, c, **kw).build()
    finally:
        os.environ.pop("MEMXCT_BUILD_CHUNK", None)
        if old is not None:
            os.environ["MEMXCT_BUILD_CHUNK"] = old


@pytest.mark.parametrize("geom,chunk", [((64, 90, 64), 20000), ((64, 90, 64), 1), ((256, 360, 256), 3_000_000)])
def test_chunked_layout_identical(geom, chunk):
    n, m, c = geom
    a = _build(n, m, c, part_rows=128, buffer_entries=2048)
    b = _build(n, m, c, chunk=chunk, part_rows=128, buffer_entries=2048)
    for d in (0, 1):
        ea, eb = a.layout_export(d), b.layout_export(d)
        for k in ea:
            assert np.array_equal(ea[k], eb[k]), (d, k)
    x = torch.from_numpy(inputs.uniform(n * n, 1)).cuda()
    assert torch.equal(a.forward(x), b.forward(x))
    y = torch.from_numpy(inputs.uniform(m * c, 2)).cuda()
    assert torch.equal(a.back(y), b.back(y))


def test_chunked_build_virtual_ranks():
    from test_gpu_multirank import build_group, gather, run_ranks, scatter
    n, m, c = 64, 90, 64
    os.environ["MEMXCT_BUILD_CHUNK"] = "30000"
    try:
        g, plans = build_group(n, m, c, 3)
    finally:
        os.environ.pop("MEMXCT_BUILD_CHUNK", None)
    g2, plans2 = build_group(n, m, c, 3)
    x = inputs.uniform(n * n, 3)
    xs = scatter(plans, x, 0, np.float32)
    y1 = gather(plans, run_ranks(3, lambda r: plans[r].forward(xs[r])), 1, m * c)
    y2 = gather(plans2, run_ranks(3, lambda r: plans2[r].forward(xs[r])), 1, m * c)
    assert np.array_equal(y1, y2)
