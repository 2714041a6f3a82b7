"""GPU SIRT against the oracle's SIRT, single GPU and virtual
ranks; plus the exchange timer of the multi-GPU path."""
import numpy as np
import pytest

from conftest import rel_l2
from paper_conf_sc_hidayetoglubgrg19_b200 import inputs

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_hidayetoglubgrg19_b200 import build_ext
    build_ext.build()


def _problem(orc, coo_cache, n, m, c):
    rows, cols, vals = coo_cache(n, m, c)
    y = orc.spmv_coo(rows, cols, vals, inputs.shepp_logan(n), m * c).astype(np.float32)
    return rows, cols, vals, y


@pytest.mark.parametrize("geom", [(64, 90, 64), (256, 360, 256)])
def test_sirt_fp32_matches_oracle(orc, coo_cache, geom):
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    n, m, c = geom
    rows, cols, vals, y = _problem(orc, coo_cache, n, m, c)
    plan = MemXCT(n, m, c).build()
    x, res = plan.sirt(torch.from_numpy(y).cuda(), 45, residuals=True)
    x_orc, res_orc = orc.sirt(rows, cols, vals, y.astype(np.float64), m * c, n * n, 45)
    assert rel_l2(x.cpu().numpy(), x_orc) <= 1e-5
    assert np.allclose(res, res_orc, rtol=1e-4)


def test_sirt_mixed_matches_oracle_tightly(orc, coo_cache):
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    n, m, c = 64, 90, 64
    rows, cols, vals, y = _problem(orc, coo_cache, n, m, c)
    v32 = vals.astype(np.float32).astype(np.float64)
    plan = MemXCT(n, m, c, precision="mixed").build()
    x, res = plan.sirt(torch.from_numpy(y.astype(np.float64)).cuda(), 45, residuals=True)
    x_orc, res_orc = orc.sirt(rows, cols, v32, y.astype(np.float64), m * c, n * n, 45)
    assert rel_l2(x.cpu().numpy(), x_orc) <= 1e-12
    assert np.allclose(res, res_orc, rtol=1e-10)


def test_sirt_virtual_ranks(orc, coo_cache):
    from test_gpu_multirank import build_group, gather, run_ranks, scatter
    n, m, c = 64, 90, 64
    rows, cols, vals, y = _problem(orc, coo_cache, n, m, c)
    g, plans = build_group(n, m, c, 3)
    ys = scatter(plans, y, 1, np.float32)
    out = run_ranks(3, lambda r: plans[r].sirt(ys[r], 45, residuals=True))
    x = gather(plans, [o[0] for o in out], 0, n * n)
    x_orc, res_orc = orc.sirt(rows, cols, vals, y.astype(np.float64), m * c, n * n, 45)
    assert rel_l2(x, x_orc) <= 1e-5
    for o in out:
        assert np.allclose(o[1], res_orc, rtol=1e-4)
    # the exchange timer is collective and returns positive device times at P > 1
    t = run_ranks(3, lambda r: plans[r].exchange_time(5))
    assert all(v["fwd_us"] > 0 and v["back_us"] > 0 for v in t)
