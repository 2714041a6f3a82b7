"""Drifting stages (spmv_f32_drift_kernel, MEMXCT_DRIFT).

Listing 3 gathers a stage's inputs into the buffer, then streams the stage's
nonzeros; the plain kernel closes every stage with a CTA barrier.  The drifting kernel rotates
three stage buffers behind mbarriers so warps run up to about one stage apart; the layout, the
stage cut and every row's fma order are unchanged, so for the same buffer size B its products
must be bit-identical to the plain kernel's, and within the SURVEY tolerance of the fp64 oracle."""
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


def _plans(monkeypatch, n, m, c, **kw):
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    monkeypatch.delenv("MEMXCT_DRIFT", raising=False)
    plain = MemXCT(n, m, c, **kw).build()
    monkeypatch.setenv("MEMXCT_DRIFT", "1")
    drift = MemXCT(n, m, c, **kw).build()
    monkeypatch.delenv("MEMXCT_DRIFT")
    assert plain.layout_info(0)["buffer_entries"] == drift.layout_info(0)["buffer_entries"]
    return plain, drift


@pytest.mark.parametrize("n,m,c", [(64, 90, 64), (256, 360, 256), (33, 17, 33), (40, 7, 97)])
@pytest.mark.parametrize("B", [256, 2048, 13312, 16384])
def test_drift_bit_identical_to_plain(monkeypatch, orc, coo_cache, n, m, c, B):
    plain, drift = _plans(monkeypatch, n, m, c, buffer_entries=B)
    rng = np.random.default_rng(n + B)
    x = torch.from_numpy(rng.random(n * n, dtype=np.float32)).cuda()
    y = torch.from_numpy(rng.random(m * c, dtype=np.float32)).cuda()
    yf0, yf1 = plain.forward(x), drift.forward(x)
    xb0, xb1 = plain.back(y), drift.back(y)
    torch.cuda.synchronize()
    assert torch.equal(yf0, yf1)
    assert torch.equal(xb0, xb1)
    rows, cols, vals = coo_cache(n, m, c)
    y_ref = orc.spmv_coo(rows, cols, vals, x.cpu().numpy().astype(np.float64), m * c)
    x_ref = orc.spmv_coo(cols, rows, vals, y.cpu().numpy().astype(np.float64), n * n)
    assert rel_l2(yf1.cpu().numpy(), y_ref) <= 1e-5
    assert rel_l2(xb1.cpu().numpy(), x_ref) <= 1e-5


@pytest.mark.parametrize("order", ["natural", "plan"])
def test_drift_cg_bit_identical(monkeypatch, order):
    """CG with the fused dots (SpMV epilogue) through the drifting kernel."""
    n, m, c = 256, 360, 256
    plain, drift = _plans(monkeypatch, n, m, c, buffer_entries=1024, vector_order=order)
    ph = inputs.shepp_logan(n).astype(np.float32)
    if order == "plan":
        ph = np.ascontiguousarray(ph[plain.local_indices(0)])
    y = plain.forward(torch.from_numpy(ph).cuda())
    x0 = plain.cg(y, 12)
    x1 = drift.cg(y, 12)
    torch.cuda.synchronize()
    assert torch.equal(x0, x1)


def test_drift_auto_buffer(monkeypatch):
    """MEMXCT_DRIFT with the auto stage size: 3 buffers of B entries fit the CTA's shared memory."""
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    monkeypatch.setenv("MEMXCT_DRIFT", "1")
    plan = MemXCT(256, 360, 256).build()
    B = plan.layout_info(0)["buffer_entries"]
    assert 12 * B <= 224 * 1024
    y = plan.forward(torch.ones(256 * 256, device="cuda"))
    assert torch.isfinite(y).all()


def test_ray_block_forward_uses_drift_by_default(orc, coo_cache):
    """Projection-block plans (few projections, wide detector) run the forward operator on the
    drifting kernel with 13312-entry stages by default; an explicit BUFFER_ENTRIES of the same
    size selects the plain kernel: the products must be bit-identical (each row's fma order is
    independent of the stage cut) and match the oracle."""
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    n, m, c = 512, 16, 512
    auto = MemXCT(n, m, c).build()
    assert auto.get_option("ray_block") > 0
    Bf = auto.layout_info(0)["buffer_entries"]
    assert Bf <= 13312
    plain = MemXCT(n, m, c, buffer_entries=Bf).build()
    rng = np.random.default_rng(7)
    x = torch.from_numpy(rng.random(n * n, dtype=np.float32)).cuda()
    y0, y1 = plain.forward(x), auto.forward(x)
    torch.cuda.synchronize()
    assert torch.equal(y0, y1)
    rows, cols, vals = coo_cache(n, m, c)
    y_ref = orc.spmv_coo(rows, cols, vals, x.cpu().numpy().astype(np.float64), m * c)
    assert rel_l2(y1.cpu().numpy(), y_ref) <= 1e-5


@pytest.mark.parametrize("n,m,c,B", [(256, 360, 256, 256), (256, 360, 256, 1024), (64, 90, 64, 256)])
def test_drift_under_jitter_bit_identical(monkeypatch, n, m, c, B):
    """The buffer-reuse protocol at its limits: MEMXCT_DRIFT_JITTER=1 makes warps sleep
    pseudo-randomly (1-6 us) before streaming some stages, so they drift as far apart as the
    mbarrier rings allow while stage buffers are regathered.  compute-sanitizer racecheck does not
    model mbarrier synchronisation (it flags the correct protocol and a deliberately broken one
    alike, scripts/racecheck_mbarrier_probe.cu), so this is the protocol's stress test: many
    stages per partition (small B), repeated launches, every output bit-identical to the plain
    kernel's."""
    plain, drift = _plans(monkeypatch, n, m, c, buffer_entries=B)
    rng = np.random.default_rng(B)
    x = torch.from_numpy(rng.random(n * n, dtype=np.float32)).cuda()
    y = torch.from_numpy(rng.random(m * c, dtype=np.float32)).cuda()
    yf0, xb0 = plain.forward(x), plain.back(y)
    monkeypatch.setenv("MEMXCT_DRIFT_JITTER", "1")
    for _ in range(3):
        assert torch.equal(drift.forward(x), yf0)
        assert torch.equal(drift.back(y), xb0)
    monkeypatch.delenv("MEMXCT_DRIFT_JITTER")
