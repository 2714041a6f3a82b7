"""Fused peer-memory exchange (EXCHANGE = 1) on virtual ranks: the SpMV
epilogue stores partials into the owners' receive buffers and the pack kernel stores ray values
into the peers' footprint buffers, synchronised by epoch / credit flags.  The reductions read the
same partials in the same peer order as the collective path, so results must be bit-identical to
EXCHANGE = 0 for any call sequence (including repeated forwards, which exercise the credits)."""
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


@pytest.mark.parametrize("nranks", [2, 3, 4])
@pytest.mark.parametrize("geom", [(64, 90, 64), (256, 360, 256)])
def test_peer_exchange_bit_identical_to_collective(orc, coo_cache, nranks, geom):
    from test_gpu_multirank import build_group, gather, run_ranks, scatter
    n, m, c = geom
    g0, coll = build_group(n, m, c, nranks)
    g1, peer = build_group(n, m, c, nranks, exchange="peer")
    x = inputs.uniform(n * n, 1)
    y = inputs.uniform(m * c, 2)
    xs0, xs1 = scatter(coll, x, 0, np.float32), scatter(peer, x, 0, np.float32)
    ys0, ys1 = scatter(coll, y, 1, np.float32), scatter(peer, y, 1, np.float32)

    def seq(plans, xs, ys):
        def body(r):
            p = plans[r]
            out = [p.forward(xs[r]), p.forward(xs[r] * 2), p.back(ys[r]), p.back(ys[r] * 3),
                   p.forward(xs[r]), p.back(ys[r])]
            return [o.clone() for o in out]
        return run_ranks(nranks, body)

    a, b = seq(coll, xs0, ys0), seq(peer, xs1, ys1)
    for r in range(nranks):
        for k in range(6):
            assert torch.equal(a[r][k], b[r][k]), (r, k)
    rows, cols, vals = coo_cache(n, m, c)
    yf = gather(peer, [o[0] for o in b], 1, m * c)
    assert rel_l2(yf, orc.spmv_coo(rows, cols, vals, x.astype(np.float64), m * c)) <= 1e-5
    xb = gather(peer, [o[2] for o in b], 0, n * n)
    assert rel_l2(xb, orc.spmv_coo(cols, rows, vals, y.astype(np.float64), n * n)) <= 1e-5


def test_peer_exchange_cg(orc, coo_cache):
    from test_gpu_multirank import build_group, gather, run_ranks, scatter
    n, m, c = 256, 360, 256
    nranks = 4
    g0, coll = build_group(n, m, c, nranks)
    g1, peer = build_group(n, m, c, nranks, exchange="peer")
    rows, cols, vals = coo_cache(n, m, c)
    xt = inputs.shepp_logan(n)
    y32 = orc.spmv_coo(rows, cols, vals, xt, m * c).astype(np.float32)
    r0 = run_ranks(nranks, lambda r: coll[r].cg(scatter(coll, y32, 1, np.float32)[r], 30))
    r1 = run_ranks(nranks, lambda r: peer[r].cg(scatter(peer, y32, 1, np.float32)[r], 30))
    for a, b in zip(r0, r1):
        assert torch.equal(a, b)
    xr = gather(peer, r1, 0, n * n)
    x_orc = orc.cgls(rows, cols, vals, y32.astype(np.float64), m * c, n * n, 30)[0]
    assert rel_l2(xr, xt) <= 1.1 * rel_l2(x_orc, xt)
