"""The target decomposition: P = 6 and P = 8 ranks (the 8 x B200 box of BASELINE configs[2-4]),
on virtual ranks (one device, one host thread per rank; tests/test_gpu_multirank.py explains the
transport).  At P = 8 a rank talks to up to 7 peers (profiles/r01h_shard_cfg3_p8.jsonl), against
at most 3 in the P <= 4 tests.  A = R C A_p with every exchange:

  * sparse all-to-allv + reduction R (default), dense reduce-scatter / allgather (EXCHANGE = 2),
    fused peer-memory stores (EXCHANGE = 1, in a child process: tests/peer_cases.py);
  * config 2 (ADS1 shape): FP32 projections within 1e-5 of the fp64 oracle, MIXED projections
    within 1e-13 and MIXED CG within 1e-6 of the oracle's CGLS, dense bit-identical to sparse;
  * config 3 (ADS3, the bench workload): 1e4 sampled rays and 1024 sampled pixels of the
    assembled projections against the oracle's traces (<= 1e-5), dense bit-identical to sparse,
    peer bit-identical to sparse (child process)."""
import os
import subprocess
import sys

import numpy as np
import pytest

from conftest import rel_l2
from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
from test_gpu_multirank import build_group, gather, run_ranks, scatter

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_hidayetoglubgrg19_b200 import build_ext
    build_ext.build()


def _projections(plans, x, y, dt):
    xs, ys = scatter(plans, x, 0, dt), scatter(plans, y, 1, dt)
    nr = len(plans)
    fw = run_ranks(nr, lambda r: plans[r].forward(xs[r]))
    bk = run_ranks(nr, lambda r: plans[r].back(ys[r]))
    n, m, c = plans[0].n, plans[0].m, plans[0].c
    return gather(plans, fw, 1, m * c), gather(plans, bk, 0, n * n)


@pytest.mark.parametrize("nranks", [6, 8])
def test_cfg2_p68_fp32_all_exchanges(orc, coo_cache, nranks):
    n, m, c = inputs.CONFIGS[2]
    rows, cols, vals = coo_cache(n, m, c)
    x = inputs.uniform(n * n, 61)
    y = inputs.uniform(m * c, 62)
    _, sparse = build_group(n, m, c, nranks)
    assert max(p.exchange_info()["peers"] for p in sparse) >= 4     # more peers than P <= 4 ever has
    nnz = [p.layout_info(0)["nnz"] for p in sparse]
    assert sum(nnz) == len(rows) and max(nnz) / np.mean(nnz) < 1.25, nnz
    ys, xs = _projections(sparse, x, y, np.float32)
    assert rel_l2(ys, orc.spmv_coo(rows, cols, vals, x.astype(np.float64), m * c)) <= 1e-5
    assert rel_l2(xs, orc.spmv_coo(cols, rows, vals, y.astype(np.float64), n * n)) <= 1e-5
    yss = scatter(sparse, y, 1, np.float32)
    cg_s = run_ranks(nranks, lambda r: sparse[r].cg(yss[r], 6, residuals=True))
    del sparse
    _, dense = build_group(n, m, c, nranks, exchange="dense")
    yd, xd = _projections(dense, x, y, np.float32)
    assert np.array_equal(yd, ys) and np.array_equal(xd, xs)
    ysd = scatter(dense, y, 1, np.float32)
    cg_d = run_ranks(nranks, lambda r: dense[r].cg(ysd[r], 6, residuals=True))
    for a, b in zip(cg_s, cg_d):
        assert torch.equal(a[0], b[0]) and np.array_equal(a[1], b[1])


@pytest.mark.parametrize("nranks", [6, 8])
def test_cfg2_p68_mixed_vs_oracle(orc, coo_cache, nranks):
    n, m, c = inputs.CONFIGS[2]
    rows, cols, vals = coo_cache(n, m, c)
    v32 = vals.astype(np.float32).astype(np.float64)
    _, plans = build_group(n, m, c, nranks, precision="mixed")
    x = inputs.normal(n * n, 63)
    y = inputs.normal(m * c, 64)
    yp, xp = _projections(plans, x, y, np.float64)
    assert rel_l2(yp, orc.spmv_coo(rows, cols, v32, x, m * c)) <= 1e-13
    assert rel_l2(xp, orc.spmv_coo(cols, rows, v32, y, n * n)) <= 1e-13
    xt = inputs.shepp_logan(n)
    ysino = orc.spmv_coo(rows, cols, vals, xt, m * c).astype(np.float32).astype(np.float64)
    yss = scatter(plans, ysino, 1, np.float64)
    # 10 iterations: fp64 iterates with another summation order agree to ~1e-8 (R16 table);
    # by iteration 28-30 the order decides up to ~2e-3 (R16: the 1e-3 x_30 gate binds the
    # single-GPU MIXED + CANONICAL mode), so 30 iterations are gated on the reconstruction
    res = run_ranks(nranks, lambda r: plans[r].cg(yss[r], 10, residuals=True))
    xr = gather(plans, [v[0] for v in res], 0, n * n)
    x_orc, res_orc, _, _ = orc.cgls(rows, cols, v32, ysino, m * c, n * n, 10)
    assert rel_l2(xr, x_orc) <= 1e-6
    assert np.allclose(res[0][1], res_orc, rtol=1e-9)
    res = run_ranks(nranks, lambda r: plans[r].cg(yss[r], 30, residuals=True))
    xr = gather(plans, [v[0] for v in res], 0, n * n)
    x_orc = orc.cgls(rows, cols, v32, ysino, m * c, n * n, 30)[0]
    print(f"P={nranks} MIXED CG x_30 drift {rel_l2(xr, x_orc):.2e}")
    assert rel_l2(xr, xt) <= 1.01 * rel_l2(x_orc, xt)


@pytest.mark.slow
def test_cfg3_p8_sparse_dense_vs_oracle(orc):
    import gc
    from fullsize import N_RAYS, pick_pixels, sampled_back_error, sampled_forward_error
    n, m, c = inputs.CONFIGS[3]
    nranks = 8
    x = inputs.uniform(n * n, 71)
    y = inputs.uniform(m * c, 72)
    _, sparse = build_group(n, m, c, nranks)
    ys, xs = _projections(sparse, x, y, np.float32)
    info = [p.exchange_info() for p in sparse]
    print("cfg3 P=8 peers per rank", [i["peers"] for i in info], "sent", [i["sent"] for i in info])
    rng = np.random.default_rng(3)
    rays = rng.choice(m * c, N_RAYS, replace=False)
    e_f = sampled_forward_error(orc, n, m, c, rays, ys[rays], x.astype(np.float64))
    pixels = pick_pixels(rng, n)
    yh = y.astype(np.float64)
    e_b = sampled_back_error(orc, n, m, c, pixels, xs[pixels], lambda r: yh[r])
    print(f"cfg3 P=8 sampled: {e_f:.2e} / {e_b:.2e}")
    assert e_f <= 1e-5 and e_b <= 1e-5
    for p in sparse:
        p.close()
    del sparse
    gc.collect()
    torch.cuda.empty_cache()
    _, dense = build_group(n, m, c, nranks, exchange="dense")
    yd, xd = _projections(dense, x, y, np.float32)
    assert np.array_equal(yd, ys) and np.array_equal(xd, xs)


def _run_case(*args, timeout=900):
    r = subprocess.run([sys.executable, os.path.join(HERE, "peer_cases.py"), *map(str, args)],
                       capture_output=True, text=True, timeout=timeout)
    assert r.returncode == 0 and "CASE OK" in r.stdout, (r.stdout[-2000:], r.stderr[-4000:])


@pytest.mark.parametrize("nranks", [6, 8])
def test_cfg2_p68_peer_bit_identical(nranks):
    _run_case("projections", nranks, *inputs.CONFIGS[2])


def test_cfg2_p8_peer_cg():
    _run_case("cg", 8, *inputs.CONFIGS[2])


@pytest.mark.slow
def test_cfg3_p8_peer_bit_identical():
    _run_case("projections", 8, *inputs.CONFIGS[3], timeout=1500)
