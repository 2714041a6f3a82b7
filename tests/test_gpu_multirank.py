"""Multi-GPU path (A = R C A_p) on ONE device through virtual ranks: P plans in one
process, each driven from its own thread; the collectives are device copies instead of NCCL,
everything else (decomposition, footprints, exchange maps, reduce-R, pack-R^T, kernels, CG) is
the code NCCL ranks run.  Results are assembled through memxct_local_indices and compared with
the single-GPU plan and the fp64 oracle."""
import threading

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


def run_ranks(nranks, fn):
    out, err = [None] * nranks, [None] * nranks

    def body(r):
        try:
            with torch.cuda.stream(torch.cuda.Stream()):
                out[r] = fn(r)
                torch.cuda.current_stream().synchronize()
        except BaseException as e:  # noqa: BLE001
            err[r] = e
    ts = [threading.Thread(target=body, args=(r,)) for r in range(nranks)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout=600)
    for e in err:
        if e is not None:
            raise e
    return out


def build_group(n, m, c, nranks, **kw):
    from paper_conf_sc_hidayetoglubgrg19_b200 import LocalGroup, MemXCT
    g = LocalGroup(nranks)
    plans = run_ranks(nranks, lambda r: MemXCT(n, m, c, group=g, rank=r, vector_order="plan", **kw).build())
    return g, plans


def scatter(plans, vec, domain, dtype):
    return [torch.from_numpy(np.ascontiguousarray(vec[p.local_indices(domain)]).astype(dtype)).cuda()
            for p in plans]


def gather(plans, parts, domain, size):
    out = np.zeros(size)
    for p, v in zip(plans, parts):
        out[p.local_indices(domain)] = v.cpu().numpy()
    return out


@pytest.mark.parametrize("nranks", [1, 2, 3, 4])
@pytest.mark.parametrize("geom", [(64, 90, 64), (256, 360, 256)])
def test_decomposition_and_fp32_projections(orc, coo_cache, nranks, geom):
    n, m, c = geom
    g, plans = build_group(n, m, c, nranks)
    # both domains are covered exactly once, identically on every rank
    for dom, size in ((0, n * n), (1, m * c)):
        b = plans[0].domain_ranges(dom)
        assert b[0] == 0 and b[-1] == size and np.all(np.diff(b) > 0)
        for p in plans[1:]:
            assert np.array_equal(p.domain_ranges(dom), b)
        idx = np.concatenate([p.local_indices(dom) for p in plans])
        assert np.array_equal(np.sort(idx), np.arange(size))
    # nonzeros of A_p sum to nnz(A) and are balanced
    rows, cols, vals = coo_cache(n, m, c)
    nnz = [p.layout_info(0)["nnz"] for p in plans]
    assert sum(nnz) == len(rows)
    assert max(nnz) / np.mean(nnz) < 1.25, nnz
    info = [p.exchange_info() for p in plans]
    assert sum(i["sent"] for i in info) == sum(i["received"] for i in info)
    # forward / back against the oracle
    x = inputs.shepp_logan(n).astype(np.float32)
    xs = scatter(plans, x, 0, np.float32)
    ys = run_ranks(nranks, lambda r: plans[r].forward(xs[r]))
    y = gather(plans, ys, 1, m * c)
    y_orc = orc.spmv_coo(rows, cols, vals, x.astype(np.float64), m * c)
    assert rel_l2(y, y_orc) <= 1e-5
    yv = inputs.uniform(m * c, 7)
    yss = scatter(plans, yv, 1, np.float32)
    xb = run_ranks(nranks, lambda r: plans[r].back(yss[r]))
    xbg = gather(plans, xb, 0, n * n)
    x_orc = orc.spmv_coo(cols, rows, vals, yv.astype(np.float64), n * n)
    assert rel_l2(xbg, x_orc) <= 1e-5


@pytest.mark.parametrize("nranks", [2, 4])
def test_mixed_projections_and_cg(orc, coo_cache, nranks):
    n, m, c = 64, 90, 64
    g, plans = build_group(n, m, c, nranks, precision="mixed")
    rows, cols, vals = coo_cache(n, m, c)
    v32 = vals.astype(np.float32).astype(np.float64)
    x = inputs.normal(n * n, 3)
    xs = scatter(plans, x, 0, np.float64)
    y = gather(plans, run_ranks(nranks, lambda r: plans[r].forward(xs[r])), 1, m * c)
    assert rel_l2(y, orc.spmv_coo(rows, cols, v32, x, m * c)) <= 1e-13
    xt = inputs.shepp_logan(n)
    ysino = orc.spmv_coo(rows, cols, vals, xt, m * c).astype(np.float32).astype(np.float64)
    yss = scatter(plans, ysino, 1, np.float64)
    res = run_ranks(nranks, lambda r: plans[r].cg(yss[r], 10, residuals=True))
    xr = gather(plans, [r[0] for r in res], 0, n * n)
    x_orc, res_orc, _, _ = orc.cgls(rows, cols, v32, ysino, m * c, n * n, 10)
    assert rel_l2(xr, x_orc) <= 1e-6
    for r in res:
        assert np.allclose(r[1], res_orc, rtol=1e-9)


def test_fp32_cg_multirank_recovers_phantom(orc, coo_cache):
    n, m, c = 256, 360, 256
    nranks = 4
    g, plans = build_group(n, m, c, nranks)
    rows, cols, vals = coo_cache(n, m, c)
    xt = inputs.shepp_logan(n)
    y32 = orc.spmv_coo(rows, cols, vals, xt, m * c).astype(np.float32)
    yss = scatter(plans, y32, 1, np.float32)
    res = run_ranks(nranks, lambda r: plans[r].cg(yss[r], 30, residuals=True))
    xr = gather(plans, [r[0] for r in res], 0, n * n)
    x_orc = orc.cgls(rows, cols, vals, y32.astype(np.float64), m * c, n * n, 30)[0]
    assert rel_l2(xr, xt) <= 1.1 * rel_l2(x_orc, xt)
    assert np.all(np.diff(res[0][1]) <= 1e-6 * res[0][1][0])


@pytest.mark.parametrize("exchange", ["collective", "peer", "dense"])
def test_one_rank_nccl_communicator(orc, coo_cache, exchange):
    """The decomposed path on a real one-rank NCCL communicator (memxct_get_unique_id + set_comm
    with nranks = 1): NCCL loading, communicator init, grouped send/recv to self, allreduce,
    allgather, CUDA IPC peer mapping and the graph-captured CG run exactly as on a multi-GPU
    node.  Projections are bit-identical to the plain plan in plan order (one partial per ray:
    the reduction adds it to zero); CG differs only in the dot summation order."""
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, get_unique_id
    n, m, c = 256, 360, 256
    dist = MemXCT(n, m, c, rank=0, nranks=1, unique_id=get_unique_id(), device=0,
                  vector_order="plan", exchange=exchange).build()
    plain = MemXCT(n, m, c, vector_order="plan").build()
    for d in (0, 1):
        assert np.array_equal(dist.local_indices(d), plain.local_indices(d))
    info = dist.exchange_info()
    assert info["sent"] == info["received"] and info["peers"] <= 1
    rows, cols, vals = coo_cache(n, m, c)
    xt = inputs.shepp_logan(n)
    x = torch.from_numpy(xt[plain.local_indices(0)].astype(np.float32)).cuda()
    y = torch.from_numpy(inputs.uniform(m * c, 5)[plain.local_indices(1)].astype(np.float32)).cuda()
    for _ in range(2):  # repeated calls exercise the peer path's credit flags
        assert torch.equal(dist.forward(x), plain.forward(x))
        assert torch.equal(dist.back(y), plain.back(y))
    y32 = orc.spmv_coo(rows, cols, vals, xt, m * c).astype(np.float32)
    ys = torch.from_numpy(y32[plain.local_indices(1)]).cuda()
    xd, rd = dist.cg(ys, 30, residuals=True)
    xp, rp = plain.cg(ys, 30, residuals=True)
    xd2 = dist.cg(ys, 30)  # graph replay
    assert torch.equal(xd, xd2)
    assert rel_l2(xd.cpu().numpy(), xp.cpu().numpy()) <= 1e-3
    xr = np.zeros(n * n)
    xr[plain.local_indices(0)] = xd.cpu().numpy()
    x_orc = orc.cgls(rows, cols, vals, y32.astype(np.float64), m * c, n * n, 30)[0]
    assert rel_l2(xr, xt) <= 1.1 * rel_l2(x_orc, xt)
    t = dist.exchange_time(5)
    assert t["fwd_us"] > 0 and t["back_us"] > 0
    dist.close()
    plain.close()


@pytest.mark.parametrize("nranks", [2, 3, 4])
@pytest.mark.parametrize("prec", ["fp32", "mixed"])
def test_dense_exchange_bit_identical_to_sparse(nranks, prec):
    """EXCHANGE = 2 (dense reduce-scatter / allgather of the whole partial sinogram, SURVEY 8(e)'s
    comparison) against the sparse all-to-allv + reduction R (default).  Ranks that do not touch a
    ray contribute exact zeros and the virtual-rank sums run in rank order, which is the reduction
    map's peer order: projections and CG iterates are bit-identical."""
    n, m, c = 64, 90, 64
    dt = np.float32 if prec == "fp32" else np.float64
    gs, sparse = build_group(n, m, c, nranks, precision=prec)
    gd, dense = build_group(n, m, c, nranks, precision=prec, exchange="dense")
    x = inputs.uniform(n * n, 21)
    y = inputs.uniform(m * c, 22)

    def run(plans):
        xs, ys = scatter(plans, x, 0, dt), scatter(plans, y, 1, dt)
        fw = run_ranks(nranks, lambda r: plans[r].forward(xs[r]))
        bk = run_ranks(nranks, lambda r: plans[r].back(ys[r]))
        cg = run_ranks(nranks, lambda r: plans[r].cg(ys[r], 8, residuals=True))
        return (gather(plans, fw, 1, m * c), gather(plans, bk, 0, n * n),
                gather(plans, [v[0] for v in cg], 0, n * n), cg[0][1])
    for a, b in zip(run(sparse), run(dense)):
        assert np.array_equal(a, b)
    assert dense[0].get_option("exchange") == 2
    ex = run_ranks(nranks, lambda r: dense[r].exchange_time(3))
    assert all(e["fwd_us"] > 0 and e["back_us"] > 0 for e in ex)


@pytest.mark.parametrize("nranks", [2, 3, 4])
def test_forward_overlap_bit_identical(monkeypatch, nranks):
    """Sparse collective exchange with the forward overlap (default: partitions holding rows of
    other owners first, the self-owned partitions concurrently on a side stream while the
    all-to-allv runs, the self slice copied after the join) against MEMXCT_FWD_OVERLAP=0: the
    same kernels write the same partials, so projections and CG are bit-identical."""
    n, m, c = 256, 360, 256
    _, on = build_group(n, m, c, nranks)
    monkeypatch.setenv("MEMXCT_FWD_OVERLAP", "0")
    _, off = build_group(n, m, c, nranks)
    x = inputs.uniform(n * n, 31)
    y = inputs.uniform(m * c, 32)

    def run(plans):
        xs, ys = scatter(plans, x, 0, np.float32), scatter(plans, y, 1, np.float32)
        fw = run_ranks(nranks, lambda r: plans[r].forward(xs[r]))
        cg = run_ranks(nranks, lambda r: plans[r].cg(ys[r], 6))
        return gather(plans, fw, 1, m * c), gather(plans, cg, 0, n * n)
    for a, b in zip(run(on), run(off)):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("nranks", [2, 3])
def test_batched_multirank_bit_identical_to_single(nranks):
    """Multi-slice calls on virtual ranks (A_p SpMM over slice-interleaved inputs, then the
    per-slice exchange): every slice equals its single-slice projection / CG on the same plans.
    The group of 5 runs as 4 + 1 slices, so the batched scratch is sized for the largest group
    and the 1-slice remainder takes the single-slice path."""
    n, m, c, k = 64, 90, 64, 5
    _, plans = build_group(n, m, c, nranks, slices=4)
    xs = [inputs.uniform(n * n, 40 + s) for s in range(k)]
    ys = [inputs.uniform(m * c, 50 + s) for s in range(k)]
    X = [torch.stack(v) for v in zip(*[scatter(plans, x, 0, np.float32) for x in xs])]
    Y = [torch.stack(v) for v in zip(*[scatter(plans, y, 1, np.float32) for y in ys])]
    fb = run_ranks(nranks, lambda r: plans[r].forward_batch(X[r]))
    bb = run_ranks(nranks, lambda r: plans[r].back_batch(Y[r]))
    cb = run_ranks(nranks, lambda r: plans[r].cg_batch(Y[r], 6, residuals=True))
    for s in range(k):
        f1 = run_ranks(nranks, lambda r: plans[r].forward(X[r][s].contiguous()))
        b1 = run_ranks(nranks, lambda r: plans[r].back(Y[r][s].contiguous()))
        c1 = run_ranks(nranks, lambda r: plans[r].cg(Y[r][s].contiguous(), 6, residuals=True))
        for r in range(nranks):
            assert torch.equal(fb[r][s], f1[r]), (s, r)
            assert torch.equal(bb[r][s], b1[r]), (s, r)
            assert torch.equal(cb[r][0][s], c1[r][0]), (s, r)
            assert np.array_equal(cb[r][1][s], c1[r][1]), (s, r)
