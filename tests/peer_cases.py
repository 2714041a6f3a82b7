"""Cases of the fused peer-memory exchange on virtual ranks, run in a child process by
tests/test_gpu_peer_exchange.py.

Virtual ranks share ONE device, so any device-wide synchronisation issued by one rank's thread
(cudaFree from a garbage-collected plan, an allocator trim, ...) waits for the other ranks'
spinning flag waits while those ranks wait for it: a deadlock that cannot happen with one
process per GPU (a rank's own waits only depend on kernels its peers have already queued).  The
cases therefore run in a fresh process with the garbage collector off and pre-allocated tensors,
and a failure (the wait kernels trap after ~20 s instead of hanging) cannot poison the main test
process's CUDA context.
"""
import gc
import os
import sys
import threading

import numpy as np

# Concurrent streams of one process share a few hardware queues (CUDA_DEVICE_MAX_CONNECTIONS,
# default 8); two virtual ranks whose streams land on the same queue serialise, and a rank's
# flag wait would then block the very kernel it waits for.  Give every stream its own queue and
# create the ranks' streams once.
os.environ["CUDA_DEVICE_MAX_CONNECTIONS"] = "32"
os.environ["CUDA_MODULE_LOADING"] = "EAGER"  # no kernel loading (and its device waits) mid-run

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, HERE)
sys.path.insert(0, os.path.dirname(HERE))

_STREAMS = {}


def run_ranks(nranks, fn):
    import torch
    for r in range(nranks):
        _STREAMS.setdefault(r, torch.cuda.Stream())
    out, err = [None] * nranks, [None] * nranks

    def body(r):
        try:
            with torch.cuda.stream(_STREAMS[r]):
                out[r] = fn(r)
        except BaseException as e:  # noqa: BLE001
            err[r] = e
    ts = [threading.Thread(target=body, args=(r,)) for r in range(nranks)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout=600)
    for r in range(nranks):  # synchronise only after every rank has queued all of its work
        _STREAMS[r].synchronize()
    for e in err:
        if e is not None:
            raise e
    return out


def build_group(n, m, c, nranks, **kw):
    from paper_conf_sc_hidayetoglubgrg19_b200 import LocalGroup, MemXCT
    g = LocalGroup(nranks)
    plans = run_ranks(nranks, lambda r: MemXCT(n, m, c, group=g, rank=r, vector_order="plan", **kw).build())
    return g, plans


def rel_l2(a, b):
    return float(np.linalg.norm(np.asarray(a) - np.asarray(b)) / np.linalg.norm(np.asarray(b)))


def case_projections(nranks, n, m, c, ray_block=None):
    import torch

    import oracle
    from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
    from test_gpu_multirank import gather, scatter
    import time
    t0 = time.time()
    so = None if ray_block is None else -1      # Hilbert stages: blocked rows are then bit-identical
    g0, coll = build_group(n, m, c, nranks, stage_order=so)
    g1, peer = build_group(n, m, c, nranks, exchange="peer", ray_block=ray_block, stage_order=so)
    print(f"built {time.time() - t0:.2f}s", flush=True)
    x = inputs.uniform(n * n, 1)
    y = inputs.uniform(m * c, 2)
    res = {}
    for name, plans in (("coll", coll), ("peer", peer)):
        xs, ys = scatter(plans, x, 0, np.float32), scatter(plans, y, 1, np.float32)
        xs2 = [v * 2 for v in xs]
        ys3 = [v * 3 for v in ys]
        outs = [[torch.empty(p.local_size(1), device="cuda") for _ in range(3)] +
                [torch.empty(p.local_size(0), device="cuda") for _ in range(3)] for p in plans]
        torch.cuda.synchronize()

        def body(r, plans=plans, xs=xs, ys=ys, xs2=xs2, ys3=ys3, outs=outs):
            p, o = plans[r], outs[r]
            p.forward(xs[r], o[0])
            p.forward(xs2[r], o[1])
            p.back(ys[r], o[3])
            p.back(ys3[r], o[4])
            p.forward(xs[r], o[2])
            p.back(ys[r], o[5])
            return o
        try:
            res[name] = run_ranks(nranks, body)
        finally:
            print(f"{name} done {time.time() - t0:.2f}s", flush=True)
    for r in range(nranks):
        for k in range(6):
            assert torch.equal(res["coll"][r][k], res["peer"][r][k]), (r, k)
    yf = gather(peer, [o[0] for o in res["peer"]], 1, m * c)
    xb = gather(peer, [o[3] for o in res["peer"]], 0, n * n)
    if n * n * m <= 256 * 256 * 360:
        rows, cols, vals = oracle.trace_all(n, m, c)
        assert rel_l2(yf, oracle.spmv_coo(rows, cols, vals, x.astype(np.float64), m * c)) <= 1e-5
        assert rel_l2(xb, oracle.spmv_coo(cols, rows, vals, y.astype(np.float64), n * n)) <= 1e-5
    else:  # full size: sampled rows against the oracle's traces
        from fullsize import N_RAYS, pick_pixels, sampled_back_error, sampled_forward_error
        rng = np.random.default_rng(n)
        rays = rng.choice(m * c, N_RAYS, replace=False)
        assert sampled_forward_error(oracle, n, m, c, rays, yf[rays], x.astype(np.float64)) <= 1e-5
        pixels = pick_pixels(rng, n)
        yh = y.astype(np.float64)
        assert sampled_back_error(oracle, n, m, c, pixels, xb[pixels], lambda r: yh[r]) <= 1e-5


def case_cg(nranks, n, m, c):
    import torch

    import oracle
    from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
    from test_gpu_multirank import gather, scatter
    g0, coll = build_group(n, m, c, nranks)
    g1, peer = build_group(n, m, c, nranks, exchange="peer")
    rows, cols, vals = oracle.trace_all(n, m, c)
    xt = inputs.shepp_logan(n)
    y32 = oracle.spmv_coo(rows, cols, vals, xt, m * c).astype(np.float32)
    out = {}
    for name, plans in (("coll", coll), ("peer", peer)):
        ys = scatter(plans, y32, 1, np.float32)
        xa = [torch.empty(p.local_size(0), device="cuda") for p in plans]
        xs = [torch.empty(p.local_size(0), device="cuda") for p in plans]
        torch.cuda.synchronize()
        # a short solve, then a longer one: the second grows the CG scalars (grow-only, no
        # cudaFree while peers' waits spin -- a device-wide sync there would deadlock)
        out[name] = run_ranks(nranks, lambda r, plans=plans, ys=ys, xa=xa, xs=xs: (
            plans[r].cg(ys[r], 10, x=xa[r]), plans[r].cg(ys[r], 30, x=xs[r]))[1])
        out[name + "10"] = xa
    for a, b in zip(out["coll"] + out["coll10"], out["peer"] + out["peer10"]):
        assert torch.equal(a, b)
    xr = gather(peer, out["peer"], 0, n * n)
    x_orc = oracle.cgls(rows, cols, vals, y32.astype(np.float64), m * c, n * n, 30)[0]
    assert rel_l2(xr, xt) <= 1.1 * rel_l2(x_orc, xt)


if __name__ == "__main__":
    import torch
    gc.disable()
    torch.cuda.init()
    case, nranks, n, m, c = sys.argv[1], *map(int, sys.argv[2:6])
    extra = [int(v) for v in sys.argv[6:]]  # projections: RAY_BLOCK of the peer group
    {"projections": case_projections, "cg": case_cg}[case](nranks, n, m, c, *extra)
    torch.cuda.synchronize()
    print("CASE OK", case, nranks, n, m, c, flush=True)
    os._exit(0)  # skip teardown frees while nothing else runs; the process ends here
