#!/usr/bin/env python
"""Small workloads for compute-sanitizer (racecheck / synccheck / memcheck / initcheck): every
kernel family of the hot path on config-1-sized inputs, one case per invocation.

    compute-sanitizer --tool racecheck python scripts/sanitize_cases.py CASE

Cases: fp32 (plain SpMV + fused-dot tickets + CG), drift (spmv_f32_drift_kernel: mbarrier
rings), mixed (fp64 canonical chains + canonical dots), spmm (K = 4 / 8 slice groups, interleave),
blocked (projection-block rows + slab stages), peer (virtual ranks, fused exchange: flags,
credits, remote stores, peer dots), collective (virtual ranks, all-to-allv + reduction R),
sirt.  Prints CASE OK when the case finished (the sanitizer's summary follows)."""
import os
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
os.environ.setdefault("CUDA_MODULE_LOADING", "EAGER")


def ranks(nranks, fn):
    import torch
    streams = [torch.cuda.Stream() for _ in range(nranks)]
    out, err = [None] * nranks, [None] * nranks

    def body(r):
        try:
            with torch.cuda.stream(streams[r]):
                out[r] = fn(r)
        except BaseException as e:  # noqa: BLE001
            err[r] = e
    ts = [threading.Thread(target=body, args=(r,)) for r in range(nranks)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    for s in streams:
        s.synchronize()
    for e in err:
        if e is not None:
            raise e
    return out


def main(case):
    import numpy as np
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import LocalGroup, MemXCT, inputs
    n, m, c = 64, 90, 64
    x = torch.from_numpy(inputs.uniform(n * n, 1)).cuda()
    y = torch.from_numpy(inputs.uniform(m * c, 2)).cuda()
    if case in ("fp32", "drift", "blocked"):
        if case == "drift":
            os.environ["MEMXCT_DRIFT"] = "1"
        kw = {"ray_block": 4, "stage_order": 1} if case == "blocked" else {}
        p = MemXCT(n, m, c, buffer_entries=1024 if case == "drift" else None, **kw).build()
        p.forward(x)
        p.back(y)
        p.cg(y, 5, residuals=True)
    elif case == "mixed":
        p = MemXCT(n, m, c, precision="mixed", canonical=True).build()
        p.forward(x.double())
        p.cg(y.double(), 5, residuals=True)
    elif case == "spmm":
        for k, s in ((4, 4), (8, 8)):
            p = MemXCT(n, m, c, slices=s, buffer_entries=2048).build()
            X = torch.from_numpy(np.random.default_rng(k).random((k, n * n), dtype=np.float32)).cuda()
            Y = torch.from_numpy(np.random.default_rng(k + 1).random((k, m * c), dtype=np.float32)).cuda()
            p.forward_batch(X)
            p.back_batch(Y)
            p.cg_batch(Y, 3)
    elif case == "sirt":
        p = MemXCT(n, m, c).build()
        p.sirt(y, 5)
    elif case in ("peer", "collective"):
        nr = 3
        g = LocalGroup(nr)
        ex = "peer" if case == "peer" else "collective"
        plans = ranks(nr, lambda r: MemXCT(n, m, c, group=g, rank=r, vector_order="plan", exchange=ex).build())
        xs = [torch.from_numpy(inputs.uniform(n * n, 1)[p.local_indices(0)]).cuda() for p in plans]
        ys = [torch.from_numpy(inputs.uniform(m * c, 2)[p.local_indices(1)]).cuda() for p in plans]
        torch.cuda.synchronize()
        ranks(nr, lambda r: (plans[r].forward(xs[r]), plans[r].back(ys[r]), plans[r].forward(xs[r]),
                             plans[r].cg(ys[r], 3)))
    else:
        raise SystemExit(f"unknown case {case}")
    torch.cuda.synchronize()
    print("CASE OK", case, flush=True)


if __name__ == "__main__":
    main(sys.argv[1])
