#!/usr/bin/env python
"""One profiled region for ncu (--profile-from-start off): build a plan, warm up, then run the
selected call between cudaProfilerStart / Stop.

    ncu --profile-from-start off ... python scripts/prof_region.py --kind collective --what cg --iters 3
kinds: plain | bench (natural order, the bench's plan) | collective | peer | dense (one-rank NCCL
communicator) | mixed (MIXED + CANONICAL)
what:  cg (a CG solve of --iters iterations) | fwd | back | pair
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--kind", default="plain")
    ap.add_argument("--what", default="cg")
    ap.add_argument("--iters", type=int, default=3)
    a = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, get_unique_id, inputs
    n, m, c = inputs.CONFIGS[a.config]
    if a.kind == "plain":
        plan = MemXCT(n, m, c, vector_order="plan").build()
    elif a.kind == "bench":  # the bench's plan: natural vector order, default options
        plan = MemXCT(n, m, c).build()
    elif a.kind == "mixed":
        plan = MemXCT(n, m, c, vector_order="plan", precision="mixed", canonical=True).build()
    else:
        plan = MemXCT(n, m, c, rank=0, nranks=1, unique_id=get_unique_id(), device=0, vector_order="plan",
                      exchange=a.kind).build()
    dt = plan.dtype
    x = torch.rand(plan.local_size(0), device="cuda", dtype=dt)
    y = torch.rand(plan.local_size(1), device="cuda", dtype=dt)
    q, s = torch.empty_like(y), torch.empty_like(x)

    def run():
        if a.what == "cg":
            plan.cg(y, a.iters, x=s)
        if a.what in ("fwd", "pair"):
            plan.forward(x, q)
        if a.what in ("back", "pair"):
            plan.back(y, s)
    run()
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    run()
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print("region done", a.kind, a.what, flush=True)


if __name__ == "__main__":
    main()
