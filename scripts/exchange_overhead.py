#!/usr/bin/env python
"""Per-call cost of the P > 1 machinery on a one-rank NCCL communicator (one GPU): forward,
back and one CG iteration of the decomposed path with each exchange (collective all-to-allv,
fused peer memory, dense reduce-scatter) against the plain single-GPU plan.  At P = 1 the
exchange moves nothing, so the differences are the fixed costs per call (extra kernels, flags,
fences, collectives) that a P-GPU run pays on top of its share of the SpMVs.

    python scripts/exchange_overhead.py [--config 3] [--reps 20]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--rounds", type=int, default=5)
    a = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, get_unique_id, inputs
    n, m, c = inputs.CONFIGS[a.config]

    def timed(fn, reps):
        fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps * 1e3  # us

    plans = {}
    for kind in ("plain", "collective", "peer", "dense"):
        if kind == "plain":
            plans[kind] = MemXCT(n, m, c, vector_order="plan").build()
        else:
            plans[kind] = MemXCT(n, m, c, rank=0, nranks=1, unique_id=get_unique_id(), device=0,
                                 vector_order="plan", exchange=kind).build()
    res = {k: {"fwd": [], "back": [], "cg": []} for k in plans}
    # interleaved rounds (ABCD ABCD ...): clock drift of the power-capped box hits every kind alike
    for _ in range(a.rounds):
        for kind, plan in plans.items():
            x = torch.rand(plan.local_size(0), device="cuda")
            y = torch.rand(plan.local_size(1), device="cuda")
            q, s = torch.empty_like(y), torch.empty_like(x)
            res[kind]["fwd"].append(timed(lambda: plan.forward(x, q), a.reps))
            res[kind]["back"].append(timed(lambda: plan.back(y, s), a.reps))
            c10 = timed(lambda: plan.cg(y, 10, x=s), 3)
            c40 = timed(lambda: plan.cg(y, 40, x=s), 3)
            res[kind]["cg"].append((c40 - c10) / 30)
    import numpy as np
    base = float(np.median(res["plain"]["cg"]))
    for kind in plans:
        med = {k: float(np.median(v)) for k, v in res[kind].items()}
        print(json.dumps({"config": a.config, "exchange": kind, "fwd_us": round(med["fwd"], 1),
                          "back_us": round(med["back"], 1), "cg_iter_us": round(med["cg"], 1),
                          "cg_iter_minus_plain_us": round(med["cg"] - base, 1), "rounds": a.rounds,
                          "cg_iter_samples": [round(v, 1) for v in res[kind]["cg"]]}), flush=True)


if __name__ == "__main__":
    main()
