#!/usr/bin/env python
"""Per-iteration cost of the CGLS graph against its two SpMVs (cfg3 by default).

    python scripts/cg_breakdown.py [--config 3] [--iters 10,40]

Times memxct_cg at two iteration counts (CUDA events, graph replays) and takes the slope as the
cost of one iteration; compares it with the forward + back SpMV kernels timed alone
(memxct_spmv_time).  The difference is the vector steps, the fused dots and the kernel
boundaries inside the graph."""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--iters", default="10,40")
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    n, m, c = inputs.CONFIGS[a.config]
    plan = MemXCT(n, m, c).build()
    x = torch.from_numpy(inputs.shepp_logan(n).astype(np.float32)).cuda()
    y = plan.forward(x)
    xo = torch.empty_like(x)
    out = {"config": a.config}
    ks = [int(v) for v in a.iters.split(",")]
    for k in ks:
        plan.cg(y, k, x=xo)
        ts = []
        for _ in range(a.reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.cg(y, k, x=xo)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        out[f"cg{k}_ms"] = float(np.median(ts))
    out["iter_ms"] = (out[f"cg{ks[1]}_ms"] - out[f"cg{ks[0]}_ms"]) / (ks[1] - ks[0])
    t = plan.spmv_time(20)
    out["spmv_pair_ms"] = (t["fwd_us"] + t["back_us"]) / 1e3
    # the same two kernels alternating on real vectors (forward into q, back into s), as in CG
    q, s_ = torch.empty_like(y), torch.empty_like(x)
    for _ in range(3):
        plan.forward(x, q)
        plan.back(y, s_)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        plan.forward(x, q)
        plan.back(y, s_)
    e1.record()
    torch.cuda.synchronize()
    out["alternating_pair_ms"] = e0.elapsed_time(e1) / 20
    out["overhead_us"] = 1e3 * (out["iter_ms"] - out["spmv_pair_ms"])
    out["overhead_frac"] = out["overhead_us"] / 1e3 / out["iter_ms"]
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
