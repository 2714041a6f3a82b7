#!/usr/bin/env python
"""Large-config probe on one GPU: build, SpMV timings, a short CG (parity lives in tests/).

    python scripts/big_config.py --config 4 [--iters 5]

Prints one JSON line (build seconds, layout sizes, device bytes, fwd/back ms and GB/s, CG ms per
iteration)."""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--iters", type=int, default=5)
    a = ap.parse_args()
    import torch

    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    n, m, c = inputs.CONFIGS[a.config]
    out = {"config": a.config, "n": n, "m": m, "c": c}
    t0 = time.perf_counter()
    plan = MemXCT(n, m, c).build()
    torch.cuda.synchronize()
    out["build_s"] = time.perf_counter() - t0
    out["stats"] = plan.stats()
    out["fwd"] = plan.layout_info(0)
    out["back"] = plan.layout_info(1)
    out["gpu_mem_used_gb"] = (torch.cuda.mem_get_info()[1] - torch.cuda.mem_get_info()[0]) / 1e9
    x = torch.from_numpy(inputs.uniform(n * n, inputs.seed_for(a.config))).cuda()
    y = plan.forward(x)
    xb = plan.back(y)
    for name, fn, info in (("fwd", lambda: plan.forward(x, y), out["fwd"]), ("back", lambda: plan.back(y, xb), out["back"])):
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(6)]
        ev[0].record()
        for i in range(5):
            fn()
            ev[i + 1].record()
        torch.cuda.synchronize()
        ms = float(np.median([ev[i].elapsed_time(ev[i + 1]) for i in range(5)]))
        algo = 6 * info["nnz"] + 8 * info["map_entries"] + 4 * info["rows"]
        out[name + "_ms"] = ms
        out[name + "_gbs"] = algo / ms / 1e6
    plan.cg(y, a.iters)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    plan.cg(y, a.iters)
    e1.record()
    torch.cuda.synchronize()
    out["cg_ms_per_iter"] = e0.elapsed_time(e1) / a.iters
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
