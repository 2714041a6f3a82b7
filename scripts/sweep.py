#!/usr/bin/env python
"""Tuning sweep of the SpMV layout parameters on one GPU (the B200 analog of the paper's
block-size x buffer-size heat maps, Fig. 10).

    python scripts/sweep.py --config 3 --rows 256,512,1024 --buffers 8192,12288,16384

For every (rows per partition, buffer entries) it builds the plan, times forward and back SpMV
with CUDA events (median of --reps launches each) and prints one JSON line.
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--rows", default="512")
    ap.add_argument("--buffers", default="12288")
    ap.add_argument("--reps", type=int, default=15)
    ap.add_argument("--cg", action="store_true", help="also time a 30-iteration CG")
    a = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    n, m, c = inputs.CONFIGS[a.config]
    x = torch.from_numpy(inputs.uniform(n * n, 1)).cuda()
    y = torch.from_numpy(inputs.uniform(m * c, 2)).cuda()
    for R in map(int, a.rows.split(",")):
        for B in map(int, a.buffers.split(",")):
            t0 = time.perf_counter()
            plan = MemXCT(n, m, c, part_rows=R, buffer_entries=B).build()
            build_s = time.perf_counter() - t0
            fi, bi = plan.layout_info(0), plan.layout_info(1)
            yo, xo = plan.forward(x), plan.back(y)
            res = {}
            for name, fn in (("fwd", lambda: plan.forward(x, yo)), ("back", lambda: plan.back(y, xo))):
                for _ in range(3):
                    fn()
                ev = [torch.cuda.Event(enable_timing=True) for _ in range(a.reps + 1)]
                ev[0].record()
                for i in range(a.reps):
                    fn()
                    ev[i + 1].record()
                torch.cuda.synchronize()
                t = float(np.median([ev[i].elapsed_time(ev[i + 1]) for i in range(a.reps)]))
                info = fi if name == "fwd" else bi
                algo = 6 * info["nnz"] + 8 * info["map_entries"] + 4 * info["rows"]
                res[name] = {"ms": t, "gbs_algo": algo / t / 1e6,
                             "gbs_stored": (6 * info["slots"] + 4 * info["map_entries"]) / t / 1e6,
                             "pad": info["slots"] / max(info["nnz"], 1) - 1, "stages": info["stages"],
                             "parts": info["parts"]}
            if a.cg:
                plan.cg(yo, 30)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                for _ in range(3):
                    plan.cg(yo, 30)
                e1.record()
                torch.cuda.synchronize()
                res["cg_ms_per_iter"] = e0.elapsed_time(e1) / 90
            print(json.dumps({"R": R, "B": B, "build_s": build_s, **res}), flush=True)
            plan.close()
            del plan
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
