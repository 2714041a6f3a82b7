#!/usr/bin/env python
"""Multi-slice SpMM tuning sweep: rows per CTA x stage buffer x slices.

    python scripts/sweep_spmm.py --config 3 --rows 512,1024 --buffers 4608,9216 --slices 4
"""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--rows", default="1024")
    ap.add_argument("--buffers", default="9216")
    ap.add_argument("--slices", default="4")
    ap.add_argument("--reps", type=int, default=10)
    a = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    n, m, c = inputs.CONFIGS[a.config]
    for K in map(int, a.slices.split(",")):
        X = torch.rand(K, n * n, device="cuda")
        Y = torch.rand(K, m * c, device="cuda")
        for R in map(int, a.rows.split(",")):
            for B in map(int, a.buffers.split(",")):
                if B * 4 * K > 227 * 1024:
                    continue
                plan = MemXCT(n, m, c, part_rows=R, buffer_entries=B, slices=K).build()
                YB, XB = plan.forward_batch(X), plan.back_batch(Y)
                res = {"K": K, "R": R, "B": B}
                for name, fn in (("fwd", lambda: plan.forward_batch(X, YB)), ("back", lambda: plan.back_batch(Y, XB))):
                    fn()
                    ev = [torch.cuda.Event(enable_timing=True) for _ in range(a.reps + 1)]
                    ev[0].record()
                    for i in range(a.reps):
                        fn()
                        ev[i + 1].record()
                    torch.cuda.synchronize()
                    res[name + "_ms"] = float(np.median([ev[i].elapsed_time(ev[i + 1]) for i in range(a.reps)]))
                res["stages"] = [plan.layout_info(0)["stages"], plan.layout_info(1)["stages"]]
                res["ms_per_slice"] = (res["fwd_ms"] + res["back_ms"]) / K
                print(json.dumps(res), flush=True)
                plan.close()
                del plan
                torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
