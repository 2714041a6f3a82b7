#!/usr/bin/env python
"""A/B of the partition launch order (MEMXCT_PART_ORDER 0 = partition order, 1 = heaviest
first) on one GPU: forward / back SpMV device time (memxct_spmv_time) and a 30-iteration CG.

    python scripts/order_ab.py --configs 2,3 [--reps 30]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="2,3")
    ap.add_argument("--orders", default="0,1,0,1")
    ap.add_argument("--reps", type=int, default=30)
    ap.add_argument("--env", default="MEMXCT_PART_ORDER")
    a = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    for cfg in map(int, a.configs.split(",")):
        n, m, c = inputs.CONFIGS[cfg]
        y = torch.from_numpy(inputs.uniform(m * c, 2)).cuda()
        for order in a.orders.split(","):
            os.environ[a.env] = order
            t0 = time.perf_counter()
            plan = MemXCT(n, m, c).build()
            build_s = time.perf_counter() - t0
            t = plan.spmv_time(a.reps)
            plan.cg(y, 30)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(3):
                plan.cg(y, 30)
            e1.record()
            torch.cuda.synchronize()
            cg_ms = e0.elapsed_time(e1) / 3
            print(json.dumps({"config": cfg, a.env: order, "fwd_us": round(t["fwd_us"], 2),
                              "back_us": round(t["back_us"], 2), "cg_iter_s": round(30e3 / cg_ms, 1),
                              "build_s": round(build_s, 2)}), flush=True)
            plan.close()
            del plan
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
