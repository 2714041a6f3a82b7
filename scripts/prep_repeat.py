#!/usr/bin/env python
"""Preprocessing timing stability: in one process, build the bench plan (config 3) and then the
paper's ADS2 shape several times, printing memxct_build_phases of each build (one JSON line per
build).  Separates first-use costs (module loading, allocator state) from the steady build time.

    python scripts/prep_repeat.py [--reps 3] [--rds1 1]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--rds1", type=int, default=1)
    ap.add_argument("--like-bench", type=int, default=0,
                    help="run what bench.py runs on the config-3 plan before the other builds (CG graph, "
                         "SpMV launches, host-buffer CG)")
    a = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    shapes = [("cfg3", (1024, 1500, 1024))] + [("ADS2", (512, 750, 512))] * a.reps
    if a.rds1:
        shapes += [("RDS1", (2048, 1501, 2048))] * 2
    keep = None
    for name, (n, m, c) in shapes:
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        p = MemXCT(n, m, c).build()
        torch.cuda.synchronize()
        wall = time.perf_counter() - t0
        free, tot = torch.cuda.mem_get_info()
        print(json.dumps({"shape": name, "build_s": wall, "phases_s": p.build_phases(),
                          "free_gb_after": free / 1e9, "module_loading": os.environ.get("CUDA_MODULE_LOADING")}),
              flush=True)
        if name == "cfg3":
            keep = p  # alive like the bench plan
            if a.like_bench:
                y = torch.rand(p.local_size(1), device="cuda")
                x = torch.empty(p.local_size(0), device="cuda")
                st = torch.cuda.current_stream()
                for _ in range(4):
                    p.cg(y, 30, x=x, stream=st)
                yb, xb = torch.empty_like(y), torch.empty_like(x)
                for _ in range(5):
                    p.forward(x, yb, stream=st)
                    p.back(y, xb, stream=st)
                torch.cuda.synchronize()
                if a.like_bench > 1:
                    yh = torch.empty(p.local_size(1), dtype=torch.float32, pin_memory=True)
                    xh = torch.empty(p.local_size(0), dtype=torch.float32, pin_memory=True)
                    yh.copy_(y.cpu())
                    for _ in range(2):
                        p.cg_host_ptr(yh.data_ptr(), xh.data_ptr(), 30, stream=st)
                torch.cuda.synchronize()
        else:
            p.close()
    del keep


if __name__ == "__main__":
    main()
