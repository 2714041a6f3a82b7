#!/usr/bin/env python
"""Build a P-rank virtual decomposition of a config on one GPU and run ONE rank's SpMV kernels
(memxct_spmv_time, reps = 1: forward, back, forward, back), for an ncu capture of that rank's
kernels, e.g.

    ncu --set full -k regex:spmv_f32 --launch-skip 3 --launch-count 1 -o rank_back \\
        python scripts/prof_rank.py --config 3 --ranks 8 --rank 1
"""
import argparse
import os
import sys
import threading

os.environ.setdefault("MEMXCT_BUILD_CHUNK", str(1 << 27))
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--rank", type=int, default=1)
    ap.add_argument("--part-rows", type=int, default=0)
    args = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import LocalGroup, MemXCT, inputs
    n, m, c = inputs.CONFIGS[args.config]
    g = LocalGroup(args.ranks)
    plans = [None] * args.ranks
    kw = {"part_rows": args.part_rows} if args.part_rows else {}

    def body(r):
        with torch.cuda.stream(torch.cuda.Stream()):
            plans[r] = MemXCT(n, m, c, group=g, rank=r, vector_order="plan", **kw).build()
            torch.cuda.current_stream().synchronize()
    ts = [threading.Thread(target=body, args=(r,)) for r in range(args.ranks)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    torch.cuda.synchronize()
    p = plans[args.rank]
    print("layout", p.layout_info(0), p.layout_info(1), flush=True)
    print("time", p.spmv_time(1), flush=True)


if __name__ == "__main__":
    main()
