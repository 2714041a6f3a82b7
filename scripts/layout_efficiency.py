#!/usr/bin/env python
"""Where a staged SpMV layout loses time to synchronisation (read from memxct_layout_export).

    python scripts/layout_efficiency.py --config 5 --shard 1/8 [--ray-block 8] [--parts 64]

For a sample of partitions (CTAs) of each direction: per stage, a warp runs max_l(n_l) chunk
iterations (lanes in lockstep) and the CTA waits at the stage barrier for its slowest warp.
Reports, over the sample:
  lane_eff    = sum of lane chunks / (32 x sum over warps and stages of the warp's max chunks)
  barrier_eff = sum over stages of the mean warp time / sum over stages of the max warp time
  chunks_per_stage, active_warps (warps with any chunk in a stage), stages per partition,
  reuse (nonzeros / map entries).
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def analyse(plan, d, parts, rng):
    info = plan.layout_info(d)
    npart = info["parts"]
    pick = np.sort(rng.choice(npart, min(parts, npart), replace=False))
    spp = info["part_rows"] // 32
    lane, warp_max, mean_w, max_w, active, nst = 0, 0, 0.0, 0.0, [], []
    for p in pick:
        ex = plan.layout_export(d, int(p), int(p) + 1)
        ns = int(ex["stage_base"][1] - ex["stage_base"][0])
        nst.append(ns)
        lc = ex["lane_chunks"].reshape(ns, spp, 32).astype(np.int64)
        wm = lc.max(axis=2)                       # [stage, warp] iterations of each warp
        lane += lc.sum()
        warp_max += wm.sum()
        mean_w += wm.mean(axis=1).sum()
        max_w += wm.max(axis=1).sum()
        active.extend((wm > 0).sum(axis=1).tolist())
    return {"dir": d, "parts_sampled": len(pick), "lane_eff": lane / (32 * warp_max),
            "barrier_eff": mean_w / max_w, "stages_per_part": float(np.mean(nst)),
            "active_warps_mean": float(np.mean(active)), "warps": spp,
            "reuse": info["nnz"] / info["map_entries"], "part_rows": info["part_rows"],
            "buffer_entries": info["buffer_entries"]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--shard", default=None, help="r/P: one rank's shard")
    ap.add_argument("--ray-block", type=int, default=0)
    ap.add_argument("--stage-order", type=int, default=0)
    ap.add_argument("--parts", type=int, default=64)
    ap.add_argument("--part-rows", type=int, default=None)
    ap.add_argument("--buffer-entries", type=int, default=None)
    args = ap.parse_args()
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    n, m, c = inputs.CONFIGS[args.config]
    kw = {"ray_block": args.ray_block, "stage_order": args.stage_order, "part_rows": args.part_rows, "buffer_entries": args.buffer_entries}
    if args.shard:
        r, P = map(int, args.shard.split("/"))
        plan = MemXCT(n, m, c, rank=r, nranks=P, shard=True, vector_order="plan", **kw).build()
    else:
        plan = MemXCT(n, m, c, **kw).build()
    rng = np.random.default_rng(0)
    t = plan.spmv_time(5)
    for d in (0, 1):
        row = analyse(plan, d, args.parts, rng)
        row.update({"config": args.config, "shard": args.shard, "ray_block": plan.get_option("ray_block"),
                    "stage_order": plan.get_option("stage_order"),
                    "us": t["fwd_us" if d == 0 else "back_us"]})
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
