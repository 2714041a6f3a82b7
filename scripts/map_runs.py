#!/usr/bin/env python
"""Run-length statistics of the forward stage maps (how many map entries are consecutive input
indices): sizes a run-length map encoding.  One JSON line.

    python scripts/map_runs.py --config 5 --rank 5 --ranks 8 --parts 200
    python scripts/map_runs.py --config 3 --parts 200          (single GPU plan)
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--rank", type=int, default=5)
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--parts", type=int, default=200)
    ap.add_argument("--dir", type=int, default=0)
    a = ap.parse_args()
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    n, m, c = inputs.CONFIGS[a.config]
    if a.config == 5:
        plan = MemXCT(n, m, c, rank=a.rank, nranks=a.ranks, shard=True, vector_order="plan").build()
    else:
        plan = MemXCT(n, m, c, vector_order="plan").build()
    info = plan.layout_info(a.dir)
    rng = np.random.default_rng(0)
    parts = np.sort(rng.choice(info["parts"], min(a.parts, info["parts"]), replace=False))
    B = info["buffer_entries"]
    runs, entries, stages = [], 0, 0
    for p in parts:
        L = plan.layout_export(a.dir, int(p), int(p) + 1)
        mp = L["map"]
        ns = int(L["stage_base"][1] - L["stage_base"][0])
        for s in range(ns):
            seg = mp[s * B:(s + 1) * B].astype(np.int64)
            if len(seg) == 0:
                continue
            brk = np.nonzero(np.diff(seg) != 1)[0]
            lens = np.diff(np.concatenate([[0], brk + 1, [len(seg)]]))
            runs.append(lens)
            entries += len(seg)
            stages += 1
    r = np.concatenate(runs)
    out = {"config": a.config, "dir": a.dir, "parts_sampled": len(parts), "stages": stages, "entries": entries,
           "runs": int(len(r)), "mean_run": entries / len(r), "median_run": float(np.median(r)),
           "frac_entries_in_runs_ge8": float(r[r >= 8].sum() / entries),
           "frac_entries_in_runs_ge32": float(r[r >= 32].sum() / entries),
           "rle_bytes_per_entry_6B_runs": 6 * len(r) / entries,
           "map_entries_total": info["map_entries"], "nnz": info["nnz"]}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
