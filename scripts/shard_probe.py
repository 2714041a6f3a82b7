#!/usr/bin/env python
"""Per-GPU share of a P-GPU job, one shard at a time on ONE GPU (memxct_plan_set_shard).

    python scripts/shard_probe.py --config 5 --ranks 8 [--which all|0,3,7] [--reps 10]

For every selected rank r of the P-way decomposition (A = R C A_p) this builds rank
r's A_p, A_p^T and exchange maps exactly as rank r of a real P-GPU job would (same tile ranges,
footprint, layouts), times its A_p / A_p^T kernels alone (memxct_spmv_time: the whole B200 to
itself, i.e. what rank r's own GPU runs), and records its memory, build time and exchange
volumes.  One JSON line per rank, then a summary: the slowest rank's forward + back SpMV bounds
a CG iteration of the P-GPU job from below (exchange not included: it needs the other GPUs).
This is how configs whose whole matrix no single GPU holds (config 5: ~346 GB per direction)
are measured in a one-GPU sandbox.  A projection of the compute share, not a multi-GPU run.
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
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--which", default="all")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--ray-block", default="0", help="comma list of MEMXCT_OPT_RAY_BLOCK values (0 = auto)")
    ap.add_argument("--part-rows", default="0", help="comma list of MEMXCT_OPT_PART_ROWS values (0 = auto)")
    args = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    n, m, c = inputs.CONFIGS[args.config]
    P = args.ranks
    which = range(P) if args.which == "all" else [int(v) for v in args.which.split(",")]
    rows = []
    cases = [(r, rb, pr) for r in which for rb in [int(v) for v in args.ray_block.split(",")]
             for pr in [int(v) for v in args.part_rows.split(",")]]
    for r, rb, pr in cases:
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        sp = MemXCT(n, m, c, rank=r, nranks=P, shard=True, vector_order="plan", ray_block=rb,
                    part_rows=pr or None).build()
        torch.cuda.synchronize()
        build_s = time.perf_counter() - t0
        t = sp.spmv_time(args.reps)
        f, b = sp.layout_info(0), sp.layout_info(1)
        cnt = sp.exchange_counts()
        row = {"config": args.config, "P": P, "rank": r, "ray_block": sp.get_option("ray_block"),
               "map_entries": [f["map_entries"], b["map_entries"]], "build_s": round(build_s, 2),
               "device_bytes": sp.stats()["device_bytes"], "nnz": f["nnz"],
               "pixels": sp.local_size(0), "owned_rays": sp.local_size(1), "footprint_rays": f["rows"],
               "fwd_us": t["fwd_us"], "back_us": t["back_us"],
               "fwd_gbs": (6 * f["nnz"] + 8 * f["map_entries"] + 4 * f["rows"]) / (t["fwd_us"] * 1e3),
               "back_gbs": (6 * b["nnz"] + 8 * b["map_entries"] + 4 * b["rows"]) / (t["back_us"] * 1e3),
               "fwd_gflops": 2 * f["nnz"] / (t["fwd_us"] * 1e3), "back_gflops": 2 * b["nnz"] / (t["back_us"] * 1e3),
               "padding": [f["slots"] / f["nnz"] - 1, b["slots"] / b["nnz"] - 1],
               "part_rows": [f["part_rows"], b["part_rows"]], "buffer_entries": [f["buffer_entries"], b["buffer_entries"]],
               "sent": int(cnt["send"].sum() - cnt["send"][r]), "received": int(cnt["recv"].sum() - cnt["recv"][r]),
               "peers": int(sum(1 for q in range(P) if q != r and (cnt["send"][q] or cnt["recv"][q])))}
        rows.append(row)
        print(json.dumps(row), flush=True)
        sp.close()
        del sp
        torch.cuda.empty_cache()
    nnz_tot = sum(x["nnz"] for x in rows)
    slow = max(rows, key=lambda x: x["fwd_us"] + x["back_us"])
    summ = {"summary": True, "config": args.config, "P": P, "ranks_probed": len(rows),
            "nnz_sum": nnz_tot if len(rows) == P else None,
            "nnz_max_over_mean": max(x["nnz"] for x in rows) / (nnz_tot / len(rows)),
            "max_fwd_us": max(x["fwd_us"] for x in rows), "max_back_us": max(x["back_us"] for x in rows),
            "slowest_rank": slow["rank"], "slowest_spmv_pair_us": slow["fwd_us"] + slow["back_us"],
            "cg_iter_s_upper_bound": 1e6 / (max(x["fwd_us"] for x in rows) + max(x["back_us"] for x in rows)),
            "aggregate_gflops": sum(2 * x["nnz"] for x in rows) * 2 / (max(x["fwd_us"] for x in rows) + max(x["back_us"] for x in rows)) / 1e3 if len(rows) == P else None,
            "max_device_gb": max(x["device_bytes"] for x in rows) / 1e9,
            "max_sent": max(x["sent"] for x in rows), "max_peers": max(x["peers"] for x in rows),
            "note": "per-rank kernels timed alone on one B200; CG bound excludes the exchange"}
    print(json.dumps(summ), flush=True)


if __name__ == "__main__":
    main()
