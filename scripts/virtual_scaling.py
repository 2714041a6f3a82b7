#!/usr/bin/env python
"""Compute share of strong scaling, measured on ONE GPU through virtual ranks.

    python scripts/virtual_scaling.py [--config 3] [--ranks 2,4,8] [--reps 20]

For each P the cfg slice is decomposed exactly as P GPUs would decompose it (A = R C A_p,
P:758-811; memxct_local_group_create), then every rank's A_p and A_p^T kernels are timed ALONE
(memxct_spmv_time: one rank at a time, the whole GPU to itself, i.e. what that rank's own B200
would run).  The slowest rank bounds the iteration; E_spmv(P) = T(1) / (P * max_r T_r(P)) is
the parallel efficiency of the SpMV share, before any exchange cost.  Exchange volumes come from
memxct_exchange_info.  This is a projection of the compute share, not a multi-GPU measurement.
"""
import argparse
import json
import os
import sys
import threading

os.environ.setdefault("MEMXCT_BUILD_CHUNK", str(1 << 27))  # P plans build concurrently on one device
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run_ranks(nranks, fn):
    import torch
    out, err = [None] * nranks, [None] * nranks

    def body(r):
        try:
            with torch.cuda.stream(torch.cuda.Stream()):
                out[r] = fn(r)
                torch.cuda.current_stream().synchronize()
        except BaseException as e:  # noqa: BLE001
            err[r] = e
    ts = [threading.Thread(target=body, args=(r,)) for r in range(nranks)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    for e in err:
        if e is not None:
            raise e
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--ranks", default="2,4,8")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--part-rows", default="0", help="comma list of PART_ROWS to sweep (0 = auto)")
    args = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import LocalGroup, MemXCT, inputs
    n, m, c = inputs.CONFIGS[args.config]
    p1 = MemXCT(n, m, c).build()
    t1 = p1.spmv_time(args.reps)
    print("P=1 layouts", json.dumps([p1.layout_info(0), p1.layout_info(1)]), flush=True)
    base = t1["fwd_us"] + t1["back_us"]
    nnz1 = p1.layout_info(0)["nnz"]
    p1.close()
    rows = [{"P": 1, "fwd_us": [t1["fwd_us"]], "back_us": [t1["back_us"]], "max_us": base, "E_spmv": 1.0}]
    print(json.dumps(rows[0]), flush=True)
    cases = [(P, R) for P in [int(v) for v in args.ranks.split(",")] for R in [int(v) for v in args.part_rows.split(",")]]
    for P, R in cases:
        g = LocalGroup(P)
        kw = {"part_rows": R} if R else {}
        plans = run_ranks(P, lambda r: MemXCT(n, m, c, group=g, rank=r, vector_order="plan", **kw).build())
        torch.cuda.synchronize()
        times = [p.spmv_time(args.reps) for p in plans]  # one rank at a time, whole GPU each
        info = [p.exchange_info() for p in plans]
        nnz = [p.layout_info(0)["nnz"] for p in plans]
        tot = [t["fwd_us"] + t["back_us"] for t in times]
        lay = [(p.layout_info(0), p.layout_info(1)) for p in plans]
        gbs = [(6 * f["slots"] + 8 * f["map_entries"] + 4 * f["rows"]) / (t["fwd_us"] * 1e3) for (f, b), t in zip(lay, times)]
        gbs_b = [(6 * b["slots"] + 8 * b["map_entries"] + 4 * b["rows"]) / (t["back_us"] * 1e3) for (f, b), t in zip(lay, times)]
        row = {"P": P, "fwd_gbs": gbs, "back_gbs": gbs_b,
               "map_entries": [(f["map_entries"], b["map_entries"]) for f, b in lay],
               "part_rows": [(p.layout_info(0)["part_rows"], p.layout_info(1)["part_rows"]) for p in plans],
               "max_fwd_us": max(t["fwd_us"] for t in times), "max_back_us": max(t["back_us"] for t in times),
               "fwd_us": [t["fwd_us"] for t in times], "back_us": [t["back_us"] for t in times],
               "max_us": max(tot), "E_spmv": base / (P * max(tot)),
               "nnz_imbalance": max(nnz) / (sum(nnz) / P), "nnz_sum_ok": sum(nnz) == nnz1,
               "footprint_rays": [i["footprint_rays"] for i in info],
               "sent_entries": [i["sent"] for i in info], "peers": [i["peers"] for i in info]}
        print(json.dumps(row), flush=True)
        rows.append(row)
        for p in plans:
            p.close()
        del plans
        g.close()
        torch.cuda.synchronize()
    print("\n| P | max rank fwd+back us | E_spmv | nnz imbalance | max sent entries/rank | max peers |")
    print("|---|---|---|---|---|---|")
    for r in rows:
        print(f"| {r['P']} | {r['max_us']:.1f} | {r['E_spmv']:.3f} | {r.get('nnz_imbalance', 1.0):.3f} | "
              f"{max(r.get('sent_entries', [0]))} | {max(r.get('peers', [0]))} |")


if __name__ == "__main__":
    main()
