#!/usr/bin/env python
"""Summarise ncu output into profiles/ (tracked):

    python scripts/ncu_summary.py --launches gpurun_out/launches.csv \
        --report gpurun_out/prof_spmv.ncu-rep --tag r01 --config 3

Writes profiles/<tag>_launches.md (per-kernel share of device time from the serialised launch
list), profiles/<tag>_spmv_full.csv (selected raw metrics of the `--set full` capture) and
profiles/ncu_spmv_cfg<config>.json (per-launch DRAM traffic that bench.py reports as
roofline.traffic).
"""
import argparse
import collections
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "dram__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "lts__t_sector_hit_rate.pct",
           "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
           "sm__throughput.avg.pct_of_peak_sustained_elapsed",
           "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "smsp__inst_executed.sum",
           "launch__grid_size", "launch__block_size", "l1tex__throughput.avg.pct_of_peak_sustained_active",
           "lts__throughput.avg.pct_of_peak_sustained_elapsed", "sm__cycles_elapsed.avg.per_second"]


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr, data = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            data.append(dict(zip(hdr, r)))
    agg = collections.OrderedDict()
    for d in data:
        name = d["Kernel Name"].split("(")[0]
        agg.setdefault(name, []).append(float(d["Metric Value"]) / 1e3)  # ns -> us
    total = sum(sum(v) for v in agg.values())
    out = ["| kernel | launches | total ms | avg us | share |", "|---|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        out.append(f"| `{k}` | {len(v)} | {sum(v)/1e3:.3f} | {sum(v)/len(v):.1f} | {100*sum(v)/total:.1f}% |")
    return "\n".join(out), agg


def report(path):
    txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    keep = ["Kernel Name"] + [m for m in METRICS if m in hdr]
    res = []
    for r in rows[2:]:
        if len(r) == len(hdr):
            res.append({k: r[hdr.index(k)] for k in keep})
    return res, {k: units[hdr.index(k)] for k in keep}


def to_bytes(v, unit):
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}[unit]
    return float(v) * scale


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--report")
    ap.add_argument("--tag", required=True)
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--note", default="")
    a = ap.parse_args()
    prof = os.path.join(ROOT, "profiles")
    os.makedirs(prof, exist_ok=True)
    if a.launches:
        md, _ = launches(a.launches)
        with open(os.path.join(prof, f"{a.tag}_launches.md"), "w") as f:
            f.write(f"# ncu launch list ({a.tag}) -- cold-cache, serialised; compare shares\n\n")
            f.write(a.note + "\n\n" + md + "\n")
    if a.report:
        res, units = report(a.report)
        with open(os.path.join(prof, f"{a.tag}_spmv_full.csv"), "w", newline="") as f:
            w = csv.DictWriter(f, fieldnames=list(units.keys()))
            w.writeheader()
            w.writerow(units)
            for r in res:
                w.writerow(r)
        traffic = [to_bytes(r["dram__bytes_read.sum"], units["dram__bytes_read.sum"]) +
                   to_bytes(r["dram__bytes_write.sum"], units["dram__bytes_write.sum"]) for r in res]
        summ = {"tag": a.tag, "config": a.config, "source": os.path.basename(a.report),
                "kernels": [r["Kernel Name"] for r in res],
                "traffic_bytes_per_launch_each": traffic,
                "traffic_bytes_per_launch": sum(traffic) / len(traffic) if traffic else None,
                "note": a.note}
        with open(os.path.join(prof, f"ncu_spmv_cfg{a.config}.json"), "w") as f:
            json.dump(summ, f, indent=1)


if __name__ == "__main__":
    main()
