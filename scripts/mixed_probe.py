#!/usr/bin/env python
"""MIXED (+ CANONICAL) SpMV and CG timing at one config (one JSON line): the parity-gated mode
of reading R16 against the FP32 default.

    python scripts/mixed_probe.py --config 3 [--canonical 1] [--iters 30]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--canonical", type=int, default=1)
    ap.add_argument("--iters", type=int, default=30)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--buffers", default="0", help="comma list of BUFFER_ENTRIES (fp32 units; 0 = auto)")
    a = ap.parse_args()
    from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
    n, m, c = inputs.CONFIGS[a.config]
    for b in map(int, a.buffers.split(",")):
        run(a, n, m, c, b or None)


def run(a, n, m, c, buf):
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    plan = MemXCT(n, m, c, precision="mixed", canonical=bool(a.canonical), buffer_entries=buf).build()
    y = plan.forward(torch.from_numpy(inputs.shepp_logan(n)).cuda())
    x = torch.empty(n * n, dtype=torch.float64, device="cuda")
    plan.cg(y, a.iters, x=x)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(a.reps):
        plan.cg(y, a.iters, x=x)
    e1.record()
    torch.cuda.synchronize()
    sp = plan.spmv_time(10)
    print(json.dumps({"config": a.config, "canonical": a.canonical, "cg_iter_s": a.iters * a.reps / (e0.elapsed_time(e1) * 1e-3),
                      "fwd_ms": sp["fwd_us"] / 1e3, "back_ms": sp["back_us"] / 1e3,
                      "buffer_entries": [plan.layout_info(0)["buffer_entries"], plan.layout_info(1)["buffer_entries"]]}),
          flush=True)
    plan.close()


if __name__ == "__main__":
    main()
