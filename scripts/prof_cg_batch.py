#!/usr/bin/env python
"""Multi-slice CG at cfg3 (for an ncu launch list: every kernel of a K-slice CGLS iteration).

    ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file out.csv \
        python scripts/prof_cg_batch.py 4 3
Also prints the CUDA-event time per iteration (uncaptured by ncu only when run without it).
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 4
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 3
n, m, c = inputs.CONFIGS[3]
plan = MemXCT(n, m, c, slices=K).build()
X0 = torch.rand(K, n * n, device="cuda")
Y = plan.forward_batch(X0)
X = plan.cg_batch(Y, iters)
torch.cuda.synchronize()
ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
ev[0].record()
plan.cg_batch(Y, iters, X)
ev[1].record()
plan.forward_batch(X0, Y)
ev[2].record()
plan.back_batch(Y, X)
ev[3].record()
torch.cuda.synchronize()
print({"K": K, "iters": iters, "cg_ms_per_iter": ev[0].elapsed_time(ev[1]) / iters,
       "fwd_batch_ms": ev[1].elapsed_time(ev[2]), "back_batch_ms": ev[2].elapsed_time(ev[3])}, flush=True)
