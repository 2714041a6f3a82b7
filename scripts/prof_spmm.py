#!/usr/bin/env python
"""Run a few multi-slice SpMMs (for ncu -k regex:spmm)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 4
n, m, c = inputs.CONFIGS[3]
plan = MemXCT(n, m, c, slices=K).build()
X = torch.rand(K, n * n, device="cuda")
Y = plan.forward_batch(X)
for _ in range(3):
    plan.forward_batch(X, Y)
    plan.back_batch(Y)
torch.cuda.synchronize()
