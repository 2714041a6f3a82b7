import sys, os
sys.path.insert(0, "/root/repo")
import torch
from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, get_unique_id, inputs
n, m, c = inputs.CONFIGS[2]
kind = sys.argv[1]
plan = MemXCT(n, m, c, rank=0, nranks=1, unique_id=get_unique_id(), device=0, vector_order="plan", exchange=kind).build()
y = torch.rand(plan.local_size(1), device="cuda")
x = torch.empty(plan.local_size(0), device="cuda")
plan.cg(y, 4, x=x)
torch.cuda.synchronize()
plan.cg(y, 4, x=x)
torch.cuda.synchronize()
