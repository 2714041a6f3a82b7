"""One rank of a multi-PROCESS job on one GPU (memxct_plan_set_comm_host), started by
tests/test_gpu_multiprocess.py: torch.distributed (gloo) only bootstraps the shared-memory name
and the final barrier; every collective and exchange of the build and of the operators runs in
libmemxct (host transport: CUDA-IPC device mailboxes; EXCHANGE = 1: cudaIpcOpenMemHandle
peer mappings, system-scope flags and credits across the process boundary).

    python proc_cases.py OUT_DIR EXCHANGE N M C      (env: RANK, WORLD_SIZE, MASTER_ADDR/PORT)

Writes OUT_DIR/rank<r>.npz with the rank's local indices and outputs."""
import os
import sys

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(HERE))


def main():
    out_dir, exchange = sys.argv[1], sys.argv[2]
    n, m, c = map(int, sys.argv[3:6])
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(0)
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, bootstrap_host_comm_name, inputs
    name = bootstrap_host_comm_name(rank)
    plan = MemXCT(n, m, c, rank=rank, nranks=world, host_comm=name, device=0, vector_order="plan",
                  exchange=exchange).build()
    pix, ray = plan.local_indices(0), plan.local_indices(1)
    x = torch.from_numpy(inputs.uniform(n * n, 1)[pix]).cuda()
    y = torch.from_numpy(inputs.uniform(m * c, 2)[ray]).cuda()
    out = {}
    out["f1"] = plan.forward(x)
    out["f2"] = plan.forward(2 * x)
    out["b1"] = plan.back(y)
    out["b3"] = plan.back(3 * y)
    out["f1b"] = plan.forward(x)
    out["b1b"] = plan.back(y)
    out["cg10"], r10 = plan.cg(y, 10, residuals=True)
    out["cg30"], r30 = plan.cg(y, 30, residuals=True)
    torch.cuda.synchronize()
    info = plan.exchange_info()
    np.savez(os.path.join(out_dir, f"rank{rank}.npz"), pix=pix, ray=ray, r10=r10, r30=r30,
             peers=info["peers"], sent=info["sent"], **{k: v.cpu().numpy() for k, v in out.items()})
    plan.close()
    dist.barrier()
    dist.destroy_process_group()
    print("CASE OK", rank, exchange, flush=True)


if __name__ == "__main__":
    main()
