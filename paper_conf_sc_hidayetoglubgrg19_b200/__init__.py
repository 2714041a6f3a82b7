"""B200-native MemXCT hot path (Hidayetoglu et al., SC'19): C-ABI CUDA library + thin binding.

    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    plan = MemXCT(1024, 1500, 1024).build()
    y = plan.forward(x); x = plan.back(y); x = plan.cg(y, iters=30)

The CUDA library (libmemxct.so, built by build_ext.py) is loaded on first use; there is no CPU
fallback.  ``inputs`` holds the seeded synthetic-input generators.
"""
from .memxct import (LocalGroup, MemXCT, MemXCTError, bootstrap_host_comm_name, bootstrap_unique_id,  # noqa: F401
                     get_unique_id, kernel_launch_count, lib, partition_ranges)
