set -x
timeout 1200 python scripts/virtual_scaling.py --config 3 --ranks 2,4,8 --reps 20 > gpurun_out/r02bc_virtual_scaling_cfg3.log 2>&1
timeout 900 python scripts/shard_probe.py --config 4 --ranks 8 --which all --reps 10 > gpurun_out/r02bc_shard_cfg4_p8.jsonl 2> gpurun_out/r02bc_shard_cfg4_p8.err
