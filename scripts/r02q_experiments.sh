set -x
scripts/ab_env.sh MEMXCT_L2_PERSIST "0 1 0.5" 2 gpurun_out/r02q_persist_cfg5.jsonl -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
scripts/ab_env.sh MEMXCT_L2_PERSIST "0 1" 2 gpurun_out/r02q_persist_cfg3.jsonl -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
MEMXCT_L2_PERSIST=1 python scripts/shard_probe.py --config 5 --which 5 --reps 1 2>&1 | grep memxct > gpurun_out/r02q_persist_info.txt
