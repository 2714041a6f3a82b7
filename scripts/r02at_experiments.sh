set -x
scripts/ab_env.sh MEMXCT_BALANCE "1 2" 3 gpurun_out/r02at_balance_bench.jsonl -- python bench.py --no-cpu-baseline --no-extras --steps 10 --warmup 3
scripts/ab_env.sh MEMXCT_BALANCE "1 2" 2 gpurun_out/r02at_balance_cfg3.jsonl -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
