set -x
scripts/ab_libs.sh gpurun_out/r02al_phead_bench.jsonl "current phead" 3 -- python bench.py --no-cpu-baseline --no-extras --steps 10 --warmup 3
scripts/ab_libs.sh gpurun_out/r02al_phead_cfg3.jsonl "current phead" 2 -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
scripts/ab_libs.sh gpurun_out/r02al_phead_cfg5.jsonl "current phead" 2 -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
