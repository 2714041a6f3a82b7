set -x
scripts/ab_libs.sh gpurun_out/r02an_pa8_bench.jsonl "current pa8" 3 -- python bench.py --no-cpu-baseline --no-extras --steps 10 --warmup 3
scripts/ab_libs.sh gpurun_out/r02an_pa8_cfg3.jsonl "current pa8" 2 -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
