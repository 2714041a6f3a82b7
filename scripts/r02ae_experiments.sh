set -x
scripts/ab_libs.sh gpurun_out/r02ae_nextpf_bench.jsonl "current nextpf" 3 -- python bench.py --no-cpu-baseline --no-extras --steps 10 --warmup 3
scripts/ab_libs.sh gpurun_out/r02ae_nextpf_cfg3.jsonl "current nextpf" 2 -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
