set -x
scripts/ab_libs.sh gpurun_out/r02ad_bench_ab.jsonl "current sync" 3 -- python bench.py --no-cpu-baseline --no-extras --steps 10 --warmup 3
