set -x
python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "mixed or canonical or cg" > gpurun_out/r02l_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02l_tests.log
scripts/ab_env.sh MEMXCT_CANONICAL_DOT_INLINE "0 1" 2 gpurun_out/r02l_canon_dot.jsonl -- python scripts/mixed_probe.py --config 3
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv python scripts/prof_region.py --kind mixed --what cg --iters 3 > gpurun_out/r02l_cg_launches_mixed.csv 2>&1
timeout 900 python bench.py --gpus 2 --transport host --config 2 --steps 3 --warmup 3 > gpurun_out/r02l_bench_host2.json 2> gpurun_out/r02l_bench_host2.err; echo "BENCH EXIT $?" >> gpurun_out/r02l_bench_host2.err
