set -x
scripts/ab_libs.sh gpurun_out/r02n_drift_prefetch_cfg5.jsonl "current nodpf" 2 -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
scripts/ab_libs.sh gpurun_out/r02n_drift_prefetch_cfg5_l2h.jsonl "current nodpf" 1 -- env MEMXCT_L2HINT=1 python scripts/shard_probe.py --config 5 --which 5 --reps 10
python -m pytest tests/test_gpu_drift.py -q -x -p no:cacheprovider > gpurun_out/r02n_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02n_tests.log
