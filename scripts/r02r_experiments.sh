set -x
python -m pytest tests/test_gpu_drift.py -q -x -p no:cacheprovider > gpurun_out/r02r_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02r_tests.log
scripts/ab_libs.sh gpurun_out/r02r_async_cfg5.jsonl "current sync" 2 -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
scripts/ab_env.sh MEMXCT_DRIFT "0 1" 2 gpurun_out/r02r_async_drift_cfg3.jsonl -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
scripts/ab_env.sh MEMXCT_DRIFT "0 1" 1 gpurun_out/r02r_async_drift_cfg5.jsonl -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
