set -x
python -m pytest tests/test_gpu_rle.py tests/test_gpu_drift.py -q -x -p no:cacheprovider > gpurun_out/r02u_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02u_tests.log
scripts/ab_env.sh MEMXCT_RLE "0 1" 2 gpurun_out/r02u_rle_async_cfg5.jsonl -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
