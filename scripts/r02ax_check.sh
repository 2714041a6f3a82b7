set -x
python -m pytest tests/test_gpu_drift.py tests/test_gpu_ray_block.py tests/test_gpu_rle.py tests/test_gpu_shard.py -q -x -p no:cacheprovider > gpurun_out/r02ax_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02ax_tests.log
python scripts/shard_probe.py --config 5 --ranks 8 --which all --reps 10 > gpurun_out/r02ax_shard_cfg5_p8.jsonl 2> gpurun_out/r02ax_shard_cfg5_p8.err
