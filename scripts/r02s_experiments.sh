set -x
python -m pytest tests/test_gpu_drift.py tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/r02s_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02s_tests.log
scripts/ab_libs.sh gpurun_out/r02s_head_cfg5.jsonl "current nohead" 2 -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
scripts/ab_libs.sh gpurun_out/r02s_head_cfg3.jsonl "current nohead" 3 -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
scripts/ab_libs.sh gpurun_out/r02s_head_mixed.jsonl "current nohead" 2 -- python scripts/mixed_probe.py --config 3
