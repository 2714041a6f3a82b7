set -x
python -m pytest tests/test_gpu_peer_exchange.py tests/test_gpu_multiprocess.py tests/test_gpu_p8.py tests/test_gpu_multirank.py tests/test_gpu_rle.py -q -x -p no:cacheprovider > gpurun_out/r02k_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02k_tests.log
python scripts/exchange_overhead.py --config 2 --rounds 3 > gpurun_out/r02k_overhead_cfg2.jsonl 2>&1
python scripts/exchange_overhead.py --config 3 --rounds 3 > gpurun_out/r02k_overhead_cfg3.jsonl 2>&1
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv python scripts/prof_region.py --kind peer --what cg --iters 3 > gpurun_out/r02k_cg_launches_peer.csv 2>&1
scripts/ab_env.sh MEMXCT_RLE "0 1" 2 gpurun_out/r02k_rle_cfg5.jsonl -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
