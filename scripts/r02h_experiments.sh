set -x
python -m pytest tests/test_gpu_rle.py -q -x -p no:cacheprovider > gpurun_out/r02h_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02h_tests.log
MEMXCT_RLE=1 python -m pytest tests/test_gpu_parity.py tests/test_gpu_drift.py tests/test_gpu_peer_exchange.py -q -x -p no:cacheprovider -k "not full_size and not cfg3" >> gpurun_out/r02h_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02h_tests.log
scripts/ab_env.sh MEMXCT_RLE "0 1" 2 gpurun_out/r02h_rle_cfg3.jsonl -- python scripts/big_config.py --config 3 --iters 5
scripts/ab_env.sh MEMXCT_RLE "0 1" 2 gpurun_out/r02h_rle_cfg5.jsonl -- python scripts/shard_probe.py --config 5 --which 5 --reps 20
scripts/ab_env.sh MEMXCT_RLE "0 1" 1 gpurun_out/r02h_rle_mixed.jsonl -- python scripts/mixed_probe.py --config 3
for r in 0 1; do MEMXCT_RLE=$r timeout 600 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -k regex:drift -c 1 python scripts/shard_probe.py --config 5 --which 5 --reps 1 > gpurun_out/r02h_ncu_rle$r.txt 2>&1; done
python -m pytest tests/test_gpu_peer_exchange.py tests/test_gpu_multiprocess.py tests/test_gpu_p8.py tests/test_gpu_multirank.py -q -x -p no:cacheprovider > gpurun_out/r02h_peer_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02h_peer_tests.log
python scripts/exchange_overhead.py --config 3 --rounds 3 > gpurun_out/r02h_overhead_cfg3.jsonl 2>&1
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv python scripts/prof_region.py --kind peer --what cg --iters 3 > gpurun_out/r02h_cg_launches_peer.csv 2>&1
