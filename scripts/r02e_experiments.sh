set -x
python -m pytest tests/test_gpu_multirank.py tests/test_gpu_p8.py tests/test_gpu_peer_exchange.py tests/test_gpu_multiprocess.py -q -x -p no:cacheprovider > gpurun_out/r02e_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02e_tests.log
python scripts/exchange_overhead.py --config 2 > gpurun_out/r02e_overhead_cfg2.jsonl 2>&1
python scripts/exchange_overhead.py --config 3 > gpurun_out/r02e_overhead_cfg3.jsonl 2>&1
scripts/ab_env.sh MEMXCT_L2HINT "0 1" 2 gpurun_out/r02e_l2hint_cfg5.jsonl -- python scripts/shard_probe.py --config 5 --which 5 --reps 20
scripts/ab_env.sh MEMXCT_L2HINT "0 1" 3 gpurun_out/r02e_l2hint_cfg3.jsonl -- python scripts/big_config.py --config 3 --iters 5
scripts/ab_libs.sh gpurun_out/r02e_mixed_u.jsonl "current u8 u16" 2 -- python scripts/mixed_probe.py --config 3
python scripts/map_runs.py --config 5 --rank 5 --parts 150 > gpurun_out/r02e_map_runs.jsonl 2>&1
python scripts/map_runs.py --config 3 --parts 300 >> gpurun_out/r02e_map_runs.jsonl 2>&1
for h in 0 1; do MEMXCT_L2HINT=$h timeout 600 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:drift -c 1 python scripts/shard_probe.py --config 5 --which 5 --reps 1 > gpurun_out/r02e_ncu_l2hint$h.txt 2>&1; done
scripts/ab_libs.sh gpurun_out/r02e_k8_swizzle.jsonl "current noswz" 2 -- python scripts/sweep_spmm.py --config 3 --rows 1024 --buffers 6144 --slices 8,4
for m in 0 1 2; do timeout 300 compute-sanitizer --tool racecheck --print-limit 3 scripts/racecheck_mbarrier_probe $m > gpurun_out/r02e_racecheck_probe_$m.txt 2>&1; done
