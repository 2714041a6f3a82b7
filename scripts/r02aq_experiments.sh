set -x
scripts/ab_env.sh MEMXCT_L2HINT "0 1" 3 gpurun_out/r02aq_l2hint_cfg5.jsonl -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
MEMXCT_L2HINT=1 timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:spmv_f32_drift -c 1 --csv python scripts/shard_probe.py --config 5 --which 5 --reps 1 > gpurun_out/r02aq_ncu_l2hint1.csv 2>&1
MEMXCT_L2HINT=0 timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:spmv_f32_drift -c 1 --csv python scripts/shard_probe.py --config 5 --which 5 --reps 1 > gpurun_out/r02aq_ncu_l2hint0.csv 2>&1
