set -x
for i in 1 2; do
for v in "0 0" "1 0" "1 32" "1 64"; do
  set -- $v
  MEMXCT_L2HINT=$1 MEMXCT_L2_SETASIDE=$2 python scripts/shard_probe.py --config 5 --which 5 --reps 10 2>>gpurun_out/r02ar.err | grep '^{' | sed "s/^{/{\"l2hint\": $1, \"setaside_mb\": $2, /" >> gpurun_out/r02ar_setaside_cfg5.jsonl
done
done
MEMXCT_L2HINT=1 MEMXCT_L2_SETASIDE=64 timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:spmv_f32_drift -c 1 --csv python scripts/shard_probe.py --config 5 --which 5 --reps 1 > gpurun_out/r02ar_ncu_sa64.csv 2>&1
