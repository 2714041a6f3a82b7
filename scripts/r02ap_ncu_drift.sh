set -x
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:spmv_f32_drift -c 1 -f -o gpurun_out/r02ap_cfg5_drift python scripts/shard_probe.py --config 5 --which 5 --reps 1 > gpurun_out/r02ap_ncu.log 2>&1
echo EXIT $?
