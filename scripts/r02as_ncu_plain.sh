set -x
timeout 1200 ncu --profile-from-start off --set full --clock-control none --import-source on -c 1 -f -o gpurun_out/r02as_cfg3_fwd python scripts/prof_region.py --kind bench --what fwd > gpurun_out/r02as_ncu.log 2>&1
echo EXIT $?
