set -x
ncu --set full --clock-control none --import-source on -k regex:spmm_f32_kernel -c 2 -f -o gpurun_out/r02aa_spmm8 python scripts/prof_spmm.py 8 > gpurun_out/r02aa_ncu.log 2>&1
echo EXIT $?
