set -x
python -m pytest tests/test_gpu_drift.py tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "drift or spmm or batched or fp32_spmv or mixed_spmv" > gpurun_out/r02f_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02f_tests.log
for m in 0 1 2; do scripts/racecheck_mbarrier_probe $m 1 >> gpurun_out/r02f_probe_jitter.txt 2>&1; done
for k in plain collective peer; do ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv python scripts/prof_region.py --kind $k --what cg --iters 3 > gpurun_out/r02f_cg_launches_$k.csv 2>&1; done
ncu --profile-from-start off --set full --clock-control none --import-source on -c 1 -o gpurun_out/r02f_mixed_fwd python scripts/prof_region.py --kind mixed --what fwd > /dev/null 2>&1
ncu --profile-from-start off --set full --clock-control none --import-source on -c 1 -o gpurun_out/r02f_fp32_fwd python scripts/prof_region.py --kind plain --what fwd > /dev/null 2>&1
python bench.py > gpurun_out/r02f_bench.json 2> gpurun_out/r02f_bench.err
