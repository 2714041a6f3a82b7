set -x
timeout 900 python bench.py --gpus 2 --transport host --config 2 --steps 3 --warmup 3 > gpurun_out/r02m_bench_host2.json 2> gpurun_out/r02m_bench_host2.err; echo "EXIT $?" >> gpurun_out/r02m_bench_host2.err
python -m pytest tests -m gpu -q -p no:cacheprovider --durations=30 > gpurun_out/r02m_gpu_tests.log 2>&1; echo "EXIT $?" >> gpurun_out/r02m_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02m_smoke.log 2>&1; echo "EXIT $?" >> gpurun_out/r02m_smoke.log
python bench.py > gpurun_out/r02m_bench.json 2> gpurun_out/r02m_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02m_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-extras > /dev/null 2>&1
ncu --profile-from-start off --set full --clock-control none --import-source on -c 2 -o gpurun_out/r02m_spmv_full python scripts/prof_region.py --kind bench --what pair > /dev/null 2>&1
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r02m_bench_ref.json 2> gpurun_out/r02m_bench_ref.err
