set -x
python -m pytest tests -m gpu -q -p no:cacheprovider --durations=20 > gpurun_out/r02t_gpu_tests.log 2>&1; echo "EXIT $?" >> gpurun_out/r02t_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02t_smoke.log 2>&1; echo "EXIT $?" >> gpurun_out/r02t_smoke.log
python bench.py > gpurun_out/r02t_bench.json 2> gpurun_out/r02t_bench.err
