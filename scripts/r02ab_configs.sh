set -x
python bench.py --config 4 --steps 3 --warmup 3 --no-cpu-baseline --no-extras > gpurun_out/r02ab_bench_cfg4.json 2> gpurun_out/r02ab_bench_cfg4.err
python bench.py --config 2 --steps 10 --warmup 3 --no-extras > gpurun_out/r02ab_bench_cfg2.json 2> gpurun_out/r02ab_bench_cfg2.err
python bench.py --config 1 --steps 10 --warmup 3 --no-extras > gpurun_out/r02ab_bench_cfg1.json 2> gpurun_out/r02ab_bench_cfg1.err
