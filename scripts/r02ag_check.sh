set -x
python -m pytest tests/test_gpu_parity.py tests/test_gpu_ray_block.py tests/test_gpu_multirank.py -q -x -p no:cacheprovider -k "batch or slice or spmm or multi" > gpurun_out/r02ag_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02ag_tests.log
for spec in "8 6144" "4 9216" "2 12288"; do
  set -- $spec
  python scripts/sweep_spmm.py --config 3 --rows 1024 --buffers $2 --slices $1 >> gpurun_out/r02ag_spmm.jsonl
done
python bench.py --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/r02ag_bench.json 2> gpurun_out/r02ag_bench.err
