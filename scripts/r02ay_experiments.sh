set -x
for i in 1 2; do
python scripts/sweep_spmm.py --config 3 --rows 1024 --buffers 6144,5120,4608 --slices 8 >> gpurun_out/r02ay_spmm8_b.jsonl
done
