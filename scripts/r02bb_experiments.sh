set -x
for i in 1 2 3; do
for b in 36864 40960; do
  python bench.py --no-cpu-baseline --no-extras --steps 10 --warmup 3 --buffer $b 2>/dev/null | grep '^{' | sed "s/^{/{\"buffer\": $b, /" >> gpurun_out/r02bb_buffer_bench.jsonl
done
done
