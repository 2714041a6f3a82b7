set -x
for i in 1 2 3; do
for b in 16384 13312 12288; do
  MEMXCT_DRIFT_B=$b python scripts/shard_probe.py --config 5 --which 5 --reps 10 2>/dev/null | grep '^{' | sed "s/^{/{\"MEMXCT_DRIFT_B\": $b, /" >> gpurun_out/r02aw_driftb_cfg5.jsonl
done
done
for b in 16384 13312; do
  MEMXCT_DRIFT_B=$b python scripts/shard_probe.py --config 5 --which 0 --reps 10 2>/dev/null | grep '^{' | sed "s/^{/{\"MEMXCT_DRIFT_B\": $b, /" >> gpurun_out/r02aw_driftb_cfg5.jsonl
done
