set -x
for i in 1 2; do
for b in 16384 14336 12288; do
  MEMXCT_DRIFT_B=$b python scripts/shard_probe.py --config 5 --which 5 --reps 10 2>/dev/null | grep '^{' | sed "s/^{/{\"MEMXCT_DRIFT_B\": $b, /" >> gpurun_out/r02av_driftb_cfg5.jsonl
done
done
for b in 12288 10240 8192; do
  MEMXCT_DRIFT=1 MEMXCT_DRIFT_B=$b python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20 2>/dev/null | grep '^{' | sed "s/^{/{\"MEMXCT_DRIFT_B\": $b, /" >> gpurun_out/r02av_driftb_cfg3.jsonl
done
python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20 2>/dev/null | grep '^{' | sed "s/^{/{\"MEMXCT_DRIFT_B\": 0, /" >> gpurun_out/r02av_driftb_cfg3.jsonl
