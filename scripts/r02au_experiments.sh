set -x
scripts/ab_env.sh MEMXCT_DRIFT "0 1" 2 gpurun_out/r02au_drift_cfg3.jsonl -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
for b in 12288 18432; do
  MEMXCT_DRIFT=1 MEMXCT_DRIFT_B=$b python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20 2>/dev/null | grep '^{' | sed "s/^{/{\"MEMXCT_DRIFT_B\": $b, /" >> gpurun_out/r02au_drift_cfg3.jsonl
done
