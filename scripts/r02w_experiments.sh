set -x
python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "canonical or mixed" > gpurun_out/r02w_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02w_tests.log
for i in 1 2; do
  scripts/ab_libs.sh gpurun_out/r02w_cd_$i.jsonl "current old" 1 -- python scripts/mixed_probe.py --config 3
  MEMXCT_CANONICAL_DOT_AFTER=1 python scripts/mixed_probe.py --config 3 2>/dev/null | grep '^{' | sed 's/^{/{"variant": "after", /' >> gpurun_out/r02w_cd_$i.jsonl
done
