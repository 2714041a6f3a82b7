set -x
PKG=paper_conf_sc_hidayetoglubgrg19_b200
scripts/ab_libs.sh gpurun_out/r02o_tail_cfg5.jsonl "current tail2 tail4" 2 -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
scripts/ab_libs.sh gpurun_out/r02o_tail_cfg3.jsonl "current tail2 tail4" 2 -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
cp $PKG/libmemxct.so /tmp/base.so
for v in tail2 tail4; do
  cp $PKG/libmemxct_$v.so $PKG/libmemxct.so
  python -m pytest tests/test_gpu_drift.py tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/r02o_tests_$v.log 2>&1; echo EXIT $? >> gpurun_out/r02o_tests_$v.log
done
cp /tmp/base.so $PKG/libmemxct.so
