set -x
PKG=paper_conf_sc_hidayetoglubgrg19_b200
scripts/ab_libs.sh gpurun_out/r02ac_async_cfg3.jsonl "current pa16 pa32" 3 -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
scripts/ab_libs.sh gpurun_out/r02ac_async_mixed.jsonl "current pa16 pa32" 2 -- python scripts/mixed_probe.py --config 3
scripts/ab_libs.sh gpurun_out/r02ac_async_cfg4.jsonl "current pa16 pa32" 1 -- python scripts/shard_probe.py --config 4 --ranks 1 --which 0 --reps 5
cp $PKG/libmemxct.so /tmp/base.so
cp $PKG/libmemxct_pa32.so $PKG/libmemxct.so
python -m pytest tests/test_gpu_parity.py tests/test_gpu_drift.py -q -x -p no:cacheprovider > gpurun_out/r02ac_tests_pa32.log 2>&1; echo EXIT $? >> gpurun_out/r02ac_tests_pa32.log
cp /tmp/base.so $PKG/libmemxct.so
