set -x
PKG=paper_conf_sc_hidayetoglubgrg19_b200
scripts/ab_libs.sh gpurun_out/r02am_rem2_bench.jsonl "current rem2" 3 -- python bench.py --no-cpu-baseline --no-extras --steps 10 --warmup 3
scripts/ab_libs.sh gpurun_out/r02am_rem2_cfg3.jsonl "current rem2" 2 -- python scripts/shard_probe.py --config 3 --ranks 1 --which 0 --reps 20
scripts/ab_libs.sh gpurun_out/r02am_rem2_cfg5.jsonl "current rem2" 2 -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
cp $PKG/libmemxct.so /tmp/base.so
cp $PKG/libmemxct_rem2.so $PKG/libmemxct.so
python -m pytest tests/test_gpu_drift.py tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/r02am_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02am_tests.log
cp /tmp/base.so $PKG/libmemxct.so
