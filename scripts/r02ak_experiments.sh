set -x
PKG=paper_conf_sc_hidayetoglubgrg19_b200
scripts/ab_libs.sh gpurun_out/r02ak_head_cfg5.jsonl "current head" 3 -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
cp $PKG/libmemxct.so /tmp/base.so
cp $PKG/libmemxct_head.so $PKG/libmemxct.so
python -m pytest tests/test_gpu_drift.py tests/test_gpu_ray_block.py -q -x -p no:cacheprovider > gpurun_out/r02ak_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02ak_tests.log
cp /tmp/base.so $PKG/libmemxct.so
