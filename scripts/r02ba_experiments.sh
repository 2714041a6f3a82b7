set -x
PKG=paper_conf_sc_hidayetoglubgrg19_b200
python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py tests/test_gpu_shard.py tests/test_gpu_peer_exchange.py tests/test_gpu_multiprocess.py -q -x -p no:cacheprovider > gpurun_out/r02ba_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02ba_tests.log
for i in 1 2; do
  scripts/ab_libs.sh gpurun_out/r02ba_prep_$i.jsonl "current nocache" 1 -- python scripts/prep_repeat.py --reps 2 --rds1 1
done
scripts/ab_libs.sh gpurun_out/r02ba_cfg4.jsonl "current nocache" 1 -- python scripts/shard_probe.py --config 4 --ranks 1 --which 0 --reps 3
