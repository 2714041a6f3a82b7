set -x
python -m pytest tests/test_gpu_multirank.py tests/test_gpu_p8.py tests/test_gpu_peer_exchange.py tests/test_gpu_multiprocess.py tests/test_gpu_drift.py -q -x -p no:cacheprovider > gpurun_out/r02g_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02g_tests.log
python scripts/exchange_overhead.py --config 2 > gpurun_out/r02g_overhead_cfg2.jsonl 2>&1
python scripts/exchange_overhead.py --config 3 > gpurun_out/r02g_overhead_cfg3.jsonl 2>&1
for k in collective peer; do ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv python scripts/prof_region.py --kind $k --what cg --iters 3 > gpurun_out/r02g_cg_launches_$k.csv 2>&1; done
python scripts/mixed_probe.py --config 3 --buffers 36864,45056,49152,28672 > gpurun_out/r02g_mixed_buffers.jsonl 2>&1
python scripts/mixed_probe.py --config 3 --canonical 0 >> gpurun_out/r02g_mixed_buffers.jsonl 2>&1
