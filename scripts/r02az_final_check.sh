# final-code check after the 13312-entry drifting stages (r02aw): full GPU suite, smoke, all
# 8 config-5 shard ranks, the default bench line
set -x
python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r02az_gpu_tests.log 2>&1; echo "EXIT $?" >> gpurun_out/r02az_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02az_smoke.log 2>&1; echo "EXIT $?" >> gpurun_out/r02az_smoke.log
python scripts/shard_probe.py --config 5 --ranks 8 --which all --reps 10 > gpurun_out/r02az_shard_cfg5_p8.jsonl 2> gpurun_out/r02az_shard_cfg5_p8.err
python bench.py > gpurun_out/r02az_bench.json 2> gpurun_out/r02az_bench.err
