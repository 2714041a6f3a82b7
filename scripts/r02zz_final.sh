# round-2 final measurement set (after the asynchronous plain / SpMM gathers) (one B200): tests, smoke, bench + launch list + ncu full set of
# the SpMV pair, reference arm, 2-rank host-transport bench, every rank of the P = 8 shards
set -x
python -m pytest tests -m gpu -q -p no:cacheprovider --durations=30 > gpurun_out/r02zz_gpu_tests.log 2>&1; echo "EXIT $?" >> gpurun_out/r02zz_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02zz_smoke.log 2>&1; echo "EXIT $?" >> gpurun_out/r02zz_smoke.log
python bench.py > gpurun_out/r02zz_bench.json 2> gpurun_out/r02zz_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02zz_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-extras > /dev/null 2>&1
ncu --profile-from-start off --set full --clock-control none --import-source on -c 2 -f -o gpurun_out/r02zz_spmv_full python scripts/prof_region.py --kind bench --what pair > /dev/null 2>&1
ncu -i gpurun_out/r02zz_spmv_full.ncu-rep --page raw --csv > gpurun_out/r02zz_spmv_full_raw.csv 2>/dev/null
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r02zz_bench_ref.json 2> gpurun_out/r02zz_bench_ref.err
timeout 900 python bench.py --gpus 2 --transport host --config 2 --steps 3 --warmup 3 > gpurun_out/r02zz_bench_host2.json 2> gpurun_out/r02zz_bench_host2.err; echo "EXIT $?" >> gpurun_out/r02zz_bench_host2.err
python scripts/shard_probe.py --config 5 --ranks 8 --which all --reps 10 > gpurun_out/r02zz_shard_cfg5_p8.jsonl 2> gpurun_out/r02zz_shard_cfg5_p8.err
python scripts/shard_probe.py --config 3 --ranks 8 --which all --reps 20 > gpurun_out/r02zz_shard_cfg3_p8.jsonl 2> gpurun_out/r02zz_shard_cfg3_p8.err
rm -f gpurun_out/r02zz_spmv_full.ncu-rep
