set -x
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,launch__shared_mem_config_size,launch__shared_mem_per_block_dynamic,lts__t_sector_hit_rate.pct,smsp__inst_executed.sum --clock-control none -k regex:spmv_f32_drift -c 1 --csv python scripts/shard_probe.py --config 5 --which 5 --reps 1 > gpurun_out/r02bd_drift13312.csv 2>&1
