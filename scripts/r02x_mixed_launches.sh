set -x
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02x_mixed_cg_launches.csv python scripts/prof_region.py --kind mixed --what cg --iters 3 > /dev/null 2>&1
MEMXCT_CANONICAL_DOT_AFTER=1 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02x_mixed_cg_launches_after.csv python scripts/prof_region.py --kind mixed --what cg --iters 3 > /dev/null 2>&1
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02x_plain_cg_launches.csv python scripts/prof_region.py --kind plain --what cg --iters 3 > /dev/null 2>&1
