set -x
for i in 1 2 3; do
  MEMXCT_ALLOC_TRACE=1 python scripts/prep_repeat.py --reps 3 --rds1 0 --like-bench 1 > gpurun_out/r02ai_prep_$i.jsonl 2> gpurun_out/r02ai_prep_$i.err
done
