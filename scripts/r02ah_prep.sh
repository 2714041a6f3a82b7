set -x
python scripts/prep_repeat.py --reps 2 --rds1 0 --like-bench 1 > gpurun_out/r02ah_prep_lb1.jsonl 2> gpurun_out/r02ah.err
python scripts/prep_repeat.py --reps 2 --rds1 0 --like-bench 2 > gpurun_out/r02ah_prep_lb2.jsonl 2>> gpurun_out/r02ah.err
python scripts/prep_repeat.py --reps 2 --rds1 0 --like-bench 0 > gpurun_out/r02ah_prep_lb0.jsonl 2>> gpurun_out/r02ah.err
