set -x
python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "canonical" > gpurun_out/r02y_tests.log 2>&1; echo EXIT $? >> gpurun_out/r02y_tests.log
python scripts/prep_repeat.py --reps 3 --rds1 1 > gpurun_out/r02y_prep_repeat.jsonl 2> gpurun_out/r02y_prep_repeat.err
CUDA_MODULE_LOADING=EAGER python scripts/prep_repeat.py --reps 2 --rds1 0 > gpurun_out/r02y_prep_repeat_eager.jsonl 2>> gpurun_out/r02y_prep_repeat.err
