set -x
scripts/ab_libs.sh gpurun_out/r02v_mbar_hint_cfg5.jsonl "current hint20000 hint1000000" 2 -- python scripts/shard_probe.py --config 5 --which 5 --reps 10
