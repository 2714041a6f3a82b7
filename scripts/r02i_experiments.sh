set -x
scripts/ab_libs.sh gpurun_out/r02i_rle_cfg5.jsonl "current u16p u8np" 1 -- env MEMXCT_RLE=1 python scripts/shard_probe.py --config 5 --which 5 --reps 10
MEMXCT_RLE=0 python scripts/shard_probe.py --config 5 --which 5 --reps 10 | grep '^{' | sed 's/^{/{"variant": "map", /' >> gpurun_out/r02i_rle_cfg5.jsonl
scripts/ab_libs.sh gpurun_out/r02i_rle_cfg3.jsonl "current u16p" 1 -- env MEMXCT_RLE=1 python scripts/big_config.py --config 3 --iters 5
MEMXCT_RLE=0 python scripts/big_config.py --config 3 --iters 5 | grep '^{' | sed 's/^{/{"variant": "map", /' >> gpurun_out/r02i_rle_cfg3.jsonl
