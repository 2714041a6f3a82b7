set -x
PKG=paper_conf_sc_hidayetoglubgrg19_b200
for spec in "8 6144" "4 9216" "2 12288"; do
  set -- $spec
  scripts/ab_libs.sh gpurun_out/r02af_spmm_k$1.jsonl "current sa4 sa8" 2 -- python scripts/sweep_spmm.py --config 3 --rows 1024 --buffers $2 --slices $1
done
cp $PKG/libmemxct.so /tmp/base.so
cp $PKG/libmemxct_sa8.so $PKG/libmemxct.so
python -m pytest tests/test_gpu_parity.py tests/test_gpu_ray_block.py tests/test_gpu_multirank.py -q -x -p no:cacheprovider -k "batch or slice or spmm or multi" > gpurun_out/r02af_tests_sa8.log 2>&1; echo EXIT $? >> gpurun_out/r02af_tests_sa8.log
cp /tmp/base.so $PKG/libmemxct.so
