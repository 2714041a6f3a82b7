#!/bin/bash
# A/B of SpMM library variants (built beside libmemxct.so): swaps the library file and sweeps.
# usage: scripts/ab_spmm_libs.sh TAG variant1 variant2 ...   (variant "current" = libmemxct.so as built,
# any other name v = libmemxct_v.so)
set -u
TAG=$1; shift
PKG=paper_conf_sc_hidayetoglubgrg19_b200
cp $PKG/libmemxct.so /tmp/libmemxct_base.so
for v in "$@"; do
  if [ "$v" = current ]; then cp /tmp/libmemxct_base.so $PKG/libmemxct.so; else cp $PKG/libmemxct_$v.so $PKG/libmemxct.so; fi
  touch $PKG/libmemxct.so
  timeout 600 python scripts/sweep_spmm.py --config 3 --rows 1024 --buffers 6144,9216,12288 --slices 2,4,8 \
    | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/${TAG}.jsonl
done
cp /tmp/libmemxct_base.so $PKG/libmemxct.so
