#!/bin/bash
# Experiment build of the library with extra nvcc flags beside the real one:
#   scripts/build_variant.sh NAME "-DFOO=1 ..."   -> paper_conf_sc_hidayetoglubgrg19_b200/libmemxct_NAME.so
MEMXCT_VARIANT=$1 MEMXCT_VARIANT_FLAGS="$2" python -m paper_conf_sc_hidayetoglubgrg19_b200.build_ext --force
