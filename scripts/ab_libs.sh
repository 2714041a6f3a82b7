#!/bin/bash
# A/B of library variants (libmemxct_<v>.so beside libmemxct.so; "current" = libmemxct.so as
# built), interleaved REPEATS times, each JSON line of the command tagged with the variant.
#   scripts/ab_libs.sh OUT "current u8 u16" REPEATS -- command...
set -u
out=$1; vals=$2; reps=$3; shift 4
PKG=paper_conf_sc_hidayetoglubgrg19_b200
cp $PKG/libmemxct.so /tmp/libmemxct_base.so
: > "$out"
for i in $(seq 1 $reps); do
  for v in $vals; do
    if [ "$v" = current ]; then cp /tmp/libmemxct_base.so $PKG/libmemxct.so; else cp $PKG/libmemxct_$v.so $PKG/libmemxct.so; fi
    touch $PKG/libmemxct.so
    timeout 900 "$@" 2>/dev/null | grep '^{' | sed "s/^{/{\"variant\": \"$v\", /" >> "$out"
  done
done
cp /tmp/libmemxct_base.so $PKG/libmemxct.so
touch $PKG/libmemxct.so
