#!/bin/bash
# A/B of an environment knob on a command, interleaved (ABAB...) on one box.
#   scripts/ab_env.sh VAR "v1 v2" REPEATS OUT -- command...
var=$1; vals=$2; reps=$3; out=$4; shift 5
: > "$out"
for i in $(seq 1 $reps); do
  for v in $vals; do
    echo "# $var=$v run $i" >> "$out"
    env $var=$v "$@" 2>/dev/null | grep '^{' | sed "s/^{/{\"$var\": \"$v\", /" >> "$out"
  done
done
