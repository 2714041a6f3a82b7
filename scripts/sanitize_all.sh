#!/bin/bash
# compute-sanitizer over every case of scripts/sanitize_cases.py; one summary line per (tool, case)
# into $1 (default gpurun_out/sanitize.log).  Each run is bounded by `timeout`.
out=${1:-gpurun_out/sanitize.log}
: > "$out"
for tool in memcheck racecheck synccheck initcheck; do
  for case in fp32 drift mixed spmm blocked sirt collective peer; do
    log=$(mktemp)
    timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
      python scripts/sanitize_cases.py $case > "$log" 2>&1
    rc=$?
    summary=$(grep -E "ERROR SUMMARY|RACECHECK SUMMARY|hazard|CASE OK" "$log" | tr '\n' ' ' | cut -c1-300)
    echo "$tool $case rc=$rc $summary" >> "$out"
    if [ $rc -ne 0 ]; then echo "---- $tool $case tail" >> "$out"; tail -40 "$log" >> "$out"; fi
    rm -f "$log"
  done
done
