# compute-sanitizer over the kernels changed in r02r-r02w: the drifting-stage kernel with the
# asynchronous (cp.async + mbarrier) gather (plain map and RLE records), the projection-block
# plan that selects it, and the fp64 kernel with the staged canonical-dot sum
out=gpurun_out/r02y_sanitize.log
: > "$out"
for tool in memcheck racecheck synccheck initcheck; do
  for case in drift blocked mixed; do
    for rle in 0 1; do
      log=$(mktemp)
      MEMXCT_RLE=$rle timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
        python scripts/sanitize_cases.py $case > "$log" 2>&1
      rc=$?
      summary=$(grep -E "ERROR SUMMARY|RACECHECK SUMMARY|hazard|CASE OK" "$log" | tr '\n' ' ' | cut -c1-300)
      echo "$tool $case rle=$rle rc=$rc $summary" >> "$out"
      if [ $rc -ne 0 ]; then echo "---- $tool $case tail" >> "$out"; tail -40 "$log" >> "$out"; fi
      rm -f "$log"
    done
  done
done
