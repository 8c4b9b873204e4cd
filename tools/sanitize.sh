#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_cases.py
mkdir -p gpurun_out
out=gpurun_out/compute_sanitizer.txt; : > $out
for t in memcheck racecheck synccheck; do
  echo "== $t" >> $out
  timeout 1200 compute-sanitizer --tool $t --target-processes all python tools/sanitize_cases.py \
     2>&1 | grep -v "^=========     \|^========= *$" | tail -8 >> $out
  echo "exit ${PIPESTATUS[0]}" >> $out
done
cat $out
