#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck of scripts/sanitize_c1.py (one GPU, gpurun)
OUT=${1:-gpurun_out/sanitize}
mkdir -p $OUT
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python scripts/sanitize_c1.py > $OUT/$tool.log 2>&1
  echo "$tool rc=$?" >> $OUT/summary.txt
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|SANITIZE_DRIVER_OK" $OUT/$tool.log >> $OUT/summary.txt
done
cat $OUT/summary.txt
