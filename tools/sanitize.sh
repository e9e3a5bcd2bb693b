#!/bin/bash
# compute-sanitizer over config 1 in every mode (tools/sanitize_case.py); summary lines under
# gpurun_out/$1/.  usage (GPU box): tools/sanitize.sh sanitize
OUT=gpurun_out/${1:-sanitize}
mkdir -p $OUT
for tool in memcheck racecheck synccheck initcheck; do
  echo "== compute-sanitizer --tool $tool" > $OUT/$tool.txt
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_case.py >> $OUT/$tool.txt 2>&1
  echo "rc=$?" >> $OUT/$tool.txt
done
tail -n 4 $OUT/*.txt
