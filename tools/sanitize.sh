#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_case.py
# (STM path + cfg1-shaped split storm); summaries into gpurun_out/sanitize_$TAG/.
TAG=${1:-x}
OUT=gpurun_out/sanitize_$TAG
mkdir -p $OUT
export EIRENE_NO_GRAPHS=${EIRENE_NO_GRAPHS:-}
for tool in memcheck racecheck synccheck; do
  for c in stm cfg1; do
    timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 20 \
      python tools/sanitize_case.py $c > $OUT/${tool}_$c.log 2>&1
    echo "$tool $c rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|case ok' $OUT/${tool}_$c.log | tr '\n' ' ')" >> $OUT/summary.txt
  done
done
cat $OUT/summary.txt
