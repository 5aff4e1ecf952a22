#!/bin/bash
# compute-sanitizer over tools/sanitize_step.py (run on the GPU box from the repo root); the
# one-line verdicts go to gpurun_out/sanitize_summary.txt
set -u
OUT=gpurun_out
mkdir -p $OUT
: > $OUT/sanitize_summary.txt
for tool in memcheck racecheck synccheck initcheck; do
  arg=""; [ $tool = synccheck ] && arg="--sync"
  timeout 2400 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_step.py $arg > $OUT/sanitize_$tool.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|workload done' $OUT/sanitize_$tool.log | tr '\n' ' ')" >> $OUT/sanitize_summary.txt
done
cat $OUT/sanitize_summary.txt
