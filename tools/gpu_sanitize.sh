#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_driver.py (one GPU)
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for part in eval exact qos ga; do
  for tool in memcheck racecheck synccheck; do
    timeout 900 $CS --tool $tool --error-exitcode 9 python tools/sanitize_driver.py $part > gpurun_out/sanitize_${tool}_${part}.log 2>&1
    echo "$tool $part rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' gpurun_out/sanitize_${tool}_${part}.log | tail -1)"
  done
done
