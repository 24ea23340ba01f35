#!/bin/bash
# compute-sanitizer on the smoke test and a small C2 + ResNet step (SURVEY §4 "Sanitizers")
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck synccheck racecheck; do
  timeout 900 $CS --tool $tool --print-limit 20 python scripts/sanitize_step.py > gpurun_out/san_${tool}.txt 2>&1
  echo "exit $?" >> gpurun_out/san_${tool}.txt
done
