#!/bin/bash
# GPU parity tests + per-layer timings (+ optional trace) -- one gpurun call
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/qc_tests.txt
: > gpurun_out/qc_layers.txt
for L in ${LAYERS:-conv1_1 conv1_2 conv2_1 conv2_2 conv3_1 conv3_2 conv4_2 conv5_2}; do
  timeout 120 python scripts/layer_bench.py $L C5 >> gpurun_out/qc_layers.txt 2>&1
done
if [ -n "$TRACE" ]; then bash scripts/trace_run.sh > gpurun_out/trace.txt 2>&1; fi
if [ -n "$BENCH" ]; then timeout 300 python bench.py --steps 10 --warmup 3 --per-layer > gpurun_out/qc_bench.json 2> gpurun_out/qc_bench.err; fi
