#!/bin/bash
mkdir -p gpurun_out
for r in 1 2; do
  timeout 300 python bench.py --config C2 --steps 20 --no-cpu-baseline > gpurun_out/nn_C2_new_$r.json 2>&1
  SPLITCNN_WIDE_N=1 timeout 300 python bench.py --config C2 --steps 20 --no-cpu-baseline > gpurun_out/nn_C2_old_$r.json 2>&1
done
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/nn_C5_new.json 2>&1
SPLITCNN_WIDE_N=1 timeout 300 python bench.py --no-cpu-baseline > gpurun_out/nn_C5_old.json 2>&1
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/nn_tests.txt 2>&1
