#!/bin/bash
mkdir -p gpurun_out
for L in conv1_1 conv1_2 conv2_1 conv4_2; do
  timeout 120 python scripts/layer_bench.py $L C5 >> gpurun_out/ab_espin.txt 2>&1
  SPLITCNN_DBG=4096 timeout 120 python scripts/layer_bench.py $L C5 | sed 's/^/ESPIN /' >> gpurun_out/ab_espin.txt 2>&1
  SPLITCNN_DBG=5120 timeout 120 python scripts/layer_bench.py $L C5 | sed 's/^/ESPIN+PSPIN /' >> gpurun_out/ab_espin.txt 2>&1
done
