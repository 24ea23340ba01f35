#!/bin/bash
mkdir -p gpurun_out
for L in conv1_1 conv1_2 conv4_2; do
  timeout 120 python scripts/layer_bench.py $L C5 >> gpurun_out/ab_pspin.txt 2>&1
  SPLITCNN_DBG=1024 timeout 120 python scripts/layer_bench.py $L C5 | sed 's/^/PSPIN /' >> gpurun_out/ab_pspin.txt 2>&1
  SPLITCNN_DBG=4 timeout 120 python scripts/layer_bench.py $L C5 | sed 's/^/NOLOAD /' >> gpurun_out/ab_pspin.txt 2>&1
  SPLITCNN_DBG=6 timeout 120 python scripts/layer_bench.py $L C5 | sed 's/^/NOLOAD_NOMMA /' >> gpurun_out/ab_pspin.txt 2>&1
done
