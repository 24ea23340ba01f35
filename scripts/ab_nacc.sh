#!/bin/bash
mkdir -p gpurun_out
for L in conv1_1 conv1_2 conv2_1 conv2_2 conv3_1; do
  timeout 120 python scripts/layer_bench.py $L C5 >> gpurun_out/ab_nacc.txt 2>&1
  SPLITCNN_NACC2=1 timeout 120 python scripts/layer_bench.py $L C5 | sed 's/^/NACC2 /' >> gpurun_out/ab_nacc.txt 2>&1
done
timeout 200 python scripts/ab_pool.py conv1_2,conv2_2 >> gpurun_out/ab_nacc.txt 2>&1
SPLITCNN_NACC2=1 timeout 200 python scripts/ab_pool.py conv1_2,conv2_2 | sed 's/^/NACC2 /' >> gpurun_out/ab_nacc.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x >> gpurun_out/ab_nacc.txt 2>&1
