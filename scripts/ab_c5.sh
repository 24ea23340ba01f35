#!/bin/bash
mkdir -p gpurun_out
for L in conv5_2 conv4_2 conv3_2; do
  timeout 120 python scripts/layer_bench.py $L C5 >> gpurun_out/ab_c5.txt 2>&1
  SPLITCNN_NO_HALO=1 timeout 120 python scripts/layer_bench.py $L C5 | sed 's/^/NOHALO /' >> gpurun_out/ab_c5.txt 2>&1
  SPLITCNN_NO_CTA2=1 timeout 120 python scripts/layer_bench.py $L C5 | sed 's/^/NOCTA2 /' >> gpurun_out/ab_c5.txt 2>&1
done
