#!/bin/bash
mkdir -p gpurun_out
for D in 0 15 31 22; do
  SPLITCNN_DBG=$D timeout 120 python scripts/layer_bench.py conv1_1 C5 | sed "s/^/DBG$D /" >> gpurun_out/ab_c11b.txt 2>&1
done
