#!/bin/bash
mkdir -p gpurun_out
timeout 200 python scripts/ab_pool.py conv1_2,conv2_2 > gpurun_out/ab_bh.txt 2>&1
for BH in 2 4 8 16; do
  SPLITCNN_HALO_BH=$BH timeout 200 python scripts/ab_pool.py conv1_2,conv2_2 | sed "s/^/BH$BH /" >> gpurun_out/ab_bh.txt 2>&1
done
for BH in 1 2 4 16; do
  SPLITCNN_HALO_BH=$BH timeout 120 python scripts/layer_bench.py conv1_2 C5 | sed "s/^/BH$BH /" >> gpurun_out/ab_bh.txt 2>&1
done
