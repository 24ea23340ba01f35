#!/bin/bash
for L in conv1_1 conv1_2 conv2_1 conv2_2 conv4_2; do
for d in 0 64 79; do SPLITCNN_DBG=$d timeout 120 python scripts/layer_bench.py $L C5 2>&1 | tail -1; done
done
