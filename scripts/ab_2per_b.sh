#!/bin/bash
mkdir -p gpurun_out
for r in 1 2; do
timeout 120 python scripts/layer_bench.py conv1_1 C5 >> gpurun_out/ab_2per_b.txt 2>&1
SPLITCNN_TWO_PER_SM=1 timeout 120 python scripts/layer_bench.py conv1_1 C5 | sed 's/^/TWO /' >> gpurun_out/ab_2per_b.txt 2>&1
done
SPLITCNN_TWO_PER_SM=1 timeout 600 python -m pytest tests/test_gpu_ops.py -q -k conv_parity >> gpurun_out/ab_2per_b.txt 2>&1
