#!/bin/bash
# A/B: staged TMA-store epilogue vs direct register->global stores (SPLITCNN_DSTORE=1)
mkdir -p gpurun_out
for L in conv1_1 conv1_2 conv2_1 conv2_2 conv3_2 conv4_2 conv5_2; do
  timeout 120 python scripts/layer_bench.py $L C5 >> gpurun_out/ab_dstore.txt 2>&1
  SPLITCNN_DSTORE=1 timeout 120 python scripts/layer_bench.py $L C5 | sed 's/^/DSTORE /' >> gpurun_out/ab_dstore.txt 2>&1
done
SPLITCNN_DSTORE=1 timeout 600 python -m pytest tests/test_gpu_ops.py -q -k conv_parity > gpurun_out/ab_dstore_tests.txt 2>&1
