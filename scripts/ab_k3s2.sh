#!/bin/bash
mkdir -p gpurun_out
timeout 120 python scripts/pool_bench.py > gpurun_out/ab_k3s2.txt 2>&1
SPLITCNN_POOL_GATHER=1 timeout 120 python scripts/pool_bench.py | sed 's/^/GATHER /' >> gpurun_out/ab_k3s2.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_ops.py tests/test_gpu_resnet.py tests/test_gpu_bn.py -q >> gpurun_out/ab_k3s2.txt 2>&1
