#!/bin/bash
mkdir -p gpurun_out
bash scripts/ab_lib.sh scripts/pool_bench.py > gpurun_out/ab_pool2.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_ops.py tests/test_gpu_stack.py tests/test_gpu_resnet.py -q -x >> gpurun_out/ab_pool2.txt 2>&1
