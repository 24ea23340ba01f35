#!/bin/bash
mkdir -p gpurun_out
timeout 120 python scripts/layer_bench.py conv1_1 C5 > gpurun_out/ab_2per.txt 2>&1
SPLITCNN_NO_2PER=1 timeout 120 python scripts/layer_bench.py conv1_1 C5 | sed 's/^/NO2PER /' >> gpurun_out/ab_2per.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_ops.py tests/test_gpu_stack.py -q -x >> gpurun_out/ab_2per.txt 2>&1
timeout 400 python bench.py --no-cpu-baseline > gpurun_out/bench_C5_2per.json 2>&1
