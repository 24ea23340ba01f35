#!/bin/bash
mkdir -p gpurun_out
git_rev=$(cat .ab_rev 2>/dev/null)
timeout 120 python scripts/layer_bench.py conv1_2 C5 > gpurun_out/ab_halo64.txt 2>&1
timeout 120 python scripts/layer_bench.py conv1_2 C4 >> gpurun_out/ab_halo64.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_ops.py tests/test_gpu_resnet.py -q -x >> gpurun_out/ab_halo64.txt 2>&1
