#!/bin/bash
mkdir -p gpurun_out
timeout 120 python scripts/layer_bench.py conv1_1 C5 > gpurun_out/ab_narrow.txt 2>&1
timeout 120 python scripts/layer_bench.py conv1_1 C4 >> gpurun_out/ab_narrow.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_ops.py -q -k "conv_parity" >> gpurun_out/ab_narrow.txt 2>&1
