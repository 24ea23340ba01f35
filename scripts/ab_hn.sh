#!/bin/bash
O=gpurun_out/ab_hn22
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_resnet.py tests/test_gpu_bn.py tests/test_gpu_fullsize.py -q -x > $O/tests.txt 2>&1
for SP in 16 64; do
timeout 300 python bench.py --config C3 --steps 10 --warmup 3 --no-cpu-baseline --stem-pad $SP --per-layer > $O/C3_pad$SP.json 2>/dev/null
done
timeout 300 python bench.py --config C1 --steps 20 --warmup 5 --no-cpu-baseline --dtype bf16 > $O/C1_bf16.json 2>/dev/null
