#!/bin/bash
O=gpurun_out/ab_mreg
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_resnet.py tests/test_gpu_stack.py tests/test_gpu_fullsize.py -q -x > $O/tests.txt 2>&1
for M in 0 1; do
  if [ $M = 1 ]; then export SPLITCNN_NO_MREG=1; fi
  timeout 120 python scripts/prof_conv12.py 10 > $O/prof12_$M.txt 2>&1
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --per-layer > $O/C5_$M.json 2>/dev/null
  timeout 300 python bench.py --config C3 --steps 10 --warmup 3 --no-cpu-baseline --per-layer > $O/C3_$M.json 2>/dev/null
done
