#!/bin/bash
timeout 300 python -m pytest tests/test_gpu_ops.py tests/test_gpu_stack.py tests/test_gpu_resnet.py -q -x 2>&1 | tail -2 > gpurun_out/ab_c2_tests.txt
for V in "1 4" "0 1"; do set -- $V
SPLITCNN_DUAL=$1 SPLITCNN_YRING=$2 timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --config C2 > gpurun_out/ab_c2b_$1_$2.json 2>/dev/null
SPLITCNN_DUAL=$1 SPLITCNN_YRING=$2 timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --config C3 > gpurun_out/ab_c3b_$1_$2.json 2>/dev/null
SPLITCNN_DUAL=$1 SPLITCNN_YRING=$2 timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --per-layer > gpurun_out/ab_c5b_$1_$2.json 2>/dev/null
done
