#!/bin/bash
# A/B of the conv epilogue staging ring (SPLITCNN_YRING cap, SPLITCNN_MINST stages kept) and dual MMA issue
O=gpurun_out/ab_dual5.txt
: > $O
timeout 300 python -m pytest tests/test_gpu_ops.py tests/test_gpu_stack.py tests/test_gpu_resnet.py -q -x 2>&1 | tail -2 >> $O
for L in conv1_1 conv1_2 conv2_1 conv2_2; do
  for V in "1 4 4" "0 1 4"; do set -- $V
    echo -n "DUAL=$1 YRING=$2 MINST=$3 " >> $O
    SPLITCNN_DUAL=$1 SPLITCNN_YRING=$2 SPLITCNN_MINST=$3 timeout 60 python scripts/layer_bench.py $L C5 2>&1 | tail -1 | cut -c1-200 >> $O
  done
done
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --per-layer > gpurun_out/ab_dual5_C5.json 2>/dev/null
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --config C3 > gpurun_out/ab_dual5_C3.json 2>/dev/null
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --config C2 > gpurun_out/ab_dual5_C2.json 2>/dev/null
