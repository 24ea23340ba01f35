#!/bin/bash
O=gpurun_out/ab_c5env
mkdir -p $O
for rep in 1 2; do
for V in "1 4" "0 1" "1 1" "0 4"; do set -- $V
SPLITCNN_DUAL=$1 SPLITCNN_YRING=$2 timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --per-layer > $O/d$1_y$2_$rep.json 2>/dev/null
done
done
