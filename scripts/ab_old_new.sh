#!/bin/bash
# same-box A/B: the committed tree (abtree/old, built in place) vs the working tree
O=gpurun_out/ab_on5
mkdir -p $O
timeout 600 python -m pytest tests -m gpu -q -x > $O/gpu_tests.txt 2>&1
for rep in 1 2; do
for C in "C2 20 5" "C3 10 3" "C5 10 3"; do set -- $C
  (cd abtree/old && timeout 300 python bench.py --config $1 --steps $2 --warmup $3 --no-cpu-baseline) > $O/old_$1_$rep.json 2>/dev/null
  timeout 300 python bench.py --config $1 --steps $2 --warmup $3 --no-cpu-baseline > $O/new_$1_$rep.json 2>/dev/null
done
done
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --per-layer > $O/new_C5_per_layer.json 2>/dev/null
