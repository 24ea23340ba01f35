#!/bin/bash
# C5 / C3 with and without one CUDA graph per step (same box, two reps)
O=gpurun_out/ab_graph2
mkdir -p $O
for rep in 1 2; do
for G in --no-graph --graph; do
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline $G > $O/C5${G}_$rep.json 2>$O/C5${G}_$rep.err
  timeout 300 python bench.py --config C3 --steps 10 --warmup 3 --no-cpu-baseline $G > $O/C3${G}_$rep.json 2>$O/C3${G}_$rep.err
done
done
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --per-layer > $O/C5_default_per_layer.json 2>$O/C5_pl.err
timeout 300 python bench.py --steps 20 --warmup 5 > $O/C5_default.json 2>$O/C5_default.err
timeout 300 python bench.py --config C3 --steps 10 --warmup 3 --no-cpu-baseline --bn --full > $O/C3_full_bn_default.json 2>$O/C3fb.err
