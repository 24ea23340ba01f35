#!/bin/bash
O=gpurun_out/c3chk
mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x > $O/gpu_tests.txt 2>&1
run() { name=$1; shift; timeout 300 python bench.py --no-cpu-baseline "$@" > $O/bench_$name.json 2> $O/bench_$name.err; }
run C3 --config C3 --steps 10 --warmup 3
run C3_bn --config C3 --steps 10 --warmup 3 --bn
run C3_full --config C3 --steps 10 --warmup 3 --full
run C3_full_bn --config C3 --steps 10 --warmup 3 --full --bn
run C3_bn_force_dist --config C3 --steps 10 --warmup 3 --bn --force-dist
