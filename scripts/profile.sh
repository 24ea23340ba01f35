#!/bin/bash
# Launch list + full ncu captures of the top kernels (run under gpurun, 1 GPU).
# usage: scripts/profile.sh <config> <tag>
set -x
CFG=${1:-C5}; TAG=${2:-r1}
mkdir -p gpurun_out
python bench.py --config $CFG --steps 5 --warmup 3 --no-cpu-baseline --per-layer > gpurun_out/bench_${CFG}_${TAG}.json 2> gpurun_out/bench_${CFG}_${TAG}.err
# every launch of one warm step (warmup 3 steps first), device time only
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${CFG}_${TAG}.csv \
    python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
