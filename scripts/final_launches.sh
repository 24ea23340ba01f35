#!/bin/bash
# ncu launch list (time + DRAM bytes per launch) of a C5 bench run: 3 warm-up steps + 1 step, serialised
TAG=${1:-r2h}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_C5_${TAG}.csv python bench.py --config C5 --steps 1 --warmup 3 --no-cpu-baseline \
    > gpurun_out/launches_C5_${TAG}.log 2>&1
ls -la gpurun_out/launches_C5_${TAG}.csv
