#!/bin/bash
O=gpurun_out/ab_ncu6
mkdir -p $O
B="--config C2 --steps 1 --warmup 3 --no-cpu-baseline --no-graph"
export SPLITCNN_DUAL=0 SPLITCNN_YRING=1 SPLITCNN_POOLSTG=1
for v in old; do
(cd abtree/$v && timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:conv_tc -c 200 --csv python bench.py $B) > $O/$v.csv 2>/dev/null
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:conv_tc -c 200 --csv python bench.py $B > $O/new.csv 2>/dev/null
