#!/bin/bash
# Runs on the GPU box (gpurun): launch list of one warm C5 step + ncu --set full of the top kernels.
TAG=${1:-r1}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C5_${TAG}.csv \
    python bench.py --config C5 --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
# fwd conv4_2 (13th conv_tc launch of a step = index 12 in warm-up step 1), halo wgrad conv3_2, pool fwd
ncu --set full --clock-control none --import-source on -k regex:conv_tc_kernel -s 13 -c 1 -o gpurun_out/ncu_conv_fwd_${TAG} \
    python bench.py --config C5 --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:wgrad_halo_kernel -s 9 -c 1 -o gpurun_out/ncu_wgrad_${TAG} \
    python bench.py --config C5 --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:pool_fwd_kernel -s 0 -c 1 -o gpurun_out/ncu_pool_${TAG} \
    python bench.py --config C5 --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out
