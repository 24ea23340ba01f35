#!/bin/bash
# ncu --set full of representative conv kernels (conv4_2 at peak, conv1_2 64-channel) -- for profiles/
TAG=${1:-r1f}
mkdir -p gpurun_out
timeout 400 ncu --set full --clock-control none --import-source on -k regex:'conv_tc|wgrad_' -s 3 -c 3 \
    -o gpurun_out/ncu_conv4_2_${TAG} python scripts/prof_layer.py conv4_2 C5 db > gpurun_out/ncu_conv4_2_${TAG}.log 2>&1
ls -la gpurun_out | grep ncu_conv4
