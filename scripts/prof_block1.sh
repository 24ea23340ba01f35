#!/bin/bash
# ncu --set full of the block-1 kernels (conv1_1 fwd + narrow wgrad, conv1_2 fwd/dgrad/halo wgrad) + pool fwd
TAG=${1:-r1}
mkdir -p gpurun_out
for L in conv1_2 conv2_1 conv4_2; do timeout 120 python scripts/layer_bench.py $L C5 >> gpurun_out/lb_${TAG}.txt 2>&1; done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:'conv_tc|wgrad_' -s 2 -c 2 \
    -o gpurun_out/ncu_conv1_1_${TAG} python scripts/prof_layer.py conv1_1 C5 db > gpurun_out/ncu_conv1_1_${TAG}.log 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:'conv_tc|wgrad_' -s 3 -c 3 \
    -o gpurun_out/ncu_conv1_2_${TAG} python scripts/prof_layer.py conv1_2 C5 db > gpurun_out/ncu_conv1_2_${TAG}.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:'conv_tc|wgrad_' -s 3 -c 3 \
    -o gpurun_out/ncu_conv4_2_${TAG} python scripts/prof_layer.py conv4_2 C5 db > gpurun_out/ncu_conv4_2_${TAG}.log 2>&1
ls -la gpurun_out
