#!/bin/bash
# block-1 ncu --set full captures + launch list with DRAM bytes for the C5 step (roofline traffic)
TAG=${1:-r1c}
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_dram_C5_${TAG}.csv python bench.py --config C5 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ld_${TAG}.log 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:'conv_tc|wgrad_' -s 3 -c 3 \
    -o gpurun_out/ncu_conv1_2_${TAG} python scripts/prof_layer.py conv1_2 C5 db > gpurun_out/ncu_conv1_2_${TAG}.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:'conv_tc|wgrad_' -s 2 -c 2 \
    -o gpurun_out/ncu_conv1_1_${TAG} python scripts/prof_layer.py conv1_1 C5 db > gpurun_out/ncu_conv1_1_${TAG}.log 2>&1
ls -la gpurun_out
