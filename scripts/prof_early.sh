#!/bin/bash
# ncu --set full captures of the early-layer kernels (conv1_1 fwd/wgrad, conv1_2 fwd/wgrad, pool1 fwd)
mkdir -p gpurun_out
NCU="ncu --set full --clock-control none --import-source on -c 1"
timeout 300 $NCU -k regex:conv_tc_kernel -s 3 -o gpurun_out/ncu_c11_fwd python scripts/layer_bench.py conv1_1 > /dev/null 2>&1
timeout 300 $NCU -k regex:wgrad -s 3 -o gpurun_out/ncu_c11_wg python scripts/layer_bench.py conv1_1 > /dev/null 2>&1
timeout 300 $NCU -k regex:conv_tc_kernel -s 3 -o gpurun_out/ncu_c12_fwd python scripts/layer_bench.py conv1_2 > /dev/null 2>&1
timeout 300 $NCU -k regex:wgrad -s 3 -o gpurun_out/ncu_c12_wg python scripts/layer_bench.py conv1_2 > /dev/null 2>&1
timeout 300 $NCU -k regex:conv_tc_kernel -s 3 -o gpurun_out/ncu_c21_fwd python scripts/layer_bench.py conv2_1 > /dev/null 2>&1
timeout 300 $NCU -k regex:pool_fwd -s 0 -o gpurun_out/ncu_pool1 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out/*.ncu-rep
