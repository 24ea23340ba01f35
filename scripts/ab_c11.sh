#!/bin/bash
mkdir -p gpurun_out
timeout 120 python scripts/layer_bench.py conv1_1 C5 > gpurun_out/ab_c11.txt 2>&1
SPLITCNN_NO_HALO=1 timeout 120 python scripts/layer_bench.py conv1_1 C5 | sed 's/^/NOHALO /' >> gpurun_out/ab_c11.txt 2>&1
SPLITCNN_NO_BRES=1 timeout 120 python scripts/layer_bench.py conv1_1 C5 | sed 's/^/NOBRES /' >> gpurun_out/ab_c11.txt 2>&1
SPLITCNN_ONE_EPI=1 timeout 120 python scripts/layer_bench.py conv1_1 C5 | sed 's/^/ONEEPI /' >> gpurun_out/ab_c11.txt 2>&1
SPLITCNN_DBG=1 timeout 120 python scripts/layer_bench.py conv1_1 C5 | sed 's/^/NOSTORE /' >> gpurun_out/ab_c11.txt 2>&1
SPLITCNN_DBG=2 timeout 120 python scripts/layer_bench.py conv1_1 C5 | sed 's/^/NOMMA /' >> gpurun_out/ab_c11.txt 2>&1
SPLITCNN_DBG=8 timeout 120 python scripts/layer_bench.py conv1_1 C5 | sed 's/^/NOTMEM2SMEM /' >> gpurun_out/ab_c11.txt 2>&1
