#!/bin/bash
# conv fwd timing of one layer under the SPLITCNN_DBG isolation flags (1 no store, 2 no MMA, 4 no loads, 8 no TMEM->smem)
L=${1:-conv1_1}
for d in 0 1 2 4 8 5 13 15; do SPLITCNN_DBG=$d timeout 120 python scripts/layer_bench.py $L C5 2>&1 | tail -1; done
