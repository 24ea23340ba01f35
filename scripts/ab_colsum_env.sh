#!/bin/bash
# same-lib A/B: SPLITCNN_COLSUM_SMEM=1 (shared-memory colsum for every width) vs default (warp colsum + row fold)
mkdir -p gpurun_out
for r in 1 2; do
  SPLITCNN_COLSUM_SMEM=1 timeout 300 python scripts/db_cost.py 2>&1 | sed 's/^/SMEM /'
  timeout 300 python scripts/db_cost.py 2>&1 | sed 's/^/WARP /'
done
for r in 1 2 3; do
  SPLITCNN_COLSUM_SMEM=1 timeout 300 python bench.py --no-cpu-baseline 2>/dev/null | cut -c1-200 | sed 's/^/SMEM /'
  timeout 300 python bench.py --no-cpu-baseline 2>/dev/null | cut -c1-200 | sed 's/^/WARP /'
done
for c in C2 C3; do for r in 1 2; do
  SPLITCNN_COLSUM_SMEM=1 timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | cut -c1-200 | sed "s/^/SMEM $c /"
  timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | cut -c1-200 | sed "s/^/WARP $c /"
done; done
