#!/bin/bash
for L in ${TLAYERS:-conv1_1 conv1_2 conv4_2}; do
SPLITCNN_TRACE=1 timeout 120 python - $L <<'PY' 2>&1 | grep -v "trace CTA (block" | head -${TLINES:-40}
import os, sys, torch
sys.argv = ["x", sys.argv[1]]
sys.path.insert(0, os.getcwd())
exec(open("scripts/layer_bench.py").read().split("r = {}")[0])
for _ in range(3): sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU)
PY
done
