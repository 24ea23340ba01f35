#!/bin/bash
# per-tile trace of the fused conv+pool forward of one C5 layer (CTA 0)
L=${1:-conv1_2}
SPLITCNN_TRACE=1 timeout 120 python - $L <<'PY' 2>&1 | grep -v "trace CTA (block" | head -${TLINES:-20}
import os, sys, torch
sys.argv = ["x", sys.argv[1]]
sys.path.insert(0, os.getcwd())
src = open("scripts/ab_pool.py").read().split("    tu = t(")[0]
exec(src.replace("for name in names:", "for name in names[:1]:"))
for _ in range(2): sc.splitcnn_conv_pool_fwd(pl.handle, 0, sc.BF16, x, w, b, yp, ap)
PY
