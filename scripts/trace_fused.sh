#!/bin/bash
# per-tile trace of the fused conv1_2 -> pool1 forward (conv_pool_fwd), C5 geometry
mkdir -p gpurun_out
timeout 300 python scripts/ab_pool.py conv1_2,conv2_2 > gpurun_out/trace_fused.txt 2>&1
SPLITCNN_TRACE=1 timeout 120 python - <<'PY' 2>&1 | grep -v "trace CTA (block" | head -40 >> gpurun_out/trace_fused.txt
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
c = synth.vgg_config("C5"); layers = c["layers"]
l, lp = layers[1], layers[2]
pl = SplitPlan([l, lp], 256, 64, 224, 224, sc.splitcnn_boundaries_even(112, 8), sc.splitcnn_boundaries_even(112, 8))
lv0, lv1, lv2 = pl.levels
x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
yp = torch.empty(lv2["total_elems"], device="cuda", dtype=torch.bfloat16)
ap = torch.empty(lv2["total_elems"], device="cuda", dtype=torch.uint8)
w = (torch.randn(64, 3, 3, 64, device="cuda") * 0.05).to(torch.bfloat16)
b = torch.zeros(64, device="cuda")
for _ in range(2): sc.splitcnn_conv_pool_fwd(pl.handle, 0, sc.BF16, x, w, b, yp, ap)
PY
