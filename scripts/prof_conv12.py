"""conv1_2 (+ fused pool1) of C5 at full size, one call of each pass after a warm-up -- for ncu:
    ncu --set full -k regex:'conv_tc|wgrad_' -s 3 -c 3 python scripts/prof_conv12.py"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_asplos_jinh19_b200 import splitcnn as sc  # noqa: E402
from paper_conf_asplos_jinh19_b200.plan import SplitPlan  # noqa: E402

N = 256
layers = [synth.conv(64, 64, name="conv1_2"), synth.maxpool(64, name="pool1")]
Ob = sc.splitcnn_boundaries_even(112, 8)
pl = SplitPlan(layers, N, 64, 224, 224, Ob, Ob)
lv0, lv1, lv2 = pl.levels
x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
yp = torch.empty(lv2["total_elems"], device="cuda", dtype=torch.bfloat16)
am = torch.empty(lv2["total_elems"], device="cuda", dtype=torch.uint8)
w = (torch.randn(64, 3, 3, 64, device="cuda") * 0.05).to(torch.bfloat16)
b = torch.zeros(64, device="cuda")
ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
dw = torch.empty((64, 3, 3, 64), device="cuda")
db = torch.empty(64, device="cuda")
fl = 2.0 * N * 64 * 224 * 224 * 64 * 9
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 1
ev = []
for it in range(2 + reps):
    e = [torch.cuda.Event(enable_timing=True) for _ in range(5)]
    e[0].record()
    sc.splitcnn_conv_pool_fwd(pl.handle, 0, sc.BF16, x, w, b, yp, am, sc.FLAG_RELU | sc.FLAG_POOL_RELU_MASK)
    e[1].record()
    sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU)
    e[2].record()
    sc.splitcnn_conv_bwd_data(pl.handle, 0, sc.BF16, y, w, x, x, ws, ws_b)
    e[3].record()
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, y, dw, db, 0.0, ws, ws_b)
    e[4].record()
    ev.append(e)
torch.cuda.synchronize()
if reps > 1:
    names = ["conv_pool_fwd", "conv_fwd", "dgrad", "wgrad+db"]
    for k, nm in enumerate(names):
        ms = sorted(ev[i][k].elapsed_time(ev[i][k + 1]) for i in range(2, 2 + reps))[reps // 2]
        print(f"{nm:14s} {ms:.4f} ms  {fl / ms / 1e9:.1f} TFLOP/s")
