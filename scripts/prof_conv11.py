"""conv1_1 of C5 at full size (3 -> 64 channels, input padded to 8, 224x224, N=256, 8x8 split): forward and
weight gradient, median of N calls after a warm-up, or one call of each for ncu (argv[1] = 1)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_asplos_jinh19_b200 import splitcnn as sc  # noqa: E402
from paper_conf_asplos_jinh19_b200.plan import SplitPlan  # noqa: E402

N = 256
l = synth.conv(3, 64, name="conv1_1")
Ob = sc.splitcnn_boundaries_even(224, 8)
pl = SplitPlan([l], N, 3, 224, 224, Ob, Ob)
lv0, lv1 = pl.levels
x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
w = (torch.randn(64, 3, 3, 8, device="cuda") * 0.1).to(torch.bfloat16)
b = torch.zeros(64, device="cuda")
ws_b = max(pl.workspace_size(0, sc.BF16, op) for op in (0, 1, 2))
ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
dw = torch.empty((64, 3, 3, 8), device="cuda")
db = torch.empty(64, device="cuda")
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
ev = []
for it in range(2 + reps):
    e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
    e[0].record()
    sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU)
    e[1].record()
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, y, dw, db, 0.0, ws, ws_b)
    e[2].record()
    ev.append(e)
torch.cuda.synchronize()
if reps > 1:
    alg = (N * 3 * 224 * 224 + N * 64 * 224 * 224) * 2
    for k, nm in enumerate(["fwd", "wgrad+db"]):
        ms = sorted(ev[i][k].elapsed_time(ev[i][k + 1]) for i in range(2, 2 + reps))[reps // 2]
        print(f"{nm:9s} {ms:.4f} ms  {alg / ms / 1e6:.0f} GB/s algorithmic (HBM roofline {alg / 6544e9 * 1e3:.3f} ms)")
