import os, sys, torch, numpy as np
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
C = 13
pl = SplitPlan([synth.conv(C, C, 1, 1, 0)], 3, C, 11, 9, [0, 3, 7, 11], [0, 5, 9])
lv = pl.levels[0]
x = torch.randn(lv["total_elems"], device="cuda")
ws_b = sc.splitcnn_bn_workspace_size(pl.handle, 0)
for fill in (0, 255):
    ws = torch.full((ws_b,), fill, dtype=torch.uint8, device="cuda")
    s_all = torch.zeros(2 * C, device="cuda"); h = torch.zeros(2 * C, device="cuda"); r = torch.zeros(2 * C, device="cuda")
    sc.splitcnn_bn_stats(pl.handle, 0, sc.FP32, x, s_all, ws, ws_b)
    sc.splitcnn_bn_stats(pl.handle, 0, sc.FP32, x, h, ws, ws_b, 0, 2)
    sc.splitcnn_bn_stats(pl.handle, 0, sc.FP32, x, r, ws, ws_b, 2, 6)
    torch.cuda.synchronize()
    xv = x.view(-1, lv["Cpad"])[:, :C].double()
    print("fill", fill, "all", (s_all[:C].double() - xv.sum(0)).abs().max().item(), "h+r", (h + r - s_all).abs().max().item())
    print(s_all[:4].tolist(), h[:4].tolist(), r[:4].tolist())
