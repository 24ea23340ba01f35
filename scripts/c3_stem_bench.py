"""Time the C3 stem (space-to-depth 4x4 s1 conv on 12(16) channels, N=256, 112x112, 2x2 split): fwd + wgrad."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
from paper_conf_asplos_jinh19_b200.resnet import s2d_stem_layer
l = s2d_stem_layer(synth.conv(3, 64, k=7, s=2, p=3))
O = sc.splitcnn_boundaries_even(112, 2)
pl = SplitPlan([l], 256, 12, 112, 112, O, O)
lv0, lv1 = pl.levels
x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
w = (torch.randn(64, 4, 4, lv0["Cpad"], device="cuda") * 0.05).to(torch.bfloat16)
b = torch.zeros(64, device="cuda")
ws_b = max(pl.workspace_size(0, sc.BF16, 2), 16)
ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
dw = torch.empty((64, 4, 4, lv0["Cpad"]), device="cuda")
def t(fn, n=10):
    for _ in range(3): fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(n): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n
print("stem fwd %.4f ms wgrad %.4f ms" % (t(lambda: sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU)),
                                          t(lambda: sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, y, dw, None, 0.0, ws, ws_b))))
