"""wgrad with and without the fused-call db (side-stream column sums) for C5 layers, in isolation."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
for name, cin, cout, H, ns in (("conv1_1", 3, 64, 224, 8), ("conv1_2", 64, 64, 224, 8), ("conv2_1", 64, 128, 112, 8),
                               ("conv2_2", 128, 128, 112, 8), ("conv3_2", 256, 256, 56, 8)):
    l = synth.conv(cin, cout, name=name)
    Ob = sc.splitcnn_boundaries_even(H, ns)
    pl = SplitPlan([l], 256, cin, H, H, Ob, Ob)
    lv0, lv1 = pl.levels
    x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
    dy = torch.randn(lv1["total_elems"], device="cuda").to(torch.bfloat16)
    ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dw = torch.empty((cout, 3, 3, lv0["Cpad"]), device="cuda")
    db = torch.empty(cout, device="cuda")
    def t(fn, n=20):
        for _ in range(3): fn()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize(); e0.record()
        for _ in range(n): fn()
        e1.record(); torch.cuda.synchronize()
        return e0.elapsed_time(e1) / n
    a = t(lambda: sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, dy, dw, None, 0.0, ws, ws_b))
    b = t(lambda: sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, dy, dw, db, 0.0, ws, ws_b))
    print(f"{name}: wgrad {a:.4f} ms, wgrad+db {b:.4f} ms, db cost {b - a:+.4f} ms, |dY| {dy.numel() * 2 / 1e9:.3f} GB")
