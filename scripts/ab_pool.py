"""A/B: fused conv+pool (conv_pool_fwd) vs conv_fwd + pool_fwd for the C5 conv->pool pairs."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
c = synth.vgg_config("C5")
layers = c["layers"] + c["tail"]
names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["conv1_2", "conv2_2", "conv4_4", "conv5_4"]
def t(fn, n=20):
    for _ in range(3): fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(n): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n
for name in names:
    idx = [l["name"] for l in layers].index(name); l = layers[idx]
    H = c["H"]
    for k in layers[:idx]:
        H = (H + k["ph_b"] + k["ph_e"] - k["kh"]) // k["sh"] + 1
    nh, nw = c["split"] if idx < len(c["layers"]) else (1, 1)
    Hp = H // 2
    pl = SplitPlan([l, layers[idx + 1]], c["N"], l["cin"], H, H, sc.splitcnn_boundaries_even(Hp, min(nh, Hp)),
                   sc.splitcnn_boundaries_even(Hp, min(nw, Hp)))
    lv0, lv1, lv2 = pl.levels
    x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
    y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
    yp = torch.empty(lv2["total_elems"], device="cuda", dtype=torch.bfloat16)
    ap = torch.empty(lv2["total_elems"], device="cuda", dtype=torch.uint8)
    w = (torch.randn(l["cout"], 3, 3, lv0["Cpad"], device="cuda") * 0.05).to(torch.bfloat16)
    b = torch.zeros(l["cout"], device="cuda")
    tu = t(lambda: (sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU),
                    sc.splitcnn_pool_fwd(pl.handle, 1, sc.BF16, y, yp, ap, sc.FLAG_POOL_RELU_MASK)))
    tc = t(lambda: sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU))
    tf = t(lambda: sc.splitcnn_conv_pool_fwd(pl.handle, 0, sc.BF16, x, w, b, yp, ap))
    print(f"{name}: conv {tc:.4f} ms, conv+pool {tu:.4f} ms, fused {tf:.4f} ms", flush=True)
