"""Time one split-conv layer (fwd, dgrad, wgrad) of a VGG config in isolation (experiments)."""
import os, sys, json, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
name = sys.argv[1] if len(sys.argv) > 1 else "conv1_2"
cfg = sys.argv[2] if len(sys.argv) > 2 else "C5"
c = synth.vgg_config(cfg)
layers = c["layers"] + c["tail"]
idx = [l["name"] for l in layers].index(name)
l = layers[idx]
in_region = idx < len(c["layers"])
# geometry of this layer's input
H = c["H"]
for k in layers[:idx]:
    H = (H + k["ph_b"] + k["ph_e"] - k["kh"]) // k["sh"] + 1
nh, nw = c["split"] if in_region else (1, 1)
# O at this layer's output, derived from the region's even split at its output level
Ho = (H + l["ph_b"] + l["ph_e"] - l["kh"]) // l["sh"] + 1
scale = 1
Oh = sc.splitcnn_boundaries_even(Ho, min(nh, Ho)); Ow = sc.splitcnn_boundaries_even(Ho, min(nw, Ho))
pl = SplitPlan([l], c["N"], l["cin"], H, H, Oh, Ow)
lv0, lv1 = pl.levels
x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
w = (torch.randn(l["cout"], l["kh"], l["kw"], lv0["Cpad"], device="cuda") * 0.05).to(torch.bfloat16)
b = torch.zeros(l["cout"], device="cuda")
ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
dw = torch.empty((l["cout"], l["kh"], l["kw"], lv0["Cpad"]), device="cuda")
fl = 2.0 * c["N"] * l["cout"] * Ho * Ho * l["cin"] * l["kh"] * l["kw"]
def t(fn, n=10):
    for _ in range(3): fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(n): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n
r = {}
r["fwd_ms"] = t(lambda: sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU))
r["dgrad_ms"] = t(lambda: sc.splitcnn_conv_bwd_data(pl.handle, 0, sc.BF16, y, w, x, x, ws, ws_b))
r["wgrad_ms"] = t(lambda: sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, y, dw, None, 0.0, ws, ws_b))
print(name, cfg, {k: round(v, 4) for k, v in r.items()},
      {k.replace("_ms", "_tflops"): round(fl / (v / 1e3) / 1e12, 1) for k, v in r.items()})
