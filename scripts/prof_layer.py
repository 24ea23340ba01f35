"""One warm-up then one call of each pass (fwd, dgrad, wgrad) of one C5 layer -- for ncu captures:
    ncu --set full -k regex:'conv_tc|wgrad_' -s 3 -c 3 python scripts/prof_layer.py conv1_2 [C5] [db]"""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
name = sys.argv[1] if len(sys.argv) > 1 else "conv1_2"
cfg = sys.argv[2] if len(sys.argv) > 2 else "C5"
with_db = len(sys.argv) > 3 and sys.argv[3] == "db"
c = synth.vgg_config(cfg)
layers = c["layers"] + c["tail"]
idx = [l["name"] for l in layers].index(name)
l = layers[idx]
H = c["H"]
for k in layers[:idx]:
    H = (H + k["ph_b"] + k["ph_e"] - k["kh"]) // k["sh"] + 1
nh, nw = c["split"] if idx < len(c["layers"]) else (1, 1)
Ho = (H + l["ph_b"] + l["ph_e"] - l["kh"]) // l["sh"] + 1
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
db = torch.empty(l["cout"], device="cuda") if with_db else None
for _ in range(2):
    sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU)
    if idx > 0:
        sc.splitcnn_conv_bwd_data(pl.handle, 0, sc.BF16, y, w, x, x, ws, ws_b)
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, y, dw, db, 0.0, ws, ws_b)
torch.cuda.synchronize()
print("done", name)
