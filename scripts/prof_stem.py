"""C3 stem (s2d 4x4 conv, 16- or 64-channel input) forward at full size, one call after warm-up -- for ncu:
    ncu --set full -k regex:conv_tc -s 2 -c 1 python scripts/prof_stem.py 16"""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
from paper_conf_asplos_jinh19_b200.resnet import s2d_stem_layer
pad = int(sys.argv[1]) if len(sys.argv) > 1 else 16
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
N = 256
l = s2d_stem_layer(synth.conv(3, 64, k=7, s=2, p=3), pad)
O = sc.splitcnn_boundaries_even(112, 8)
pl = SplitPlan([l], N, l["cin"], 112, 112, O, O)
lv0, lv1 = pl.levels
x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
w = (torch.randn(64, 4, 4, lv0["Cpad"], device="cuda") * 0.05).to(torch.bfloat16)
b = torch.zeros(64, device="cuda")
ev = [torch.cuda.Event(enable_timing=True) for _ in range(reps + 1)]
for i in range(reps):
    ev[i].record()
    sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU)
ev[reps].record()
torch.cuda.synchronize()
print(f"stem pad {pad}: " + " ".join(f"{ev[i].elapsed_time(ev[i + 1]):.4f}" for i in range(reps)) + " ms")
