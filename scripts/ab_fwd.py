"""A/B of conv fwd + dgrad of C5 layers in ONE process: env flag unset (A) vs set (B), interleaved."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
flag = sys.argv[1]
names = sys.argv[2].split(",")
c = synth.vgg_config("C5")
layers = c["layers"] + c["tail"]
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
    Ho = (H + l["ph_b"] + l["ph_e"] - l["kh"]) // l["sh"] + 1
    pl = SplitPlan([l], c["N"], l["cin"], H, H, sc.splitcnn_boundaries_even(Ho, min(nh, Ho)), sc.splitcnn_boundaries_even(Ho, min(nw, Ho)))
    lv0, lv1 = pl.levels
    x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
    y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
    w = (torch.randn(l["cout"], l["kh"], l["kw"], lv0["Cpad"], device="cuda") * 0.05).to(torch.bfloat16)
    b = torch.zeros(l["cout"], device="cuda")
    ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    res = {"A": [], "B": []}
    for rep in range(3):
        for k in ("A", "B"):
            if k == "B": os.environ[flag] = "1"
            else: os.environ.pop(flag, None)
            res[k].append((t(lambda: sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU)),
                           t(lambda: sc.splitcnn_conv_bwd_data(pl.handle, 0, sc.BF16, y, w, x, x, ws, ws_b))))
    os.environ.pop(flag, None)
    f = lambda L: "fwd " + " ".join(f"{a:.4f}" for a, _ in L) + " | dgrad " + " ".join(f"{d:.4f}" for _, d in L)
    print(f"{name}: A {f(res['A'])}   B({flag}) {f(res['B'])}", flush=True)
