"""A/B of the weight-gradient call (with db) of C5 layers: env toggles flipped between repeats."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
flag = sys.argv[1] if len(sys.argv) > 1 else "SPLITCNN_NO_FUSED_DB"
names = sys.argv[2].split(",") if len(sys.argv) > 2 else ["conv1_2", "conv2_1", "conv2_2", "conv3_2", "conv4_2", "conv5_2"]
c = synth.vgg_config("C5")
layers = c["layers"] + c["tail"]
def setup(name):
    idx = [l["name"] for l in layers].index(name); l = layers[idx]
    H = c["H"]
    for k in layers[:idx]:
        H = (H + k["ph_b"] + k["ph_e"] - k["kh"]) // k["sh"] + 1
    nh, nw = c["split"] if idx < len(c["layers"]) else (1, 1)
    Ho = (H + l["ph_b"] + l["ph_e"] - l["kh"]) // l["sh"] + 1
    pl = SplitPlan([l], c["N"], l["cin"], H, H, sc.splitcnn_boundaries_even(Ho, min(nh, Ho)), sc.splitcnn_boundaries_even(Ho, min(nw, Ho)))
    lv0, lv1 = pl.levels
    x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
    y = torch.randn(lv1["total_elems"], device="cuda").to(torch.bfloat16)
    ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dw = torch.empty((l["cout"], l["kh"], l["kw"], lv0["Cpad"]), device="cuda")
    db = torch.empty(l["cout"], device="cuda")
    return lambda: sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, y, dw, db, 0.0, ws, ws_b), (dw, db)
def t(fn, n=20):
    for _ in range(3): fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(n): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n
for name in names:
    fn, (dw, db) = setup(name)
    res = {"A": [], "B": []}
    for rep in range(3):
        for k in ("A", "B"):
            if k == "B": os.environ[flag] = "1"
            else: os.environ.pop(flag, None)
            res[k].append(t(fn))
    os.environ.pop(flag, None); fn(); ref = (dw.clone(), db.clone())
    os.environ[flag] = "1"; fn(); os.environ.pop(flag, None)
    print(name, "A(default) ms", [round(v, 4) for v in res["A"]], f"B({flag}) ms", [round(v, 4) for v in res["B"]],
          "db maxdiff", float((ref[1] - db).abs().max() / db.abs().max()), "dW eq", torch.equal(ref[0], dw), flush=True)
