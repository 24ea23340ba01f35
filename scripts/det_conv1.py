"""Repeat conv1_1 forward (C5 geometry, N images) and locate non-reproducible output elements."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
N = int(sys.argv[1]) if len(sys.argv) > 1 else 16
c = synth.vgg_config("C5", N=N)
l = c["layers"][0]
pl = SplitPlan([l], N, 3, 224, 224, sc.splitcnn_boundaries_even(224, 8), sc.splitcnn_boundaries_even(224, 8))
lv0, lv1 = pl.levels
g = torch.Generator().manual_seed(0)
x = torch.randn(lv0["total_elems"], generator=g).to("cuda", torch.bfloat16)
w = (torch.randn(64, 3, 3, 8, generator=g) * 0.2).to("cuda", torch.bfloat16)
b = torch.zeros(64, device="cuda")
outs = []
for r in range(12):
    y = torch.full((lv1["total_elems"],), float("nan"), device="cuda", dtype=torch.bfloat16)
    sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU)
    torch.cuda.synchronize()
    outs.append(y.clone())
for r in range(1, 12):
    d = (outs[r].float() - outs[0].float()).abs()
    d[torch.isnan(d)] = 1e9
    idx = (d > 0).nonzero().flatten()
    if len(idx) == 0:
        print("rep", r, "same"); continue
    per_patch = N * 28 * 28 * 64
    p = idx // per_patch; rem = idx % per_patch
    n = rem // (28 * 28 * 64); rem = rem % (28 * 28 * 64)
    h = rem // (28 * 64); rem = rem % (28 * 64)
    wcol = rem // 64; ch = rem % 64
    print("rep", r, "ndiff", len(idx), "patches", sorted(set(p.tolist()))[:10], "imgs", sorted(set(n.tolist()))[:10],
          "rows", sorted(set(h.tolist())), "cols", sorted(set(wcol.tolist())), "chans", len(set(ch.tolist())),
          "nan", int(torch.isnan(outs[r].float()).sum()))
