"""Time the BN ops on a C3-sized level (N=256, 56x56x64 and 28x28x128 bf16)."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan
def t(fn, n=20):
    for _ in range(3): fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(n): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n
for C, H in ((64, 56), (128, 28)):
    O = sc.splitcnn_boundaries_even(H, 2)
    pl = SplitPlan([synth.conv(C, C, 1, 1, 0)], 256, C, H, H, O, O)
    lv = pl.levels[0]
    x = torch.randn(lv["total_elems"], device="cuda").to(torch.bfloat16)
    dy = torch.randn_like(x); y = torch.empty_like(x); dx = torch.empty_like(x)
    f = lambda n: torch.zeros(n, dtype=torch.float32, device="cuda")
    sums, mi, t2, gm, bt = f(2 * C), f(2 * C), f(2 * C), f(C) + 1, f(C)
    wsb = sc.splitcnn_bn_workspace_size(pl.handle, 0)
    ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    nb = x.numel() * 2
    a = t(lambda: sc.splitcnn_bn_stats(pl.handle, 0, sc.BF16, x, sums, ws, wsb))
    b = t(lambda: sc.splitcnn_bn_fwd(pl.handle, 0, sc.BF16, x, sums, 256.0 * H * H, gm, bt, 1e-5, mi, y, sc.FLAG_RELU))
    c = t(lambda: sc.splitcnn_bn_bwd_sums(pl.handle, 0, sc.BF16, dy, x, y, mi, t2, ws, wsb))
    d = t(lambda: sc.splitcnn_bn_bwd(pl.handle, 0, sc.BF16, dy, x, y, mi, gm, t2, 256.0 * H * H, dx))
    print(f"C={C} H={H}: stats {a:.4f} ms ({nb/a/1e6:.0f} GB/s) fwd {b:.4f} ({2*nb/b/1e6:.0f}) bwd_sums {c:.4f} ({3*nb/c/1e6:.0f}) bwd {d:.4f} ({4*nb/d/1e6:.0f})")
