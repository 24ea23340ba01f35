"""Time max-pool fwd / bwd of C5 pool1, pool2 (2x2 s2, 8x8 split) and C3's 3x3 s2 p1 pool (2x2 split)."""
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


cases = [("C5 pool1", 256, 64, 224, 2, 2, 0, 8), ("C5 pool2", 256, 128, 112, 2, 2, 0, 8),
         ("C3 maxpool", 256, 64, 112, 3, 2, 1, 2)]
for name, N, C, H, k, s, p, ns in cases:
    l = synth.maxpool(C, k, s, p)
    Ho = (H + 2 * p - k) // s + 1
    O = sc.splitcnn_boundaries_even(Ho, ns)
    pl = SplitPlan([l], N, C, H, H, O, O)
    lv0, lv1 = pl.levels
    x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
    y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
    a = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.uint8)
    dx = torch.empty_like(x)
    f = t(lambda: sc.splitcnn_pool_fwd(pl.handle, 0, sc.BF16, x, y, a, sc.FLAG_POOL_RELU_MASK))
    b = t(lambda: sc.splitcnn_pool_bwd(pl.handle, 0, sc.BF16, y, a, dx, sc.FLAG_POOL_RELU_MASK))
    byt = x.numel() * 2 + y.numel() * 3
    print(f"{name}: fwd {f:.4f} ms {byt / f / 1e6:.0f} GB/s | bwd {b:.4f} ms {byt / b / 1e6:.0f} GB/s")
