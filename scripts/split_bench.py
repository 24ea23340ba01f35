"""Time the input split (NCHW bf16 -> patch buffers) of C5 (N=256, 3x224x224, 8x8) and C3's S2D split."""
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
O = sc.splitcnn_boundaries_even(224, 8)
pl = SplitPlan([synth.conv(3, 64)], 256, 3, 224, 224, O, O)
x = torch.randn(256, 3, 224, 224, device="cuda").to(torch.bfloat16)
p = torch.empty(pl.levels[0]["total_elems"], device="cuda", dtype=torch.bfloat16)
ms = t(lambda: sc.splitcnn_split(pl.handle, 0, sc.BF16, x, sc.NCHW, p))
print(f"C5 input split {ms:.4f} ms {(x.numel() * 2 + p.numel() * 2) / ms / 1e6:.0f} GB/s (actual bytes)")
y = torch.empty_like(x)
ms = t(lambda: sc.splitcnn_merge(pl.handle, 0, sc.BF16, p, y, sc.NCHW))
print(f"C5 merge to NCHW {ms:.4f} ms; roundtrip exact: {torch.equal(x, y)}")
