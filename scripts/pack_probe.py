"""How much do partially filled 8-wide M groups cost?  One 3x3 conv (fwd / dgrad) at patch widths that are
(32, 16, 8) and are not (28, 14, 7) multiples of 8, same channels and batch -- TFLOP/s of algorithmic work."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan

def run(C, H, split, N):
    l = synth.conv(C, C, name="c")
    O = sc.splitcnn_boundaries_even(H, split)
    pl = SplitPlan([l], N, C, H, H, O, O)
    lv0, lv1 = pl.levels
    x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
    y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
    w = (torch.randn(C, 3, 3, lv0["Cpad"], device="cuda") * 0.05).to(torch.bfloat16)
    b = torch.zeros(C, device="cuda")
    ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    fl = 2.0 * N * C * H * H * C * 9
    def t(fn, n=10):
        for _ in range(3): fn()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize(); e0.record()
        for _ in range(n): fn()
        e1.record(); torch.cuda.synchronize()
        return e0.elapsed_time(e1) / n
    f = t(lambda: sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU))
    d = t(lambda: sc.splitcnn_conv_bwd_data(pl.handle, 0, sc.BF16, y, w, x, x, ws, ws_b))
    print(f"C={C} H={H} split={split} N={N} patch={H // split}: fwd {f:.4f} ms {fl / f / 1e9:.0f} TF/s, dgrad {d:.4f} ms {fl / d / 1e9:.0f} TF/s")

for C, H, split, N in [(512, 28, 1, 256), (512, 32, 1, 256), (512, 14, 1, 256), (512, 16, 1, 256),
                       (256, 56, 8, 256), (256, 64, 8, 256), (128, 112, 8, 256), (128, 128, 8, 256),
                       (64, 224, 8, 256), (64, 256, 8, 256)]:
    run(C, H, split, N)
