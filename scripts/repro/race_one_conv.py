"""One small 2-CTA tcgen05 forward conv (64 -> 256 channels, 2x2 split, N = 4) for compute-sanitizer racecheck."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import synth  # noqa: E402
from paper_conf_asplos_jinh19_b200 import splitcnn as sc  # noqa: E402
from paper_conf_asplos_jinh19_b200.plan import SplitPlan  # noqa: E402

l = synth.conv(64, 256)
pl = SplitPlan([l], 4, 64, 32, 32, [0, 16, 32], [0, 16, 32])
lv0, lv1 = pl.levels
x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
w = (torch.randn(256, 3, 3, 64, device="cuda") * 0.05).to(torch.bfloat16)
sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, None, y, 0)
torch.cuda.synchronize()
print("conv ok")
