"""Host issue time per step (CPU wall time of enqueueing one step, GPU work asynchronous) vs the device
time of the step, for a config (default C5).  python scripts/host_time.py [C5|C2|C4] [N]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_jinh19_b200.net import SplitNet  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
c = synth.vgg_config(cfg, N=int(sys.argv[2]) if len(sys.argv) > 2 else None)
net = SplitNet(c["layers"], c["tail"], c["N"], 3, c["H"], c["W"], split=c["split"], mode=c["mode"],
               omega=c.get("omega", 0.2), seed=c["seed"], static_pool=True)
g = synth.rng(c["seed"])
net.set_params([(torch.from_numpy(W), torch.from_numpy(b)) for W, b in
                (p for p in synth.layer_params(g, c["layers"] + c["tail"]) if p is not None)])
x = torch.rand((c["N"], 3, c["H"], c["W"]), device="cuda").to(torch.bfloat16)
dy = torch.randn(net.output_numel(), device="cuda").to(torch.bfloat16)
for _ in range(3):
    net.step(x, dy)
torch.cuda.synchronize()
host, dev = [], []
for _ in range(10):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    t0 = time.perf_counter()
    net.step(x, dy)
    host.append(time.perf_counter() - t0)
    e1.record()
    torch.cuda.synchronize()
    dev.append(e0.elapsed_time(e1) / 1e3)
print(f"{cfg} N={c['N']}: host issue {1e3 * sorted(host)[5]:.3f} ms/step (median), device {1e3 * sorted(dev)[5]:.3f} ms/step")
