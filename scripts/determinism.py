"""Run the same SplitNet step repeatedly and report which gradients are not bitwise reproducible."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200.net import SplitNet
cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
N = int(sys.argv[2]) if len(sys.argv) > 2 else 2
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 20
c = synth.vgg_config(cfg, N=N)
g = synth.rng(4)
params = [p for p in synth.layer_params(g, c["layers"] + c["tail"]) if p is not None]
tp = [(torch.from_numpy(W), torch.from_numpy(b)) for W, b in params]
x = torch.from_numpy(synth.uniform(g, (N, 3, c["H"], c["W"]))).to("cuda", torch.bfloat16)
net = SplitNet(c["layers"], c["tail"], N, 3, c["H"], c["W"], split=c["split"], mode=c["mode"], seed=c["seed"])
net.set_params(tp)
dy = torch.randn(net.output_numel(), generator=torch.Generator().manual_seed(0)).to("cuda", torch.bfloat16)
net.step(x, dy); torch.cuda.synchronize()
ref = {k: (v[0].clone(), v[1].clone()) for k, v in net.grads.items()}
out = net.output_numel()
acts = [a.clone() for a in net.act_r + net.act_t]
nbad = 0
for r in range(reps):
    net.step(x, dy); torch.cuda.synchronize()
    bad = [k for k, v in net.grads.items() if not (torch.equal(v[0], ref[k][0]) and torch.equal(v[1], ref[k][1]))]
    badact = [i for i, a in enumerate(net.act_r + net.act_t) if not torch.equal(a, acts[i])]
    if bad or badact:
        nbad += 1
        a1 = (net.act_r + net.act_t)[badact[0]] if badact else None
        d = (a1.float() - acts[badact[0]].float()).abs() if badact else None
        print("rep", r, "grads differ:", len(bad), "acts differ:", badact[:5],
              "first act: n diff", int((d > 0).sum()) if d is not None else 0, "max", float(d.max()) if d is not None else 0,
              "first idx", int((d > 0).nonzero()[0]) if d is not None else -1, flush=True)
    ref = {k: (v[0].clone(), v[1].clone()) for k, v in net.grads.items()}
    acts = [a.clone() for a in net.act_r + net.act_t]
print(cfg, "N", N, "reps", reps, "non-reproducible reps:", nbad)
