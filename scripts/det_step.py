"""Locate non-reproducibility inside one SplitNet step: compare activations after forward and after
backward, and the gradients, across repeated steps."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200.net import SplitNet
N = int(sys.argv[1]) if len(sys.argv) > 1 else 16
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 8
c = synth.vgg_config("C5", N=N)
g = synth.rng(4)
params = [p for p in synth.layer_params(g, c["layers"] + c["tail"]) if p is not None]
tp = [(torch.from_numpy(W), torch.from_numpy(b)) for W, b in params]
x = torch.from_numpy(synth.uniform(g, (N, 3, 224, 224))).to("cuda", torch.bfloat16)
net = SplitNet(c["layers"], c["tail"], N, 3, 224, 224, split=c["split"], mode=c["mode"], seed=c["seed"])
net.set_params(tp)
dy = torch.randn(net.output_numel(), generator=torch.Generator().manual_seed(0)).to("cuda", torch.bfloat16)
snap = lambda: [a.clone() for a in net.act_r + net.act_t]
ref_f = ref_b = None
for r in range(reps):
    net.forward(x); torch.cuda.synchronize(); f = snap()
    net.backward(dy); torch.cuda.synchronize(); b = snap()
    if ref_f is None:
        ref_f, ref_b = f, b; continue
    df = [i for i in range(len(f)) if not torch.equal(f[i], ref_f[i])]
    db = [i for i in range(len(b)) if not torch.equal(b[i], ref_b[i])]
    fb = [i for i in range(len(b)) if not torch.equal(b[i], f[i])]
    print("rep", r, "fwd acts differ", df[:6], "post-bwd acts differ", db[:6], "acts changed by bwd", fb[:6], flush=True)
