"""One small C2 step (N=2), a C5-geometry step (224x224, 8x8 split, N=2) and a C3-shaped ResNet step for
compute-sanitizer runs."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200.net import SplitNet
from paper_conf_asplos_jinh19_b200.resnet import ResSplitNet
c = synth.vgg_config("C2", N=2)
g = synth.rng(1)
params = [p for p in synth.layer_params(g, c["layers"] + c["tail"]) if p is not None]
net = SplitNet(c["layers"], c["tail"], 2, 3, 32, 32, split=c["split"], static_pool=True)
net.set_params([(torch.from_numpy(W), torch.from_numpy(b)) for W, b in params])
x = torch.from_numpy(synth.uniform(g, (2, 3, 32, 32))).to("cuda", torch.bfloat16)
dy = torch.randn(net.output_numel()).to("cuda", torch.bfloat16)
net.step(x, dy)
c5 = synth.vgg_config("C5", N=2)
p5 = [p for p in synth.layer_params(g, c5["layers"] + c5["tail"]) if p is not None]
n5 = SplitNet(c5["layers"], c5["tail"], 2, 3, 224, 224, split=c5["split"])
n5.set_params([(torch.from_numpy(W), torch.from_numpy(b)) for W, b in p5])
x5 = torch.from_numpy(synth.uniform(g, (2, 3, 224, 224))).to("cuda", torch.bfloat16)
n5.step(x5, torch.randn(n5.output_numel()).to("cuda", torch.bfloat16))
rc, rb = synth.resnet18_blocks()
rn = ResSplitNet(rc, rb, 2, 3, 64, 64, split=(2, 2))
rn.set_params([(torch.from_numpy(W), torch.from_numpy(b)) for W, b in synth.resnet_params(g, rc, rb)])
xr = torch.from_numpy(synth.uniform(g, (2, 3, 64, 64))).to("cuda", torch.bfloat16)
rn.step(xr, torch.randn(rn.output_numel()).to("cuda", torch.bfloat16))
torch.cuda.synchronize()
print("step ok")
