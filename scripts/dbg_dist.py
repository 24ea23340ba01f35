import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
import torch.distributed as dist
from paper_conf_asplos_jinh19_b200.dist import DistSplitNet
from paper_conf_asplos_jinh19_b200.net import SplitNet
os.environ.setdefault("MASTER_ADDR", "127.0.0.1"); os.environ.setdefault("MASTER_PORT", "29533")
dist.init_process_group("nccl", rank=0, world_size=1)
c = synth.vgg_config("C5", N=2)
g = synth.rng(4)
params = [p for p in synth.layer_params(g, c["layers"] + c["tail"]) if p is not None]
tp = [(torch.from_numpy(W), torch.from_numpy(b)) for W, b in params]
x = torch.from_numpy(synth.uniform(g, (2, 3, 224, 224))).to("cuda", torch.bfloat16)
nets = []
for k in range(3):
    n = SplitNet(c["layers"], c["tail"], 2, 3, 224, 224, split=c["split"], mode=c["mode"], seed=c["seed"]) if k < 2 else DistSplitNet(c, 1, 0)
    n.set_params(tp); nets.append(n)
dy = torch.randn(nets[0].output_numel(), generator=torch.Generator().manual_seed(0)).to("cuda", torch.bfloat16)
for n in nets: n.step(x, dy)
torch.cuda.synchronize()
for key, (dW, db) in nets[0].grads.items():
    for k in (1, 2):
        dW2, db2 = nets[k].grads[key]
        print(k, key, "dW eq", torch.equal(dW, dW2), float((dW - dW2).abs().max()), "db eq", torch.equal(db, db2), float((db - db2).abs().max()))
