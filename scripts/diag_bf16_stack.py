"""Diagnostic (GPU): whole-stack bf16 errors vs the oracle for VGG / ResNet stacks, Kaiming draws
(decision flips re-route gradient elements) and dyadic draws (exact sums, same decisions).
Prints one JSON line per case with the max dW / db / out normwise error (R13)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import __graft_entry__  # noqa: E402
from tests import test_gpu_bn as TB, test_gpu_resnet as TR, test_gpu_stack as TS  # noqa: E402

__graft_entry__.build()
from paper_conf_asplos_jinh19_b200 import splitcnn as sc  # noqa: E402


def summ(tag, errs):
    dw = {k: v for k, v in errs.items() if k.startswith("dW")}
    db = {k: v for k, v in errs.items() if k.startswith("d") and not k.startswith("dW")}
    print(json.dumps({"case": tag, "out": errs.get("out"), "dW_max": max(dw.values()), "db_max": max(db.values()),
                      "flip": errs.get("argmax_flip_frac")}), flush=True)


def guard(tag, fn):
    try:
        summ(tag, fn())
    except AssertionError as e:
        print(json.dumps({"case": tag, "assert": str(e)[:200]}), flush=True)


cases = sys.argv[1:] or ["vgg", "res", "bn"]
for exact in (False, True):
    if "vgg" in cases:
        for N in (2, 8):
            guard(f"C2 N={N} exact={exact}", lambda: TS._run(sc, "C2", N, sc.BF16, exact=exact, seed=100))
        for H, N in ((64, 1), (128, 2)):
            guard(f"C4 H={H} N={N} exact={exact}", lambda: TS._run(sc, "C4", N, sc.BF16, H=H, exact=exact, seed=102))
    if "res" in cases:
        for N, H in ((2, 64), (2, 224)):
            guard(f"res N={N} H={H} exact={exact}", lambda: TR._run(sc, sc.BF16, N=N, H=H, exact=exact, seed=200))
    if "bn" in cases:
        for N, H in ((2, 64), (2, 128)):
            guard(f"bn N={N} H={H} exact={exact}", lambda: TB._run_stack(sc, sc.BF16, N=N, H=H, exact=exact))
torch.cuda.synchronize()
