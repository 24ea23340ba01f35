"""Seeded synthetic inputs and model/config definitions shared by the oracle and
the CUDA path.  This module holds NONE of the method's arithmetic: only layer
lists (pure data), the BASELINE.json configs, and numpy ``PCG64(seed)`` draws.

Input recipe:
    X    ~ U[-1, 1)
    W    ~ N(0, 2 / fan_in)          (Kaiming)
    bias ~ U[-0.1, 0.1)
    dY   ~ N(0, 1)                   (loss = <Y, G> with G fixed; no FC head / labels)
Seeds: C1 = 0, C2 = 1, C3 = 2, C4 = 3 (boundary seed 3, step = iteration), C5 = 4.
"""
from __future__ import annotations

import numpy as np


# --------------------------------------------------------------------------- layers (pure data)
def conv(cin, cout, k=3, s=1, p=1, relu=True, name=""):
    return dict(op="conv", kh=k, kw=k, sh=s, sw=s, ph_b=p, ph_e=p, pw_b=p, pw_e=p,
                cin=cin, cout=cout, relu=relu, name=name)


def maxpool(c, k=2, s=2, p=0, name=""):
    return dict(op="maxpool", kh=k, kw=k, sh=s, sw=s, ph_b=p, ph_e=p, pw_b=p, pw_e=p,
                cin=c, cout=c, relu=False, name=name)


def vgg19_layers():
    """The VGG-19 convolutional stack: 16 conv3x3(+ReLU), 5 max-pool 2x2 s2 (no BN)."""
    cfg = [(64, 2), (128, 2), (256, 4), (512, 4), (512, 4)]
    layers, c = [], 3
    for b, (w, reps) in enumerate(cfg, start=1):
        for r in range(1, reps + 1):
            layers.append(conv(c, w, name=f"conv{b}_{r}"))
            c = w
        layers.append(maxpool(c, name=f"pool{b}"))
    return layers


def resnet18_split_stack():
    """BN-free ResNet-18-shaped split stack through layer2:
    conv1 7x7 s2 p3 -> ReLU -> maxpool 3x3 s2 p1 -> layer1 (4 conv3x3) ->
    layer2 (conv3x3 s2, 3 conv3x3).  The 1x1 s2 downsample is a separate branch."""
    L = [conv(3, 64, k=7, s=2, p=3, name="conv1"), maxpool(64, k=3, s=2, p=1, name="maxpool")]
    for i in range(4):
        L.append(conv(64, 64, name=f"layer1_{i}"))
    L.append(conv(64, 128, s=2, name="layer2_0"))
    for i in range(1, 4):
        L.append(conv(128, 128, name=f"layer2_{i}"))
    return L


def resnet18_blocks(w1: int = 64, w2: int = 128):
    """The same stack as ``resnet18_split_stack`` with its residual structure (BN-free; P:203
    residual adds): ``chain`` is the main branch as one layer chain (every block's second conv has
    no ReLU of its own -- the ReLU follows the add), ``blocks`` lists per basic block the chain
    index of its first conv and its shortcut (None = identity, else the 1x1 s2 downsample conv)."""
    L = [conv(3, w1, k=7, s=2, p=3, name="conv1"), maxpool(w1, k=3, s=2, p=1, name="maxpool")]
    blocks = []
    c = w1
    for stage, (w, s0) in enumerate(((w1, 1), (w2, 2)), start=1):
        for b in range(2):
            s = s0 if b == 0 else 1
            ds = conv(c, w, k=1, s=s, p=0, relu=False, name=f"layer{stage}_{b}_ds") if (s != 1 or c != w) else None
            blocks.append(dict(a=len(L), ds=ds))
            L.append(conv(c, w, s=s, name=f"layer{stage}_{b}_a"))
            L.append(conv(w, w, relu=False, name=f"layer{stage}_{b}_b"))
            c = w
    return L, blocks


def resnet18_tail_blocks(cin: int = 128, w3: int = 256, w4: int = 512):
    """The unsplit ResNet-18 tail (layer3, layer4; each first block stride 2 with a 1x1 downsample) in
    the same (chain, blocks) form as resnet18_blocks; the global average pool follows it."""
    L, blocks, c = [], [], cin
    for stage, w in ((3, w3), (4, w4)):
        for b in range(2):
            s = 2 if b == 0 else 1
            ds = conv(c, w, k=1, s=s, p=0, relu=False, name=f"layer{stage}_{b}_ds") if (s != 1 or c != w) else None
            blocks.append(dict(a=len(L), ds=ds))
            L.append(conv(c, w, s=s, name=f"layer{stage}_{b}_a"))
            L.append(conv(w, w, relu=False, name=f"layer{stage}_{b}_b"))
            c = w
    return L, blocks


def split_region(layers, depth_convs: int, include_next_pool: bool):
    """First ``depth_convs`` convolutions (plus interleaved pools, plus the pool right
    after the last split conv when ``include_next_pool``) -> (region, tail)."""
    n_conv, cut = 0, len(layers)
    for idx, l in enumerate(layers):
        if l["op"] == "conv":
            n_conv += 1
            if n_conv == depth_convs:
                cut = idx + 1
                if include_next_pool and cut < len(layers) and layers[cut]["op"] == "maxpool":
                    cut += 1
                break
    return layers[:cut], layers[cut:]


# --------------------------------------------------------------------------- BASELINE.json configs
CONFIGS = {
    "C1": dict(name="C1", desc="single split conv3x3 layer, N=2, C=16->16, 32x32, 2x2 split, fp32",
               layers=[conv(16, 16, relu=False, name="conv")], tail=[], N=2, C=16, H=32, W=32,
               split=(2, 2), mode="even", dtype="fp32", seed=0),
    "C2": dict(name="C2", desc="VGG-19 conv stack, CIFAR-shaped 32x32, N=128, 2x2 split, depth 50%",
               N=128, H=32, W=32, split=(2, 2), mode="even", depth=8, pool_inside=True,
               dtype="bf16", seed=1),
    "C3": dict(name="C3", desc="ResNet-18 224x224 (BN-free split stack conv1..layer2), N=256, 2x2 split",
               N=256, H=224, W=224, split=(2, 2), mode="even", dtype="bf16", seed=2, resnet=True),
    "C4": dict(name="C4", desc="VGG-19 224x224, N=512, stochastic 4x4 split at depth 75%, offload",
               N=512, H=224, W=224, split=(4, 4), mode="random", omega=0.2, depth=12,
               pool_inside=False, dtype="bf16", seed=3),
    "C5": dict(name="C5", desc="VGG-19 224x224, N=256, 8x8 split at depth 50%",
               N=256, H=224, W=224, split=(8, 8), mode="even", depth=8, pool_inside=False,
               dtype="bf16", seed=4),
}


def vgg_config(name: str, N: int | None = None):
    """Region/tail layer lists of a VGG config, optionally at a reduced batch ``N``."""
    c = dict(CONFIGS[name])
    if "layers" in c:                      # C1: one explicit layer, no VGG region/tail split
        if N is not None:
            c["N"] = N
        return c
    if c.get("resnet"):
        c["layers"], c["blocks"] = resnet18_blocks()
        c["tail"], c["C"] = [], 3
        if N is not None:
            c["N"] = N
        return c
    region, tail = split_region(vgg19_layers(), c["depth"], c["pool_inside"])
    c["layers"], c["tail"] = region, tail
    c["C"] = 3
    if N is not None:
        c["N"] = N
    return c


# --------------------------------------------------------------------------- seeded draws
def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def uniform(g: np.random.Generator, shape, lo=-1.0, hi=1.0, dtype=np.float32):
    return g.uniform(lo, hi, size=shape).astype(dtype)


def kaiming(g: np.random.Generator, cout, cin, kh, kw, dtype=np.float32):
    std = np.sqrt(2.0 / (cin * kh * kw))
    return (g.standard_normal((cout, cin, kh, kw)) * std).astype(dtype)


def normal(g: np.random.Generator, shape, dtype=np.float32):
    return g.standard_normal(shape).astype(dtype)


def to_bf16_f32(a: np.ndarray) -> np.ndarray:
    """Round float32 values to the nearest bfloat16 (ties to even), returned as float32.
    Used so both sides see the exact same bf16 input bits (R13)."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    u = a.view(np.uint32).astype(np.uint64)
    r = ((u + 0x7FFF + ((u >> 16) & 1)) >> 16) << 16
    return r.astype(np.uint32).view(np.float32)


def resnet_params(g: np.random.Generator, chain, blocks, dtype=np.float32):
    """(W, b) per conv of the chain in order, then per downsample conv in block order."""
    ps = [p for p in layer_params(g, chain, dtype) if p is not None]
    ps += [p for p in layer_params(g, [b["ds"] for b in blocks if b["ds"] is not None], dtype)]
    return ps


def bn_params(g: np.random.Generator, channels, dtype=np.float32):
    """(gamma, beta) per BN: gamma ~ U[0.5, 1.5), beta ~ U[-0.1, 0.1) (so the affine part is exercised)."""
    return [(uniform(g, (c,), 0.5, 1.5, dtype), uniform(g, (c,), -0.1, 0.1, dtype)) for c in channels]


def layer_params(g: np.random.Generator, layers, dtype=np.float32):
    """(W, b) per conv layer in order, None for pools.  W is OIHW, b is [Cout]."""
    out = []
    for l in layers:
        if l["op"] == "conv":
            W = kaiming(g, l["cout"], l["cin"], l["kh"], l["kw"], dtype)
            b = uniform(g, (l["cout"],), -0.1, 0.1, dtype)
            out.append((W, b))
        else:
            out.append(None)
    return out


# --------------------------------------------------------------------------- exact-arithmetic draws
# "Dyadic" inputs for the bf16 whole-stack checks: every value is a small multiple of 1/4 and every
# weight a small integer on a few taps, so every sum the forward / data-gradient passes form is an
# integer multiple of 1/4 far below 2^24 units -- EXACT in fp32 and in fp64, in any order.  Both sides
# then round the same exact value to bf16 (RNE), so the activation and gradient levels, every ReLU mask
# and every pool argmax are the same on both sides, and a whole deep stack can be compared in bf16
# without near-tie decisions (a decision flip would otherwise re-route a whole gradient element).
def dyadic(g: np.random.Generator, shape, lim: int = 8, dtype=np.float32):
    """Integers in [-lim, lim] divided by 4 (exact in bf16)."""
    return (g.integers(-lim, lim + 1, size=shape) / 4.0).astype(dtype)


def sparse_int_weight(g: np.random.Generator, cout, cin, kh, kw, taps: int = 3, dtype=np.float32):
    """OIHW weight with `taps` nonzero entries per output channel at random (ci, r, c), values in
    {-2, -1, 1, 2}."""
    W = np.zeros((cout, cin * kh * kw), dtype=np.float64)
    for co in range(cout):
        pos = g.choice(cin * kh * kw, size=min(taps, cin * kh * kw), replace=False)
        W[co, pos] = g.choice(np.array([-2.0, -1.0, 1.0, 2.0]), size=len(pos))
    return W.reshape(cout, cin, kh, kw).astype(dtype)


def exact_layer_params(g: np.random.Generator, layers, taps: int = 3, dtype=np.float32):
    """layer_params with dyadic values: sparse integer W, bias in {-2..2}/4; None for pools."""
    out = []
    for l in layers:
        if l["op"] == "conv":
            out.append((sparse_int_weight(g, l["cout"], l["cin"], l["kh"], l["kw"], taps, dtype),
                        dyadic(g, (l["cout"],), 2, dtype)))
        else:
            out.append(None)
    return out
