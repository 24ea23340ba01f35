"""CPU pins for tests/oracle_chain.run -- the oracle composition of a whole VGG split stack
(split -> chained split region -> merge -> unsplit tail; forward and every dW / db) that the
whole-stack GPU parity tests compare against.  What fixes the expected values: torch CPU fp64
autograd (library routines), NOT the oracle's own composition rules:

* pin-1 for the composition: with a 1x1 region split, Split-CNN is the ordinary network
  (the only patch gets the layer's own (p_b, p_e)), so the whole step must equal
  F.conv2d / F.relu / F.max_pool2d under autograd;
* pin-2 for the composition: a 2x2 (and a ragged) region split equals torch autograd of the
  network written patch by patch -- F.pad by the patch-local pads of R2 (interior pads
  (p_b, k-s-p_b)), F.conv2d(padding=0), ReLU, max-pool per patch, torch.cat at the merge (Eq. 4-7,
  P:163).  Autograd decides which tensors carry a ReLU mask (including the join level between
  region and tail), independently of oracle_chain's own mask rule.
"""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

import synth
from tests import oracle_chain


def _slim_vgg(pool_inside):
    """A narrow VGG-shaped stack: 3 conv blocks in the region, 2 in the tail.  pool_inside puts the
    pool after the last region conv inside the region (C2 layout), else it opens the tail (C4/C5)."""
    c, p = synth.conv, synth.maxpool
    region = [c(3, 4), c(4, 4), p(4), c(4, 8), c(8, 8), p(8), c(8, 8), c(8, 8)]
    tail = [c(8, 16), p(16), c(16, 16)]
    if pool_inside:
        region.append(p(8))
    else:
        tail = [p(8)] + tail
    return region, tail


def _in_bounds(layers, O):
    """R2 backwards through the chain (I = s * O at every layer): the boundaries at each layer input."""
    Bs = [list(O)]
    for l in reversed(layers):
        Bs.append([l["sh"] * o for o in Bs[-1]])
    return Bs[::-1]          # Bs[m] = boundaries at the input of layer m; Bs[-1] = region output


def _torch_patchwise(region, tail, X, params, Oh, Ow):
    """The split stack in torch fp64, patch by patch (R2 pads), then the unsplit tail.  Returns
    (output, list of (W, b) leaf tensors in conv order)."""
    Bh, Bw = _in_bounds(region, Oh), _in_bounds(region, Ow)
    ps = [(torch.tensor(W, requires_grad=True), torch.tensor(b, requires_grad=True)) for W, b in params]
    it = iter(ps)
    x = torch.tensor(X)
    P = [[x[:, :, Bh[0][i]:Bh[0][i + 1], Bw[0][j]:Bw[0][j + 1]] for j in range(len(Bw[0]) - 1)]
         for i in range(len(Bh[0]) - 1)]
    for l in region:
        k, s, pb, pe = l["kh"], l["sh"], l["ph_b"], l["ph_e"]
        nh, nw = len(P), len(P[0])
        if l["op"] == "conv":
            W, b = next(it)
        out = []
        for i in range(nh):
            row = []
            for j in range(nw):
                t, bo = pb, (pe if i == nh - 1 else k - s - pb)
                le, ri = pb, (pe if j == nw - 1 else k - s - pb)
                if l["op"] == "conv":
                    y = F.conv2d(F.pad(P[i][j], (le, ri, t, bo)), W, b, stride=s)
                    row.append(F.relu(y) if l.get("relu", True) else y)
                else:
                    row.append(F.max_pool2d(F.pad(P[i][j], (le, ri, t, bo), value=-np.inf), k, s))
            out.append(row)
        P = out
    h = torch.cat([torch.cat(row, 3) for row in P], 2)
    for l in tail:
        if l["op"] == "conv":
            W, b = next(it)
            h = F.conv2d(h, W, b, stride=l["sh"], padding=l["ph_b"])
            h = F.relu(h) if l.get("relu", True) else h
        else:
            h = F.max_pool2d(h, l["kh"], l["sh"], l["ph_b"])
    return h, ps


def _region_out(region, H):
    for l in region:
        H = (H + l["ph_b"] + l["ph_e"] - l["kh"]) // l["sh"] + 1
    return H


def _check(region, tail, N, H, Oh, Ow, seed, rel=1e-10):
    g = synth.rng(seed)
    X = synth.uniform(g, (N, 3, H, H)).astype(np.float64)
    params = [(W.astype(np.float64), b.astype(np.float64))
              for W, b in (p for p in synth.layer_params(g, region + tail) if p is not None)]
    Y, ps = _torch_patchwise(region, tail, X, params, Oh, Ow)
    G = synth.normal(g, tuple(Y.shape)).astype(np.float64)
    (Y * torch.tensor(G)).sum().backward()
    out, dWs, dbs, _ = oracle_chain.run(region, tail, N, 3, H, H, Oh, Ow, params, X, G)
    assert out.shape == tuple(Y.shape)
    assert np.abs(out - Y.detach().numpy()).max() <= 1e-12 * max(1.0, np.abs(out).max())
    assert len(dWs) == len(ps)
    for (Wt, bt), dW, db in zip(ps, dWs, dbs):
        assert np.abs(dW - Wt.grad.numpy()).max() <= rel * max(1.0, np.abs(dW).max())
        assert np.abs(db - bt.grad.numpy()).max() <= rel * max(1.0, np.abs(db).max())


@pytest.mark.parametrize("pool_inside", [True, False])
def test_vgg_chain_1x1_split_equals_unsplit_torch(pool_inside):
    """pin-1: 1x1 split -> the ordinary network (F.conv2d(padding=1) / F.max_pool2d) under autograd."""
    region, tail = _slim_vgg(pool_inside)
    L = _region_out(region, 32)
    _check(region, tail, 2, 32, [0, L], [0, L], seed=31)


@pytest.mark.parametrize("pool_inside", [True, False])
def test_vgg_chain_2x2_split_equals_patchwise_torch(pool_inside):
    """pin-2: even 2x2 split -> the patch-by-patch torch network under autograd."""
    region, tail = _slim_vgg(pool_inside)
    L = _region_out(region, 32)
    _check(region, tail, 2, 32, [0, L // 2, L], [0, L // 2, L], seed=32)


def test_vgg_chain_ragged_split_equals_patchwise_torch():
    """pin-2 with uneven (stochastic-like) boundaries: 3 x 2 patches of unequal size."""
    region, tail = _slim_vgg(False)
    L = _region_out(region, 64)          # 64 -> 16 at the region output (two pools inside)
    _check(region, tail, 1, 64, [0, 5, 11, L], [0, 9, L], seed=33)


def test_vgg_chain_1x1_split_equals_patchwise_vs_unsplit_differ():
    """Sanity of the pins above: the 2x2 split network is NOT the unsplit one (Split-CNN changes
    the result), so the two pins are not the same check twice."""
    region, tail = _slim_vgg(True)
    g = synth.rng(34)
    X = synth.uniform(g, (1, 3, 32, 32)).astype(np.float64)
    params = [(W.astype(np.float64), b.astype(np.float64))
              for W, b in (p for p in synth.layer_params(g, region + tail) if p is not None)]
    L = _region_out(region, 32)
    a, _ = _torch_patchwise(region, tail, X, params, [0, L], [0, L])
    b, _ = _torch_patchwise(region, tail, X, params, [0, L // 2, L], [0, L // 2, L])
    assert not torch.allclose(a, b)


@pytest.mark.slow
def test_c2_chain_2x2_split_equals_patchwise_torch():
    """pin-2 on the real C2 composition (VGG-19 widths, depth 50%, pool inside), N=1."""
    c = synth.vgg_config("C2", N=1)
    L = _region_out(c["layers"], 32)
    _check(c["layers"], c["tail"], 1, 32, [0, L // 2, L], [0, L // 2, L], seed=1, rel=1e-9)
