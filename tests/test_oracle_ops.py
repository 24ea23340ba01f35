"""Pins for oracle.ops (O2-O8) -- CPU only.  What fixes each value:
library routines of torch CPU fp64 (F.conv2d, F.max_pool2d, autograd), closed
forms, invariants and finite differences.  See DESIGN.md."""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

import synth
from oracle import ops as O
from oracle import plan as P

torch.set_default_dtype(torch.float64)


def _plan1(k, s, p, cin, cout, H, W, Oh, Ow, op="conv", N=1):
    l = synth.conv(cin, cout, k, s, p) if op == "conv" else synth.maxpool(cin, k, s, p)
    return P.plan([l], N, cin, H, W, Oh, Ow).layers[0]


def _torch_split_conv(X, Wt, b, lp):
    """pin-2 composition: per patch F.pad(p_i) + F.conv2d(padding=0), concatenated (Eq. 4-7).
    Negative pads (k < s, R2) crop, which F.pad does."""
    rows = []
    for i in range(len(lp.Ih) - 1):
        row = []
        for j in range(len(lp.Iw) - 1):
            xp = X[:, :, lp.Ih[i]:lp.Ih[i + 1], lp.Iw[j]:lp.Iw[j + 1]]
            xp = F.pad(xp, (lp.pads_w[j][0], lp.pads_w[j][1], lp.pads_h[i][0], lp.pads_h[i][1]))
            row.append(F.conv2d(xp, Wt, b, stride=(lp.sh, lp.sw)))
        rows.append(torch.cat(row, 3))
    return torch.cat(rows, 2)


def _merged_conv(X, W, b, lp, relu=False):
    Xp = O.split(X, lp.Ih, lp.Iw)
    return O.merge(O.conv_fwd(Xp, W, b, lp, relu))


GEOMS = [  # (k, s, p, H, W, Oh_count, Ow_count)
    (3, 1, 1, 13, 11, 3, 2),
    (3, 1, 1, 16, 16, 2, 2),
    (7, 2, 3, 22, 18, 2, 3),
    (3, 2, 1, 15, 12, 2, 2),
    (1, 2, 0, 12, 14, 2, 3),   # k < s downsample (R2)
    (5, 1, 2, 9, 10, 2, 2),
]


@pytest.mark.parametrize("k,s,p,H,W,nh,nw", GEOMS)
def test_split_conv_equals_padded_patch_conv_pin2(k, s, p, H, W, nh, nw):
    g = synth.rng(10 + k)
    X = synth.uniform(g, (2, 3, H, W)).astype(np.float64)
    Wt = synth.kaiming(g, 4, 3, k, k).astype(np.float64)
    b = synth.uniform(g, (4,), -0.1, 0.1).astype(np.float64)
    Ho, Wo = P.out_len(H, k, s, p, p), P.out_len(W, k, s, p, p)
    lp = _plan1(k, s, p, 3, 4, H, W, P.boundaries_even(Ho, nh), P.boundaries_even(Wo, nw))
    got = _merged_conv(X, Wt, b, lp)
    ref = _torch_split_conv(torch.from_numpy(X), torch.from_numpy(Wt), torch.from_numpy(b), lp).numpy()
    assert got.shape == ref.shape == (2, 4, Ho, Wo)
    np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("k,s,p", [(3, 1, 1), (7, 2, 3), (1, 2, 0), (3, 2, 1)])
def test_one_by_one_split_is_ordinary_conv_pin1(k, s, p):
    """pin-1: with a single patch, p_0 = (p_b, p_e) and Eq. 6 is F.conv2d."""
    g = synth.rng(20 + k)
    X = synth.uniform(g, (2, 5, 17, 14)).astype(np.float64)
    Wt = synth.kaiming(g, 6, 5, k, k).astype(np.float64)
    b = synth.uniform(g, (6,), -0.1, 0.1).astype(np.float64)
    Ho, Wo = P.out_len(17, k, s, p, p), P.out_len(14, k, s, p, p)
    lp = _plan1(k, s, p, 5, 6, 17, 14, [0, Ho], [0, Wo])
    got = _merged_conv(X, Wt, b, lp, relu=True)
    ref = F.relu(F.conv2d(torch.from_numpy(X), torch.from_numpy(Wt), torch.from_numpy(b), stride=s, padding=p))
    np.testing.assert_allclose(got, ref.numpy(), rtol=1e-12, atol=1e-12)


def test_interior_outputs_equal_unsplit_pin4_and_independence_pin5():
    g = synth.rng(3)
    X = synth.uniform(g, (2, 4, 32, 32)).astype(np.float64)
    Wt = synth.kaiming(g, 4, 4, 3, 3).astype(np.float64)
    lp = _plan1(3, 1, 1, 4, 4, 32, 32, [0, 16, 32], [0, 16, 32])
    got = _merged_conv(X, Wt, None, lp)
    ref = F.conv2d(torch.from_numpy(X), torch.from_numpy(Wt), padding=1).numpy()
    keep = np.ones(32, bool)
    keep[[15, 16]] = False                                    # rows/cols whose window crosses a cut
    np.testing.assert_allclose(got[:, :, keep][:, :, :, keep], ref[:, :, keep][:, :, :, keep], rtol=1e-13, atol=1e-13)
    assert not np.allclose(got[:, :, 15], ref[:, :, 15])
    # pin-5: perturbing patch (1,1)'s input leaves every other patch's output unchanged
    X2 = X.copy()
    X2[:, :, 16:, 16:] += synth.uniform(g, (2, 4, 16, 16)).astype(np.float64)
    got2 = _merged_conv(X2, Wt, None, lp)
    assert np.array_equal(got2[:, :, :16], got[:, :, :16]) and np.array_equal(got2[:, :, :, :16], got[:, :, :, :16])
    assert not np.array_equal(got2[:, :, 16:, 16:], got[:, :, 16:, 16:])


def test_all_ones_closed_form_pin6():
    """pin-6 on the C1 geometry: Y = 16 v_h v_w (v = in-patch taps: 3 interior, 2 at a
    patch edge) -> 144/96/64; dY = 1 gives dX with the same pattern and
    dW[r,c] = N * sum_patches (P - [r != 1])(P - [c != 1]) -> 2048 / 1920 / 1800."""
    X = np.ones((2, 16, 32, 32))
    Wt = np.ones((16, 16, 3, 3))
    lp = _plan1(3, 1, 1, 16, 16, 32, 32, [0, 16, 32], [0, 16, 32])
    Y = _merged_conv(X, Wt, None, lp)
    v = np.full(32, 3.0)
    v[[0, 15, 16, 31]] = 2.0
    assert np.array_equal(Y[0, 0], 16 * np.outer(v, v))
    assert set(np.unique(Y)) == {64.0, 96.0, 144.0}
    dYp = O.split(np.ones_like(Y), lp.Oh, lp.Ow)
    dX = O.merge(O.conv_bwd_data(dYp, Wt, lp))
    assert np.array_equal(dX[1, 3], 16 * np.outer(v, v))
    dW, db = O.conv_bwd_filter(O.split(X, lp.Ih, lp.Iw), dYp, lp)
    exp = np.array([[1800, 1920, 1800], [1920, 2048, 1920], [1800, 1920, 1800]], float)
    assert np.array_equal(dW[5, 7], exp) and np.all(db == 2048)


@pytest.mark.parametrize("k,s,p,H,W,nh,nw", GEOMS)
def test_backward_equals_autograd_of_composition(k, s, p, H, W, nh, nw):
    """dgrad / wgrad (a4, a5) equal torch autograd of the pin-2 composition (a library
    routine), including the ReLU-output mask on dX and db = sum dY (R12)."""
    g = synth.rng(30 + k + s)
    X = synth.uniform(g, (2, 3, H, W)).astype(np.float64)
    Wt = synth.kaiming(g, 4, 3, k, k).astype(np.float64)
    b = synth.uniform(g, (4,), -0.1, 0.1).astype(np.float64)
    Ho, Wo = P.out_len(H, k, s, p, p), P.out_len(W, k, s, p, p)
    lp = _plan1(k, s, p, 3, 4, H, W, P.boundaries_even(Ho, nh), P.boundaries_even(Wo, nw))
    G = synth.normal(g, (2, 4, Ho, Wo)).astype(np.float64)
    Mask = synth.uniform(g, (2, 3, H, W)).astype(np.float64)  # plays "ReLU output" (positive part)
    xt = torch.from_numpy(X).requires_grad_()
    wt = torch.from_numpy(Wt).requires_grad_()
    bt = torch.from_numpy(b).requires_grad_()
    (_torch_split_conv(xt, wt, bt, lp) * torch.from_numpy(G)).sum().backward()
    dYp = O.split(G, lp.Oh, lp.Ow)
    dX = O.merge(O.conv_bwd_data(dYp, Wt, lp))
    dXm = O.merge(O.conv_bwd_data(dYp, Wt, lp, O.split(Mask, lp.Ih, lp.Iw)))
    dW, db = O.conv_bwd_filter(O.split(X, lp.Ih, lp.Iw), dYp, lp)
    np.testing.assert_allclose(dX, xt.grad.numpy(), rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(dXm, np.where(Mask > 0, xt.grad.numpy(), 0), rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(dW, wt.grad.numpy(), rtol=1e-11, atol=1e-11)
    np.testing.assert_allclose(db, bt.grad.numpy(), rtol=1e-12, atol=1e-12)


def test_wgrad_linearity_pin10():
    """pin-10: dW_split = sum over patches of dW of each padded-patch conv, computed
    independently per patch by torch autograd (Eq. 6 is linear in the patches)."""
    g = synth.rng(40)
    X = synth.uniform(g, (1, 2, 10, 9)).astype(np.float64)
    Wt = synth.kaiming(g, 3, 2, 3, 3).astype(np.float64)
    lp = _plan1(3, 1, 1, 2, 3, 10, 9, [0, 3, 10], [0, 5, 9])
    G = synth.normal(g, (1, 3, 10, 9)).astype(np.float64)
    total = np.zeros_like(Wt)
    for i in range(2):
        for j in range(2):
            wt = torch.from_numpy(Wt).requires_grad_()
            xp = torch.from_numpy(X[:, :, lp.Ih[i]:lp.Ih[i + 1], lp.Iw[j]:lp.Iw[j + 1]])
            xp = F.pad(xp, (*lp.pads_w[j], *lp.pads_h[i]))
            gp = torch.from_numpy(G[:, :, lp.Oh[i]:lp.Oh[i + 1], lp.Ow[j]:lp.Ow[j + 1]])
            (F.conv2d(xp, wt) * gp).sum().backward()
            total += wt.grad.numpy()
    dW, _ = O.conv_bwd_filter(O.split(X, lp.Ih, lp.Iw), O.split(G, lp.Oh, lp.Ow), lp)
    np.testing.assert_allclose(dW, total, rtol=1e-12, atol=1e-12)


def test_finite_differences_pin9():
    """pin-9: central finite differences in fp64 on N=1, C 2->3, 6x6, boundaries
    (0,3,6) x (0,2,6), loss = <Y, G> (brute force, no library)."""
    g = synth.rng(9)
    X = synth.uniform(g, (1, 2, 6, 6)).astype(np.float64)
    Wt = synth.kaiming(g, 3, 2, 3, 3).astype(np.float64)
    lp = _plan1(3, 1, 1, 2, 3, 6, 6, [0, 3, 6], [0, 2, 6])
    G = synth.normal(g, (1, 3, 6, 6)).astype(np.float64)

    def loss(x, w):
        return float((_merged_conv(x, w, None, lp) * G).sum())

    dYp = O.split(G, lp.Oh, lp.Ow)
    dX = O.merge(O.conv_bwd_data(dYp, Wt, lp))
    dW, _ = O.conv_bwd_filter(O.split(X, lp.Ih, lp.Iw), dYp, lp)
    h = 1e-6
    for idx in np.ndindex(X.shape):
        e = np.zeros_like(X)
        e[idx] = h
        fd = (loss(X + e, Wt) - loss(X - e, Wt)) / (2 * h)
        assert abs(fd - dX[idx]) < 1e-7
    for idx in np.ndindex(Wt.shape):
        e = np.zeros_like(Wt)
        e[idx] = h
        fd = (loss(X, Wt + e) - loss(X, Wt - e)) / (2 * h)
        assert abs(fd - dW[idx]) < 1e-7


# --------------------------------------------------------------------------- max-pool
def test_pool_k_eq_s_is_natural_pin3():
    """pin-3: with k = s and even boundaries the split pool is the unsplit F.max_pool2d,
    values and indices (after the R8 mapping) bit-exact (P:128-130 + P:122)."""
    g = synth.rng(50)
    X = synth.uniform(g, (2, 3, 32, 24)).astype(np.float64)
    X = np.maximum(X, 0)                                     # ReLU output: many all-zero windows (R9 ties)
    lp = _plan1(2, 2, 0, 3, 3, 32, 24, [0, 8, 16], [0, 4, 12], op="maxpool")
    Yp, Ap = O.pool_fwd(O.split(X, lp.Ih, lp.Iw), lp)
    Y = O.merge(Yp)
    idx = O.merge([[O.argmax_to_plane_index(Ap[i][j], lp, i, j) for j in range(2)] for i in range(2)])
    ry, ri = F.max_pool2d(torch.from_numpy(X), 2, 2, return_indices=True)
    assert np.array_equal(Y, ry.numpy()) and np.array_equal(idx, ri.numpy())


def test_pool_padded_overlapping_per_patch():
    """3x3 s2 p1 (ResNet) per patch == F.max_pool2d of the -inf-padded patch (R7, R9);
    backward equals autograd of that composition (R10: overlapping windows accumulate)."""
    g = synth.rng(51)
    X = synth.uniform(g, (2, 3, 20, 18)).astype(np.float64)
    Ho, Wo = P.out_len(20, 3, 2, 1, 1), P.out_len(18, 3, 2, 1, 1)
    lp = _plan1(3, 2, 1, 3, 3, 20, 18, [0, 5, Ho], [0, 4, Wo], op="maxpool")
    xt = torch.from_numpy(X).requires_grad_()
    rows = []
    for i in range(2):
        row = []
        for j in range(2):
            xp = xt[:, :, lp.Ih[i]:lp.Ih[i + 1], lp.Iw[j]:lp.Iw[j + 1]]
            xp = F.pad(xp, (*lp.pads_w[j], *lp.pads_h[i]), value=-np.inf)
            row.append(F.max_pool2d(xp, 3, 2))
        rows.append(torch.cat(row, 3))
    ref = torch.cat(rows, 2)
    G = synth.normal(g, tuple(ref.shape)).astype(np.float64)
    (ref * torch.from_numpy(G)).sum().backward()
    Yp, Ap = O.pool_fwd(O.split(X, lp.Ih, lp.Iw), lp)
    assert np.array_equal(O.merge(Yp), ref.detach().numpy())
    dX = O.merge(O.pool_bwd(O.split(G, lp.Oh, lp.Ow), Ap, lp))
    np.testing.assert_allclose(dX, xt.grad.numpy(), rtol=1e-14, atol=1e-14)


def test_pool_tie_break_first_max_r9():
    X = np.zeros((1, 1, 2, 2))
    _, A = O.pool_fwd_patch(X, 2, 2, 2, 2, (0, 0), (0, 0))
    assert A[0, 0, 0, 0] == 0
    X = np.array([[[[1.0, 3.0], [3.0, 2.0]]]])
    _, A = O.pool_fwd_patch(X, 2, 2, 2, 2, (0, 0), (0, 0))
    assert A[0, 0, 0, 0] == 1


def test_split_merge_identity_pin8():
    g = synth.rng(52)
    X = synth.uniform(g, (2, 3, 13, 11)).astype(np.float64)
    for Ih, Iw in [([0, 13], [0, 11]), ([0, 4, 9, 13], [0, 6, 11])]:
        assert np.array_equal(O.merge(O.split(X, Ih, Iw)), X)
    assert np.array_equal(O.offload_roundtrip(X), X)
    assert np.array_equal(O.allreduce_sum([X, 2 * X]), 3 * X)


# --------------------------------------------------------------------------- ResNet split stack
def _torch_resnet(chain, blocks, X, params, x_tensor=None):
    """Unsplit BN-free ResNet stack in torch fp64 (library routines), for the 1x1-split pin."""
    import torch
    import torch.nn.functional as F
    x = torch.tensor(X, requires_grad=True) if x_tensor is None else x_tensor
    ps = [(torch.tensor(W, requires_grad=True), torch.tensor(b, requires_grad=True)) for W, b in params]
    nconv = sum(1 for l in chain if l["op"] == "conv")
    cidx = {m: i for i, m in enumerate(m for m, l in enumerate(chain) if l["op"] == "conv")}
    dsi = {k: nconv + i for i, k in enumerate(k for k, b in enumerate(blocks) if b["ds"] is not None)}
    at = {b["a"]: k for k, b in enumerate(blocks)}

    def conv(h, l, p):
        return F.conv2d(h, p[0], p[1], stride=l["sh"], padding=l["ph_b"])

    h, m = x, 0
    while m < len(chain):
        l = chain[m]
        if m in at:
            k = at[m]
            t = F.relu(conv(h, l, ps[cidx[m]]))
            z = conv(t, chain[m + 1], ps[cidx[m + 1]])
            s = conv(h, blocks[k]["ds"], ps[dsi[k]]) if k in dsi else h
            h = F.relu(z + s)
            m += 2
            continue
        if l["op"] == "conv":
            h = conv(h, l, ps[cidx[m]])
            if l.get("relu", True):
                h = F.relu(h)
        else:
            h = F.max_pool2d(h, l["kh"], l["sh"], l["ph_b"])
        m += 1
    return h, x, ps


def test_resnet_stack_1x1_split_equals_unsplit_torch():
    """pin-1 for the ResNet composition (residual joins, 1x1 s2 downsample, 3x3 s2 p1 pool):
    a 1x1 split reduces to the unsplit network; forward and all weight gradients vs torch fp64
    autograd (loss = <Y, G>)."""
    import torch
    from tests import oracle_chain
    chain, blocks = synth.resnet18_blocks(8, 16)
    g = synth.rng(7)
    N, H = 2, 32
    X = synth.uniform(g, (N, 3, H, H)).astype(np.float64)
    params = [(W.astype(np.float64), b.astype(np.float64)) for W, b in synth.resnet_params(g, chain, blocks)]
    Y, x, ps = _torch_resnet(chain, blocks, X, params)
    G = synth.normal(g, tuple(Y.shape)).astype(np.float64)
    (Y * torch.tensor(G)).sum().backward()
    out, dWs, dbs = oracle_chain.run_resnet(chain, blocks, N, 3, H, H, [0, Y.shape[2]], [0, Y.shape[3]],
                                            params, X, G)
    assert np.abs(out - Y.detach().numpy()).max() < 1e-12
    assert len(dWs) == len(ps)
    for (Wt, bt), dW, db in zip(ps, dWs, dbs):
        assert np.abs(dW - Wt.grad.numpy()).max() < 1e-10 * max(1.0, np.abs(dW).max())
        assert np.abs(db - bt.grad.numpy()).max() < 1e-10 * max(1.0, np.abs(db).max())


def test_resnet_stack_split_patch_independence_and_interior():
    """The 2x2-split ResNet stack keeps patches independent: perturbing the input of one
    patch leaves every other patch's output bitwise unchanged, and the split output differs from
    the unsplit one (Split-CNN changes the result)."""
    from tests import oracle_chain
    chain, blocks = synth.resnet18_blocks(8, 16)
    g = synth.rng(8)
    N, H = 1, 32
    X = synth.uniform(g, (N, 3, H, H)).astype(np.float64)
    params = [(W.astype(np.float64), b.astype(np.float64)) for W, b in synth.resnet_params(g, chain, blocks)]
    G = np.zeros((N, 16, 4, 4))
    O2 = [0, 2, 4]
    out, _, _ = oracle_chain.run_resnet(chain, blocks, N, 3, H, H, O2, O2, params, X, G)
    X2 = X.copy()
    X2[:, :, :16, :16] += 0.5          # patch (0, 0) at the input (I = 8 * O at the input level)
    out2, _, _ = oracle_chain.run_resnet(chain, blocks, N, 3, H, H, O2, O2, params, X2, G)
    assert not np.array_equal(out[:, :, :2, :2], out2[:, :, :2, :2])
    assert np.array_equal(out[:, :, 2:, :], out2[:, :, 2:, :])
    assert np.array_equal(out[:, :, :, 2:], out2[:, :, :, 2:])
    full, _, _ = oracle_chain.run_resnet(chain, blocks, N, 3, H, H, [0, 4], [0, 4], params, X, G)
    assert not np.allclose(full, out)


def _torch_resnet_bn(chain, blocks, X, params, bn, eps=1e-5):
    import torch
    import torch.nn.functional as F
    x = torch.tensor(X, requires_grad=True)
    ws = [torch.tensor(W, requires_grad=True) for W, _ in params]
    bns = [(torch.tensor(gm, requires_grad=True), torch.tensor(bt, requires_grad=True)) for gm, bt in bn]
    conv_ms = [m for m, l in enumerate(chain) if l["op"] == "conv"]
    ci = {m: i for i, m in enumerate(conv_ms)}
    dsi = {k: len(conv_ms) + i for i, k in enumerate(k for k, b in enumerate(blocks) if b["ds"] is not None)}
    at = {b["a"]: k for k, b in enumerate(blocks)}

    def cbn(h, l, i, relu):
        z = F.conv2d(h, ws[i], None, stride=l["sh"], padding=l["ph_b"])
        y = F.batch_norm(z, None, None, bns[i][0], bns[i][1], training=True, eps=eps)
        return F.relu(y) if relu else y

    h, m = x, 0
    while m < len(chain):
        l = chain[m]
        if m in at:
            k = at[m]
            t = cbn(h, l, ci[m], True)
            zb = cbn(t, chain[m + 1], ci[m + 1], False)
            s = cbn(h, blocks[k]["ds"], dsi[k], False) if k in dsi else h
            h = F.relu(zb + s)
            m += 2
            continue
        h = cbn(h, l, ci[m], True) if l["op"] == "conv" else F.max_pool2d(h, l["kh"], l["sh"], l["ph_b"])
        m += 1
    return h, ws, bns


def test_resnet_bn_stack_1x1_split_equals_unsplit_torch():
    """pin-1 for the BN ResNet composition (R11: BN statistics over the logical tensor): a 1x1 split
    reduces to the unsplit network with training-mode F.batch_norm; forward, every dW, dgamma, dbeta
    vs torch fp64 autograd."""
    import torch
    from tests import oracle_chain
    chain, blocks = synth.resnet18_blocks(8, 16)
    g = synth.rng(9)
    N, H = 2, 32
    X = synth.uniform(g, (N, 3, H, H)).astype(np.float64)
    params = [(W.astype(np.float64), b.astype(np.float64)) for W, b in synth.resnet_params(g, chain, blocks)]
    chans = [W.shape[0] for W, _ in params]
    bn = [(gm.astype(np.float64), bt.astype(np.float64)) for gm, bt in synth.bn_params(g, chans)]
    Y, ws, bns = _torch_resnet_bn(chain, blocks, X, params, bn)
    G = synth.normal(g, tuple(Y.shape)).astype(np.float64)
    (Y * torch.tensor(G)).sum().backward()
    out, dWs, dgs, dbs = oracle_chain.run_resnet_bn(chain, blocks, N, 3, H, H, [0, Y.shape[2]], [0, Y.shape[3]],
                                                    params, bn, X, G)
    assert np.abs(out - Y.detach().numpy()).max() < 1e-11
    for w, dW in zip(ws, dWs):
        assert np.abs(dW - w.grad.numpy()).max() < 1e-9 * max(1.0, np.abs(dW).max())
    for (gm, bt), dg, db in zip(bns, dgs, dbs):
        assert np.abs(dg - gm.grad.numpy()).max() < 1e-9 * max(1.0, np.abs(dg).max())
        assert np.abs(db - bt.grad.numpy()).max() < 1e-9 * max(1.0, np.abs(db).max())


def test_batch_norm_split_invariant():
    """R11: whole-tensor BN on patches equals BN of the merged tensor cut the same way (a split never
    changes BN, unlike the window ops), for uneven patches."""
    g = synth.rng(10)
    X = synth.normal(g, (2, 5, 9, 7)).astype(np.float64)
    gm, bt = synth.uniform(g, (5,), 0.5, 1.5).astype(np.float64), synth.uniform(g, (5,), -0.1, 0.1).astype(np.float64)
    P1, _, _ = O.batch_norm(O.split(X, [0, 9], [0, 7]), gm, bt, relu=True)
    P2, _, _ = O.batch_norm(O.split(X, [0, 2, 9], [0, 4, 5, 7]), gm, bt, relu=True)
    assert np.array_equal(O.merge(P1), O.merge(P2))


def test_resnet18_full_trunk_1x1_split_equals_unsplit_torch():
    """pin-1 for the whole trunk oracle (split region -> merge -> unsplit tail -> global average pool):
    with a 1x1 region split it is the unsplit BN-free ResNet-18 trunk; pooled output and every weight /
    bias gradient vs torch fp64 autograd."""
    import torch
    from tests import oracle_chain
    rc, rb = synth.resnet18_blocks(8, 16)
    tc, tb = synth.resnet18_tail_blocks(16, 16, 32)
    g = synth.rng(12)
    N, H = 2, 64
    X = synth.uniform(g, (N, 3, H, H)).astype(np.float64)
    p_r = [(W.astype(np.float64), b.astype(np.float64)) for W, b in synth.resnet_params(g, rc, rb)]
    p_t = [(W.astype(np.float64), b.astype(np.float64)) for W, b in synth.resnet_params(g, tc, tb)]
    Yr, x, ps_r = _torch_resnet(rc, rb, X, p_r)
    # the tail on the region output, then the global average pool
    Yt, _, ps_t = _torch_resnet(tc, tb, None, p_t, x_tensor=Yr)
    pooled = Yt.mean(dim=(2, 3))
    G = synth.normal(g, tuple(pooled.shape)).astype(np.float64)
    (pooled * torch.tensor(G)).sum().backward()
    out, dWs, dbs = oracle_chain.run_resnet18_full(rc, rb, tc, tb, N, 3, H, H, [0, Yr.shape[2]], [0, Yr.shape[3]],
                                                   p_r + p_t, X, G)
    assert np.abs(out - pooled.detach().numpy()).max() < 1e-12
    for (Wt, bt), dW, db in zip(ps_r + ps_t, dWs, dbs):
        assert np.abs(dW - Wt.grad.numpy()).max() < 1e-10 * max(1.0, np.abs(dW).max())
        assert np.abs(db - bt.grad.numpy()).max() < 1e-10 * max(1.0, np.abs(db).max())
