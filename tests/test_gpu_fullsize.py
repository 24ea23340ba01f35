"""Parity at BASELINE.json's full size, in the launch configuration bench.py times:
C5's conv1_2 -> pool1 (N=256, 64 channels, 224x224, 8x8 split) through the same calls the executor
makes (conv_pool_fwd, bwd_data with the ReLU mask, bwd_filter with db).  Image n of the batch is
S[n,0] B0 + S[n,1] B1 -- the seeded base image split into its two checkerboard pixel classes, with a
distinct pair of exact scales per image (all 256 images differ; _Batch), and dY likewise, so
  * forward / data gradient are checked on sampled (image, patch) pairs against the oracle one by one;
  * the weight gradient, a sum over all 256 images and 64 patches, is bilinear in (X, dY), so it equals
    sum_{k,l} (sum_n S_x[n,k] S_g[n,l]) dW(Bx_k, Bg_l): four single-image oracle weight gradients."""
import numpy as np
import pytest

import synth
from oracle import ops as O
from oracle import plan as OP
from tests.helpers import normwise

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

N, C, H = 256, 64, 224


@pytest.fixture(scope="module")
def sc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_asplos_jinh19_b200 import splitcnn
    return splitcnn


_TABLE = np.array([m * 2.0 ** -e for e in range(4) for m in (1.0, 1.25, 1.5, 1.75)])   # 16 scales, 3-bit mantissas


def _round5(a):
    """Keep 5 significant bits (a seeded draw rounded to bf16, low 3 mantissa bits cleared), so a 5-bit
    value times a 3-bit scale is exact in bf16."""
    u = synth.to_bf16_f32(np.asarray(a, dtype=np.float32)).view(np.uint32) & np.uint32(0xFFF8FFFF)
    return u.view(np.float32).astype(np.float64)


class _Batch:
    """N DISTINCT images: image n = S[n,0] * B0 + S[n,1] * B1 with B0 / B1 the base image on the two
    checkerboard pixel classes (disjoint supports, so every image is exact in bf16) and (S[n,0], S[n,1])
    = two base-16 digits of n through _TABLE -- no two of the 256 images are equal, so an image-offset
    bug is visible.  swap=True reverses the digits (the dY batch)."""

    def __init__(self, base, swap=False):
        b = _round5(base)
        h, w = b.shape[1:]
        m = ((np.arange(h)[:, None] + np.arange(w)[None, :]) % 2 == 0)[None]
        self.B = [b * m, b * ~m]
        n = np.arange(N)
        d0, d1 = (n // 16, n % 16) if swap else (n % 16, n // 16)
        self.S = np.stack([_TABLE[d0], _TABLE[d1]], 1)

    def img(self, n):
        return self.S[n, 0] * self.B[0] + self.S[n, 1] * self.B[1]

    def patch(self, n, hs, ws):
        return self.img(n)[:, hs[0]:hs[1], ws[0]:ws[1]][None]


def _bilinear(xb, gb, fn):
    """sum_n fn(X_n, G_n) for fn bilinear: sum over (k, l) of (sum_n S_x[n,k] S_g[n,l]) fn(Bx_k, Bg_l)."""
    out = None
    for k in range(2):
        for l in range(2):
            c = float(np.sum(xb.S[:, k] * gb.S[:, l]))
            v = c * fn(xb.B[k][None], gb.B[l][None])
            out = v if out is None else out + v
    return out


def _fill_level(lv, batch, device="cuda"):
    """Level buffer (bf16) of the batch's N images, patch-major NHWC (layout glue)."""
    Cp, W = lv["Cpad"], lv["W"]
    buf = torch.zeros(lv["total_elems"], dtype=torch.bfloat16, device=device)
    S = torch.from_numpy(batch.S.astype(np.float32)).to(device)
    bh, bw = lv["bh"], lv["bw"]
    C = batch.B[0].shape[0]
    for i in range(lv["n_h"]):
        hp = bh[i + 1] - bh[i]
        for j in range(lv["n_w"]):
            wp = bw[j + 1] - bw[j]
            off = N * Cp * (bh[i] * W + hp * bw[j])
            blk = torch.zeros((2, hp, wp, Cp), dtype=torch.float32, device=device)
            for k in range(2):
                blk[k, ..., :C] = torch.from_numpy(np.ascontiguousarray(
                    batch.B[k][:, bh[i]:bh[i + 1], bw[j]:bw[j + 1]].transpose(1, 2, 0))).to(device)
            imgs = S[:, 0, None, None, None] * blk[0][None] + S[:, 1, None, None, None] * blk[1][None]
            buf[off:off + N * hp * wp * Cp] = imgs.reshape(-1).to(torch.bfloat16)
    return buf


def _patch(buf, lv, i, j, n):
    Cp, W = lv["Cpad"], lv["W"]
    bh, bw = lv["bh"], lv["bw"]
    hp, wp = bh[i + 1] - bh[i], bw[j + 1] - bw[j]
    off = N * Cp * (bh[i] * W + hp * bw[j]) + n * hp * wp * Cp
    return buf[off:off + hp * wp * Cp].float().cpu().numpy().reshape(hp, wp, Cp).transpose(2, 0, 1)[None].astype(np.float64)


def test_c5_conv1_2_full_size(sc):
    from paper_conf_asplos_jinh19_b200.net import pack_weight
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    layers = [synth.conv(C, C, name="conv1_2"), synth.maxpool(C, name="pool1")]
    Ob = sc.splitcnn_boundaries_even(112, 8)
    pl = SplitPlan(layers, N, C, H, H, Ob, Ob)
    assert sc.splitcnn_conv_pool_supported(pl.handle, 0, sc.BF16)
    lv0, lv1, lv2 = pl.levels
    ref = OP.plan(layers, 1, C, H, H, Ob, Ob)
    g = synth.rng(44)
    base = synth.to_bf16_f32(synth.uniform(g, (C, H, H))).astype(np.float64)
    Wt = synth.to_bf16_f32(synth.kaiming(g, C, C, 3, 3)).astype(np.float64)
    b = synth.uniform(g, (C,), -0.1, 0.1).astype(np.float64)
    gbase = synth.to_bf16_f32(synth.normal(g, (C, H, H))).astype(np.float64)
    xb, gbt = _Batch(base), _Batch(gbase, swap=True)   # positive scales: sum S_x S_g far from 0
    x = _fill_level(lv0, xb)
    dy = _fill_level(lv1, gbt)
    w = pack_weight(torch.from_numpy(Wt), lv0["Cpad"], torch.bfloat16).cuda().contiguous()
    bias = torch.from_numpy(b.astype(np.float32)).cuda()
    yp = torch.empty(lv2["total_elems"], dtype=torch.bfloat16, device="cuda")
    am = torch.empty(lv2["total_elems"], dtype=torch.uint8, device="cuda")
    sc.splitcnn_conv_pool_fwd(pl.handle, 0, sc.BF16, x, w, bias, yp, am)
    ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dx = torch.empty_like(x)
    sc.splitcnn_conv_bwd_data(pl.handle, 0, sc.BF16, dy, w, dx, x, ws, ws_b)
    dw = torch.zeros((C, 3, 3, lv0["Cpad"]), dtype=torch.float32, device="cuda")
    db = torch.zeros(C, dtype=torch.float32, device="cuda")
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, dy, dw, db, 0.0, ws, ws_b)
    torch.cuda.synchronize()
    lp0, lp1 = ref.layers
    for n, i, j in ((0, 0, 0), (137, 3, 5), (255, 7, 7), (64, 7, 0)):
        X = xb.patch(n, lp0.Ih[i:i + 2], lp0.Iw[j:j + 2])
        Y = O.conv_fwd_patch(X, Wt, b, 1, 1, lp0.pads_h[i], lp0.pads_w[j], relu=True)
        Yb = synth.to_bf16_f32(Y.astype(np.float32)).astype(np.float64)   # the GPU pools the bf16 conv outputs
        P, A = O.pool_fwd_patch(Yb, 2, 2, 2, 2, lp1.pads_h[i], lp1.pads_w[j])
        got = _patch(yp, lv2, i, j, n)[:, :C]
        assert normwise(got, P) <= 2e-2, (n, i, j)
        Ag = _patch(am, lv2, i, j, n)[:, :C].astype(np.int64) & 0x7F
        assert np.mean(Ag != A) < 1e-2, (n, i, j)           # equal up to bf16 near-ties (R9, R13)
        G = gbt.patch(n, lp0.Ih[i:i + 2], lp0.Iw[j:j + 2])
        dX = O.conv_bwd_data_patch(G, Wt, X.shape[2], X.shape[3], 1, 1, lp0.pads_h[i], lp0.pads_w[j], mask=X)
        assert normwise(_patch(dx, lv0, i, j, n)[:, :C], dX) <= 2e-2, (n, i, j)
    # weight / bias gradient over all 256 images and 64 patches, by linearity in the per-image scales
    dW_ref = _bilinear(xb, gbt, lambda X1, G1: O.conv_bwd_filter(O.split(X1, lp0.Ih, lp0.Iw),
                                                                 O.split(G1, lp0.Ih, lp0.Iw), lp0)[0])
    db_ref = sum(float(np.sum(gbt.S[:, l])) * O.conv_bwd_filter(O.split(xb.B[0][None], lp0.Ih, lp0.Iw),
                                                               O.split(gbt.B[l][None], lp0.Ih, lp0.Iw), lp0)[1]
                 for l in range(2))
    dWg = dw[..., :C].permute(0, 3, 1, 2).double().cpu().numpy()
    assert normwise(dWg, dW_ref) <= 2e-2
    assert normwise(db.double().cpu().numpy(), db_ref) <= 2e-2


@pytest.mark.parametrize("name,Cin,Cout,Hin,nsplit", [
    ("conv1_1", 3, 64, 224, 8),      # 8-channel padded input: halo8 forward, narrow wgrad
    ("conv2_1", 64, 128, 112, 8),    # 64 -> 128 channels, 14x14 patches
    ("conv3_1", 128, 256, 56, 8),    # 128 -> 256 channels, 7x7 patches
    ("conv3_2", 256, 256, 56, 8),
    ("conv4_2", 512, 512, 28, 1),
    ("conv5_2", 512, 512, 14, 1),    # the smallest tail layer (few tiles per SM)
])
def test_c5_deep_layers_full_size(sc, name, Cin, Cout, Hin, nsplit):
    """C5's split-region layers (conv1_1 on the 3->8 padded input, conv2_1, conv3_1, conv3_2 with 2-CTA
    halo kernels) and unsplit tail layers (conv4_2, conv5_2) at N=256: conv_fwd (+bias+ReLU), bwd_data
    (ReLU mask), bwd_filter (+db) as the executor calls them (the executor skips conv1_1's bwd_data;
    it is checked anyway)."""
    from paper_conf_asplos_jinh19_b200.net import pack_weight
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    l = synth.conv(Cin, Cout, name=name)
    Ob = sc.splitcnn_boundaries_even(Hin, nsplit)
    pl = SplitPlan([l], N, Cin, Hin, Hin, Ob, Ob)
    lv0, lv1 = pl.levels
    lp = OP.plan([l], 1, Cin, Hin, Hin, Ob, Ob).layers[0]
    g = synth.rng(45 + Cin)
    base = synth.to_bf16_f32(synth.uniform(g, (Cin, Hin, Hin))).astype(np.float64)
    Wt = synth.to_bf16_f32(synth.kaiming(g, Cout, Cin, 3, 3)).astype(np.float64)
    b = synth.uniform(g, (Cout,), -0.1, 0.1).astype(np.float64)
    gbase = synth.to_bf16_f32(synth.normal(g, (Cout, Hin, Hin))).astype(np.float64)
    xb, gbt = _Batch(base), _Batch(gbase, swap=True)
    x = _fill_level(lv0, xb)
    dy = _fill_level(lv1, gbt)
    w = pack_weight(torch.from_numpy(Wt), lv0["Cpad"], torch.bfloat16).cuda().contiguous()
    bias = torch.from_numpy(b.astype(np.float32)).cuda()
    y = torch.empty(lv1["total_elems"], dtype=torch.bfloat16, device="cuda")
    sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, bias, y, sc.FLAG_RELU)
    ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dx = torch.empty_like(x)
    sc.splitcnn_conv_bwd_data(pl.handle, 0, sc.BF16, dy, w, dx, x, ws, ws_b)
    dw = torch.zeros((Cout, 3, 3, lv0["Cpad"]), dtype=torch.float32, device="cuda")
    db = torch.zeros(Cout, dtype=torch.float32, device="cuda")
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, dy, dw, db, 0.0, ws, ws_b)
    torch.cuda.synchronize()
    last = nsplit - 1
    for n, i, j in ((3, 0, 0), (200, last, last), (129, last // 2, 0)):
        X = xb.patch(n, lp.Ih[i:i + 2], lp.Iw[j:j + 2])
        Y = O.conv_fwd_patch(X, Wt, b, 1, 1, lp.pads_h[i], lp.pads_w[j], relu=True)
        assert normwise(_patch(y, lv1, i, j, n)[:, :Cout], Y) <= 2e-2, (n, i, j)
        G = gbt.patch(n, lp.Oh[i:i + 2], lp.Ow[j:j + 2])
        dX = O.conv_bwd_data_patch(G, Wt, X.shape[2], X.shape[3], 1, 1, lp.pads_h[i], lp.pads_w[j], mask=X)
        assert normwise(_patch(dx, lv0, i, j, n)[:, :Cin], dX) <= 2e-2, (n, i, j)
    wg = lambda X1, G1: O.conv_bwd_filter(O.split(X1, lp.Ih, lp.Iw), O.split(G1, lp.Oh, lp.Ow), lp)
    dW_ref = _bilinear(xb, gbt, lambda X1, G1: wg(X1, G1)[0])
    db_ref = sum(float(np.sum(gbt.S[:, l])) * wg(xb.B[0][None], gbt.B[l][None])[1] for l in range(2))
    dWg = dw[..., :Cin].permute(0, 3, 1, 2).double().cpu().numpy()
    assert normwise(dWg, dW_ref) <= 2e-2
    assert normwise(db.double().cpu().numpy(), db_ref) <= 2e-2


def test_c3_stride2_and_stem_full_size(sc):
    """C3 at N=256: layer2_0_a (3x3 s2, 64->128, 56->28, 2x2 split; phase-decomposed tcgen05 dgrad) and
    the stem (7x7 s2 on 3 channels run as the space-to-depth 4x4 s1 conv: NCHW_S2D split + conv), same
    sampled-pair / linearity checks against the oracle's own 7x7 s2 / 3x3 s2 definitions."""
    from paper_conf_asplos_jinh19_b200.net import pack_weight
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    from paper_conf_asplos_jinh19_b200.resnet import s2d_stem_grad, s2d_stem_layer, s2d_stem_weight
    g = synth.rng(46)
    # ---- layer2_0_a: 3x3 s2 p1, 64 -> 128
    l = synth.conv(64, 128, s=2, name="layer2_0_a")
    Ob = sc.splitcnn_boundaries_even(28, 2)
    pl = SplitPlan([l], N, 64, 56, 56, Ob, Ob)
    lv0, lv1 = pl.levels
    lp = OP.plan([l], 1, 64, 56, 56, Ob, Ob).layers[0]
    base = synth.to_bf16_f32(synth.uniform(g, (64, 56, 56))).astype(np.float64)
    Wt = synth.to_bf16_f32(synth.kaiming(g, 128, 64, 3, 3)).astype(np.float64)
    gbase = synth.to_bf16_f32(synth.normal(g, (128, 28, 28))).astype(np.float64)
    xb, gbt = _Batch(base), _Batch(gbase, swap=True)
    x, dy = _fill_level(lv0, xb), _fill_level(lv1, gbt)
    w = pack_weight(torch.from_numpy(Wt), lv0["Cpad"], torch.bfloat16).cuda().contiguous()
    y = torch.empty(lv1["total_elems"], dtype=torch.bfloat16, device="cuda")
    sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, None, y, sc.FLAG_RELU)
    ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dx = torch.empty_like(x)
    sc.splitcnn_conv_bwd_data(pl.handle, 0, sc.BF16, dy, w, dx, x, ws, ws_b)
    dw = torch.zeros((128, 3, 3, lv0["Cpad"]), dtype=torch.float32, device="cuda")
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, dy, dw, None, 0.0, ws, ws_b)
    torch.cuda.synchronize()
    for n, i, j in ((5, 0, 1), (250, 1, 1)):
        X = xb.patch(n, lp.Ih[i:i + 2], lp.Iw[j:j + 2])
        Y = O.conv_fwd_patch(X, Wt, None, 2, 2, lp.pads_h[i], lp.pads_w[j], relu=True)
        assert normwise(_patch(y, lv1, i, j, n)[:, :128], Y) <= 2e-2, (n, i, j)
        G = gbt.patch(n, lp.Oh[i:i + 2], lp.Ow[j:j + 2])
        dX = O.conv_bwd_data_patch(G, Wt, X.shape[2], X.shape[3], 2, 2, lp.pads_h[i], lp.pads_w[j], mask=X)
        assert normwise(_patch(dx, lv0, i, j, n)[:, :64], dX) <= 2e-2, (n, i, j)
    dW_ref = _bilinear(xb, gbt, lambda X1, G1: O.conv_bwd_filter(O.split(X1, lp.Ih, lp.Iw),
                                                                 O.split(G1, lp.Oh, lp.Ow), lp)[0])
    assert normwise(dw[..., :64].permute(0, 3, 1, 2).double().cpu().numpy(), dW_ref) <= 2e-2
    # ---- the stem: 7x7 s2 p3 on 3 channels through the space-to-depth split and 4x4 s1 conv
    l7 = synth.conv(3, 64, k=7, s=2, p=3, name="conv1")
    Ob = sc.splitcnn_boundaries_even(112, 2)
    ls = s2d_stem_layer(l7)
    pls = SplitPlan([ls], N, 12, 112, 112, Ob, Ob)
    lvs0, lvs1 = pls.levels
    lp7 = OP.plan([l7], 1, 3, H, H, Ob, Ob).layers[0]
    img = synth.to_bf16_f32(synth.uniform(g, (3, H, H))).astype(np.float64)
    W7 = synth.to_bf16_f32(synth.kaiming(g, 64, 3, 7, 7)).astype(np.float64)
    gst = synth.to_bf16_f32(synth.normal(g, (64, 112, 112))).astype(np.float64)
    ib, gsb = _Batch(img), _Batch(gst, swap=True)
    Sd = torch.from_numpy(ib.S.astype(np.float32)).cuda()
    Bd = [torch.from_numpy(B.astype(np.float32)).cuda() for B in ib.B]
    xf = (Sd[:, 0, None, None, None] * Bd[0][None] + Sd[:, 1, None, None, None] * Bd[1][None]).to(torch.bfloat16)
    xs = torch.empty(lvs0["total_elems"], dtype=torch.bfloat16, device="cuda")
    sc.splitcnn_split(pls.handle, 0, sc.BF16, xf, sc.NCHW_S2D, xs)
    ws7 = pack_weight(s2d_stem_weight(torch.from_numpy(W7)), lvs0["Cpad"], torch.bfloat16).cuda().contiguous()
    ys = torch.empty(lvs1["total_elems"], dtype=torch.bfloat16, device="cuda")
    sc.splitcnn_conv_fwd(pls.handle, 0, sc.BF16, xs, ws7, None, ys, sc.FLAG_RELU)
    dys = _fill_level(lvs1, gsb)
    wsb = max(pls.workspace_size(0, sc.BF16, 2), 16)
    wss = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    dws = torch.zeros((64, 4, 4, lvs0["Cpad"]), dtype=torch.float32, device="cuda")
    sc.splitcnn_conv_bwd_filter(pls.handle, 0, sc.BF16, xs, dys, dws, None, 0.0, wss, wsb)
    torch.cuda.synchronize()
    for n, i, j in ((1, 0, 0), (254, 1, 0)):
        X = ib.patch(n, lp7.Ih[i:i + 2], lp7.Iw[j:j + 2])
        Y = O.conv_fwd_patch(X, W7, None, 2, 2, lp7.pads_h[i], lp7.pads_w[j], relu=True)
        assert normwise(_patch(ys, lvs1, i, j, n)[:, :64], Y) <= 2e-2, (n, i, j)
    dW7 = _bilinear(ib, gsb, lambda X1, G1: O.conv_bwd_filter(O.split(X1, lp7.Ih, lp7.Iw),
                                                              O.split(G1, lp7.Oh, lp7.Ow), lp7)[0])
    assert normwise(s2d_stem_grad(dws, 3).double().cpu().numpy(), dW7) <= 2e-2


def test_c5_split_merge_pool_full_size(sc):
    """Bit-exact HBM ops at full size: the C5 input split / merge round trip (N=256, 3x224x224, 8x8,
    NCHW), and the standalone 2x2 pool (pool2 geometry: N=256, 128 channels, 112x112, 8x8) forward
    values + argmax and backward on sampled (image, patch) pairs against the oracle."""
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    Ob = sc.splitcnn_boundaries_even(224, 8)
    pl = SplitPlan([synth.conv(3, 64)], N, 3, H, H, Ob, Ob)
    gen = torch.Generator(device="cpu").manual_seed(47)
    x = (torch.rand((N, 3, H, H), generator=gen) * 2 - 1).to("cuda", torch.bfloat16)
    p = torch.empty(pl.levels[0]["total_elems"], dtype=torch.bfloat16, device="cuda")
    sc.splitcnn_split(pl.handle, 0, sc.BF16, x, sc.NCHW, p)
    back = torch.empty_like(x)
    sc.splitcnn_merge(pl.handle, 0, sc.BF16, p, back, sc.NCHW)
    torch.cuda.synchronize()
    assert torch.equal(back, x)
    # 2x2 pool at pool2's geometry
    lpool = synth.maxpool(128)
    Op = sc.splitcnn_boundaries_even(56, 8)
    pp = SplitPlan([lpool], N, 128, 112, 112, Op, Op)
    lv0, lv1 = pp.levels
    lref = OP.plan([lpool], 1, 128, 112, 112, Op, Op).layers[0]
    g = synth.rng(48)
    base = synth.to_bf16_f32(synth.normal(g, (128, 112, 112))).astype(np.float64)
    gb = synth.to_bf16_f32(synth.normal(g, (128, 56, 56))).astype(np.float64)
    xb, gbt = _Batch(base), _Batch(gb, swap=True)
    xin, dy = _fill_level(lv0, xb), _fill_level(lv1, gbt)
    y = torch.empty(lv1["total_elems"], dtype=torch.bfloat16, device="cuda")
    a = torch.empty(lv1["total_elems"], dtype=torch.uint8, device="cuda")
    sc.splitcnn_pool_fwd(pp.handle, 0, sc.BF16, xin, y, a, 0)
    dx = torch.empty_like(xin)
    sc.splitcnn_pool_bwd(pp.handle, 0, sc.BF16, dy, a, dx, 0)
    torch.cuda.synchronize()
    for n, i, j in ((0, 0, 0), (255, 7, 7), (77, 2, 5)):
        X = xb.patch(n, lref.Ih[i:i + 2], lref.Iw[j:j + 2])
        Y, A = O.pool_fwd_patch(X, 2, 2, 2, 2, lref.pads_h[i], lref.pads_w[j])
        assert np.array_equal(_patch(y, lv1, i, j, n)[:, :128], Y), (n, i, j)
        assert np.array_equal(_patch(a, lv1, i, j, n)[:, :128].astype(np.int64) & 0x7F, A), (n, i, j)
        G = gbt.patch(n, lref.Oh[i:i + 2], lref.Ow[j:j + 2])
        dX = O.pool_bwd_patch(G, A, X.shape[2], X.shape[3], 2, 2, 2, 2, lref.pads_h[i], lref.pads_w[j])
        assert np.array_equal(_patch(dx, lv0, i, j, n)[:, :128], dX), (n, i, j)


@pytest.mark.parametrize("dtype_name,N_,C_,H_", [
    ("fp32", 64, 64, 64),     # 67 MB fp32 dY: warp colsum (8 channel groups) + row fold
    ("bf16", 32, 256, 56),    # 51 MB bf16 dY, 32 channel groups: warp colsum, one row per pixel lane
    ("bf16", 8, 64, 56),      # 3.2 MB: below the 32 MB cut, shared-memory colsum
])
def test_db_column_sums_both_kernels(sc, dtype_name, N_, C_, H_):
    """a5's bias gradient db[co] = sum over n, h, w of dY (P:153 adjoint) through
    splitcnn_conv_bwd_filter, at sizes that select each colsum kernel; beta = 1 accumulates.  The
    expected value is that sum taken in fp64 on the host over the same (rounded) dY."""
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    dtype = sc.BF16 if dtype_name == "bf16" else sc.FP32
    tdt = torch.bfloat16 if dtype == sc.BF16 else torch.float32
    l = synth.conv(C_, C_, name="db")
    Ob = sc.splitcnn_boundaries_even(H_, 2)
    pl = SplitPlan([l], N_, C_, H_, H_, Ob, Ob)
    lv0, lv1 = pl.levels
    g = torch.Generator().manual_seed(77 + C_)
    x = torch.randn(lv0["total_elems"], generator=g).to(tdt).cuda()
    dyh = (torch.randn(lv1["total_elems"], generator=g) + 0.25).to(tdt)
    dy = dyh.cuda()
    ws_b = pl.workspace_size(0, dtype, 2)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dw = torch.zeros((C_, 3, 3, lv0["Cpad"]), dtype=torch.float32, device="cuda")
    db = torch.full((C_,), 5.0, dtype=torch.float32, device="cuda")
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, dy, dw, db, 0.0, ws, ws_b)
    torch.cuda.synchronize()
    ref = dyh.double().numpy().reshape(-1, lv1["Cpad"])[:, :C_].sum(axis=0)
    assert normwise(db.double().cpu().numpy(), ref) <= 1e-5
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, dy, dw, db, 1.0, ws, ws_b)
    torch.cuda.synchronize()
    assert normwise(db.double().cpu().numpy(), 2 * ref) <= 1e-5
