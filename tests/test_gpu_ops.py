"""GPU parity of every split operator against the CPU oracle, through the C ABI.

Bars (BASELINE.json north_star): plan / boundaries / split / merge / pool values /
argmax / k=s pool backward / offload BIT-EXACT; conv fwd / dgrad / wgrad normwise
||y - y*||_inf / ||y*||_inf <= 1e-4 for FP32 (FFMA) and <= 2e-2 for BF16 inputs with fp32
accumulation.  The oracle accumulates in fp64 on the exact (bf16-rounded) inputs the GPU sees.
"""
import numpy as np
import pytest

import synth
from oracle import ops as O
from oracle import plan as OP
from tests.helpers import normwise, pack_level, unpack_level, w_lib_to_oihw, w_oihw_to_lib

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = {0: 2e-2, 1: 1e-4, 2: 2e-3}   # BF16, FP32 (3xTF32 / FFMA), TF32 (R13: plain TF32 cannot meet 1e-4)


@pytest.fixture(scope="module")
def sc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_asplos_jinh19_b200 import splitcnn
    return splitcnn


def _td(sc, dtype):
    return torch.bfloat16 if dtype == sc.BF16 else torch.float32


def _dev(sc, a, dtype):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to("cuda", _td(sc, dtype))


def _host(t):
    return t.float().cpu().numpy().astype(np.float64)


def _round(a, dtype, sc):
    return synth.to_bf16_f32(a).astype(np.float64) if dtype == sc.BF16 else a.astype(np.float32).astype(np.float64)


def _make(sc, layers, N, C, H, W, nh, nw, seed):
    L_h, L_w = H, W
    for l in layers:
        L_h = OP.out_len(L_h, l["kh"], l["sh"], l["ph_b"], l["ph_e"])
        L_w = OP.out_len(L_w, l["kw"], l["sw"], l["pw_b"], l["pw_e"])
    Oh, Ow = OP.boundaries_random(L_h, nh, L_w, nw, 0.3, seed, 0)
    ref = OP.plan(layers, N, C, H, W, Oh, Ow)
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    return ref, SplitPlan(layers, N, C, H, W, Oh, Ow)


# (name, N, cin, cout, k, s, p, H, W, nh, nw, relu)
CONV_CASES = [
    ("C1", 2, 16, 16, 3, 1, 1, 32, 32, 2, 2, False),
    ("ragged", 3, 13, 24, 3, 1, 1, 19, 23, 3, 2, True),
    ("conv1_7x7s2", 2, 3, 16, 7, 2, 3, 30, 26, 2, 2, True),
    ("3x3s2", 2, 16, 32, 3, 2, 1, 20, 18, 2, 3, True),
    ("1x1s2_k<s", 2, 16, 32, 1, 2, 0, 14, 12, 2, 2, False),
    ("vgg64", 4, 64, 64, 3, 1, 1, 32, 32, 2, 2, True),
    ("vgg_first", 2, 3, 64, 3, 1, 1, 32, 28, 2, 2, True),
    ("vgg128_256", 2, 128, 256, 3, 1, 1, 16, 16, 3, 3, True),
    ("c5_7x7patch", 2, 256, 256, 3, 1, 1, 28, 28, 4, 4, True),
    ("wg_c16", 2, 16, 64, 3, 1, 1, 20, 20, 2, 2, True),
    ("wg_c32", 2, 32, 128, 3, 1, 1, 18, 22, 2, 3, True),
    ("s2_c64", 2, 64, 128, 3, 2, 1, 28, 28, 2, 2, True),
    ("7x7s2_c3_64", 2, 3, 64, 7, 2, 3, 30, 30, 2, 2, True),
    ("c512", 1, 512, 512, 3, 1, 1, 14, 14, 2, 2, True),
    ("halo_odd_n", 3, 64, 64, 3, 1, 1, 14, 14, 2, 2, True),
    ("halo_uneven", 2, 128, 128, 3, 1, 1, 23, 19, 3, 2, True),
    ("cta2_ragged", 3, 64, 256, 3, 1, 1, 21, 19, 3, 2, True),    # 2-CTA fwd + wgrad, odd M-box count
    ("groups_81", 1, 64, 128, 3, 1, 1, 38, 36, 9, 9, True),      # > 64 patches: two launches per pass
    ("narrow_groups_81", 1, 3, 64, 3, 1, 1, 38, 36, 9, 9, True),
]


@pytest.mark.parametrize("case", CONV_CASES, ids=[c[0] for c in CONV_CASES])
@pytest.mark.parametrize("mode", ["fp32", "fp32_simt", "tf32", "bf16_tc", "bf16_simt"])
def test_conv_parity(sc, case, mode):
    """Forward, data gradient (ReLU mask) and weight gradient (+db, beta, determinism) of one split conv
    against the oracle, per precision: fp32 = 3xTF32 forward / data gradient + 3-way bf16-split weight
    gradient on the tensor cores (FFMA where the shape does not fit), fp32_simt = FFMA throughout, tf32 =
    one kind::tf32 pass + 2-way bf16-split weight gradient, bf16 on tcgen05 or forced onto FFMA."""
    name, N, cin, cout, k, s, p, H, W, nh, nw, relu = case
    dtype = {"fp32": sc.FP32, "fp32_simt": sc.FP32, "tf32": sc.TF32}.get(mode, sc.BF16)
    extra = sc.FLAG_FORCE_SIMT if mode.endswith("_simt") else 0
    layers = [synth.conv(cin, cout, k, s, p, relu=relu)]
    ref, pl = _make(sc, layers, N, cin, H, W, nh, nw, seed=sum(map(ord, name)))
    lp = ref.layers[0]
    lv0, lv1 = pl.levels
    g = synth.rng(100 + len(name))
    X = _round(synth.uniform(g, (N, cin, H, W)), dtype, sc)
    Wt = _round(synth.kaiming(g, cout, cin, k, k), dtype, sc)
    b = synth.uniform(g, (cout,), -0.1, 0.1).astype(np.float64)
    Ho, Wo = lp.H_out, lp.W_out
    G = _round(synth.normal(g, (N, cout, Ho, Wo)), dtype, sc)
    M = _round(synth.uniform(g, (N, cin, H, W)), dtype, sc)     # ReLU-output stand-in for the mask

    x = _dev(sc, pack_level(X, lv0), dtype)
    w = _dev(sc, w_oihw_to_lib(Wt, lv0["Cpad"]), dtype)
    bias = torch.from_numpy(b.astype(np.float32)).cuda()
    y = torch.full((lv1["total_elems"],), 7.0, dtype=_td(sc, dtype), device="cuda")
    flags = (sc.FLAG_RELU if relu else 0) | extra
    ws_b = max(pl.workspace_size(0, dtype, 0), pl.workspace_size(0, dtype, 1), pl.workspace_size(0, dtype, 2), 16)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    sc.splitcnn_conv_fwd_ws(pl.handle, 0, dtype, x, w, bias, y, flags, ws, ws_b)
    Xp = O.split(X, lp.Ih, lp.Iw)
    Yref = O.conv_fwd(Xp, Wt, b, lp, relu)
    Ygot = unpack_level(_host(y), lv1, keep_pad=True)
    err = max(normwise(Ygot[i][j][:, :cout], Yref[i][j]) for i in range(nh) for j in range(nw))
    assert err <= TOL[dtype], f"fwd normwise {err}"
    for row in Ygot:
        for blk in row:
            assert np.all(blk[:, cout:] == 0), "channel padding of Y must be zero"

    dy = _dev(sc, pack_level(G, lv1), dtype)
    mask = _dev(sc, pack_level(M, lv0), dtype)
    dx = torch.full((lv0["total_elems"],), 7.0, dtype=_td(sc, dtype), device="cuda")
    sc.splitcnn_conv_bwd_data(pl.handle, 0, dtype, dy, w, dx, mask, ws, ws_b, extra)
    Gp = O.split(G, lp.Oh, lp.Ow)
    dXref = O.conv_bwd_data(Gp, Wt, lp, O.split(M, lp.Ih, lp.Iw))
    dXgot = unpack_level(_host(dx), lv0, keep_pad=True)
    err = max(normwise(dXgot[i][j][:, :cin], dXref[i][j]) for i in range(nh) for j in range(nw))
    assert err <= TOL[dtype], f"dgrad normwise {err}"
    for row in dXgot:
        for blk in row:
            assert np.all(blk[:, cin:] == 0), "channel padding of dX must be zero"
    # dgrad-ready weights built once (splitcnn_conv_dgrad_weights) + FLAG_DGRAD_WEIGHTS: bitwise the same dX
    wt_b = sc.splitcnn_conv_dgrad_weights_size(pl.handle, 0, dtype)
    if mode == "bf16_tc" and wt_b:
        wt = torch.empty(wt_b, dtype=torch.uint8, device="cuda")
        sc.splitcnn_conv_dgrad_weights(pl.handle, 0, dtype, w, wt, wt_b)
        dx2 = torch.full_like(dx, 5.0)
        sc.splitcnn_conv_bwd_data(pl.handle, 0, dtype, dy, wt, dx2, mask, None, 0, sc.FLAG_DGRAD_WEIGHTS)
        assert torch.equal(dx2, dx), "prepared dgrad weights must give the in-call flip's dX bit for bit"
    elif dtype != sc.BF16:
        assert wt_b == 0
        with pytest.raises(sc.SplitCNNError):
            sc.splitcnn_conv_bwd_data(pl.handle, 0, dtype, dy, w, dx, mask, ws, ws_b, sc.FLAG_DGRAD_WEIGHTS)

    dw = torch.full((cout, k, k, lv0["Cpad"]), 3.0, dtype=torch.float32, device="cuda")
    db = torch.full((cout,), 3.0, dtype=torch.float32, device="cuda")
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, dy, dw, db, 0.0, ws, ws_b, extra)
    dWref, dbref = O.conv_bwd_filter(Xp, Gp, lp)
    dWgot = _host(dw)
    assert normwise(w_lib_to_oihw(dWgot, cin), dWref) <= TOL[dtype]
    assert normwise(_host(db), dbref) <= TOL[dtype]
    if lv0["Cpad"] > cin:
        assert np.all(dWgot[..., cin:] == 0)
    # beta = 1 accumulates; the reduction order is fixed, so the result is exactly 2x (the split-operand
    # fp32 / tf32 weight gradient adds its partial products one by one: 2x up to fp32 rounding)
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, dy, dw, db, 1.0, ws, ws_b, extra)
    if dtype == sc.BF16 or extra:
        np.testing.assert_array_equal(_host(dw), 2 * dWgot)
    else:
        np.testing.assert_allclose(_host(dw), 2 * dWgot, rtol=1e-5, atol=1e-6 * np.abs(dWgot).max())
    # determinism run to run
    dw2 = torch.zeros_like(dw)
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, dy, dw2, None, 0.0, ws, ws_b, extra)
    np.testing.assert_array_equal(_host(dw2), dWgot)


def test_conv_patch_range_sharding(sc):
    """Patches computed in two ranges [0,q) + [q,P) equal one call; wgrad partial sums add up."""
    dtype = sc.BF16
    layers = [synth.conv(64, 64, 3, 1, 1)]
    ref, pl = _make(sc, layers, 2, 64, 32, 32, 2, 2, seed=5)
    lv0, lv1 = pl.levels
    g = synth.rng(5)
    x = _dev(sc, pack_level(_round(synth.uniform(g, (2, 64, 32, 32)), dtype, sc), lv0), dtype)
    w = _dev(sc, w_oihw_to_lib(_round(synth.kaiming(g, 64, 64, 3, 3), dtype, sc), lv0["Cpad"]), dtype)
    y1 = torch.zeros(lv1["total_elems"], dtype=torch.bfloat16, device="cuda")
    y2 = torch.zeros_like(y1)
    sc.splitcnn_conv_fwd(pl.handle, 0, dtype, x, w, None, y1, sc.FLAG_RELU)
    sc.splitcnn_conv_fwd(pl.handle, 0, dtype, x, w, None, y2, sc.FLAG_RELU, 0, 1)
    sc.splitcnn_conv_fwd(pl.handle, 0, dtype, x, w, None, y2, sc.FLAG_RELU, 1, 4)
    assert torch.equal(y1, y2)
    ws_b = pl.workspace_size(0, dtype, 2)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dw = torch.zeros((64, 3, 3, 64), dtype=torch.float32, device="cuda")
    dwa = torch.zeros_like(dw)
    dwb = torch.zeros_like(dw)
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, y1, dw, None, 0.0, ws, ws_b)
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, y1, dwa, None, 0.0, ws, ws_b, 0, 0, 2)
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, y1, dwb, None, 0.0, ws, ws_b, 0, 2, 4)
    torch.testing.assert_close(dwa + dwb, dw, rtol=1e-5, atol=1e-5 * dw.abs().max().item())


@pytest.mark.parametrize("k,pad", [(1, 0), (3, 1)])
def test_strided_dgrad_patch_ranges(sc, k, pad):
    """Stride-2 data gradient over patch ranges: [0, q) + [q, P) equal one call bit for bit, and a range call
    writes exactly its own patches (the phases no tap reaches are zeroed by one memset of the range, k < s;
    the other patches keep a sentinel)."""
    dtype = sc.BF16
    layers = [synth.conv(64, 128, k, 2, pad)]
    ref, pl = _make(sc, layers, 2, 64, 32, 32, 2, 2, seed=11)
    lv0, lv1 = pl.levels
    g = synth.rng(11)
    dy = _dev(sc, pack_level(_round(synth.normal(g, (2, 128, ref.layers[0].H_out, ref.layers[0].W_out)), dtype, sc), lv1),
              dtype)
    w = _dev(sc, w_oihw_to_lib(_round(synth.kaiming(g, 128, 64, k, k), dtype, sc), lv0["Cpad"]), dtype)
    ws_b = pl.workspace_size(0, dtype, 1)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dx1 = torch.full((lv0["total_elems"],), 7.0, dtype=torch.bfloat16, device="cuda")
    dx2 = torch.full_like(dx1, 7.0)
    sc.splitcnn_conv_bwd_data(pl.handle, 0, dtype, dy, w, dx1, None, ws, ws_b)
    assert not torch.any(dx1 == 7.0), "every dX element is written"
    sc.splitcnn_conv_bwd_data(pl.handle, 0, dtype, dy, w, dx2, None, ws, ws_b, 0, 0, 1)
    host = _host(dx2)
    blocks = unpack_level(host, lv0, keep_pad=True)
    assert np.all(blocks[0][1] == 7.0) and np.all(blocks[1][0] == 7.0) and np.all(blocks[1][1] == 7.0), \
        "a range call leaves the other patches alone"
    sc.splitcnn_conv_bwd_data(pl.handle, 0, dtype, dy, w, dx2, None, ws, ws_b, 0, 1, 4)
    assert torch.equal(dx1, dx2)


# --------------------------------------------------------------------------- split / merge
@pytest.mark.parametrize("dtype_name", ["bf16", "fp32"])
def test_split_merge_bit_exact(sc, dtype_name):
    dtype = sc.BF16 if dtype_name == "bf16" else sc.FP32
    for (N, C, H, W, nh, nw, seed) in [(2, 3, 32, 32, 2, 2, 0), (3, 13, 23, 17, 3, 2, 1), (2, 64, 28, 28, 4, 4, 2),
                                       (1, 256, 56, 56, 8, 8, 3)]:
        layers = [synth.conv(C, 8, 3, 1, 1)]
        ref, pl = _make(sc, layers, N, C, H, W, nh, nw, seed)
        lv0 = pl.levels[0]
        g = synth.rng(seed)
        X = _round(synth.uniform(g, (N, C, H, W)), dtype, sc)
        xt = _dev(sc, X, dtype)
        P = torch.full((lv0["total_elems"],), 5.0, dtype=_td(sc, dtype), device="cuda")
        sc.splitcnn_split(pl.handle, 0, dtype, xt, sc.NCHW, P)
        np.testing.assert_array_equal(_host(P), pack_level(X, lv0))
        back = torch.zeros_like(xt)
        sc.splitcnn_merge(pl.handle, 0, dtype, P, back, sc.NCHW)
        assert torch.equal(back, xt)
        # NHWC layout, and a partial patch range
        xh = xt.permute(0, 2, 3, 1).contiguous()
        P2 = torch.zeros_like(P)
        npat = nh * nw
        sc.splitcnn_split(pl.handle, 0, dtype, xh, sc.NHWC, P2, 0, npat // 2)
        sc.splitcnn_split(pl.handle, 0, dtype, xh, sc.NHWC, P2, npat // 2, npat)
        assert torch.equal(P2, P)
        back2 = torch.zeros_like(xh)
        sc.splitcnn_merge(pl.handle, 0, dtype, P2, back2, sc.NHWC)
        assert torch.equal(back2, xh)


# --------------------------------------------------------------------------- max-pool
@pytest.mark.parametrize("dtype_name", ["bf16", "fp32"])
@pytest.mark.parametrize("kind", ["2x2s2", "3x3s2p1"])
def test_pool_parity(sc, dtype_name, kind):
    dtype = sc.BF16 if dtype_name == "bf16" else sc.FP32
    k, s, p = (2, 2, 0) if kind == "2x2s2" else (3, 2, 1)
    N, C, H, W = 3, 24, 30, 22
    layers = [synth.maxpool(C, k, s, p)]
    ref, pl = _make(sc, layers, N, C, H, W, 3, 2, seed=11)
    lp = ref.layers[0]
    lv0, lv1 = pl.levels
    g = synth.rng(11)
    X = np.maximum(_round(synth.uniform(g, (N, C, H, W)), dtype, sc), 0)   # ReLU output: ties at 0 (R9)
    X[:, :, ::3] = _round(synth.uniform(g, (N, C, (H + 2) // 3, W)), dtype, sc)
    G = _round(synth.normal(g, (N, C, lp.H_out, lp.W_out)), dtype, sc)
    x = _dev(sc, pack_level(X, lv0), dtype)
    y = torch.zeros(lv1["total_elems"], dtype=_td(sc, dtype), device="cuda")
    a = torch.zeros(lv1["total_elems"], dtype=torch.uint8, device="cuda")
    sc.splitcnn_pool_fwd(pl.handle, 0, dtype, x, y, a, sc.FLAG_POOL_RELU_MASK)
    Yref, Aref = O.pool_fwd(O.split(X, lp.Ih, lp.Iw), lp)
    Ygot = unpack_level(_host(y), lv1)
    Agot = unpack_level(a.cpu().numpy().astype(np.float64), lv1)
    for i in range(3):
        for j in range(2):
            np.testing.assert_array_equal(Ygot[i][j], Yref[i][j])
            np.testing.assert_array_equal(Agot[i][j].astype(np.int64) & 0x7F, Aref[i][j])
            np.testing.assert_array_equal((Agot[i][j].astype(np.int64) >> 7) & 1, (Yref[i][j] > 0).astype(np.int64))
    dy = _dev(sc, pack_level(G, lv1), dtype)
    for flag in (0, sc.FLAG_POOL_RELU_MASK):
        dx = torch.full((lv0["total_elems"],), 9.0, dtype=_td(sc, dtype), device="cuda")
        sc.splitcnn_pool_bwd(pl.handle, 0, dtype, dy, a, dx, flag)
        dXref = O.pool_bwd(O.split(G, lp.Oh, lp.Ow), Aref, lp)
        if flag:
            dXref = O.relu_mask(dXref, O.split(X, lp.Ih, lp.Iw))
        dXgot = unpack_level(_host(dx), lv0)
        for i in range(3):
            for j in range(2):
                if k == s:          # no overlap: a pure scatter, bit-exact
                    np.testing.assert_array_equal(dXgot[i][j], dXref[i][j])
                else:               # R10: overlapping windows accumulate in fp32
                    assert normwise(dXgot[i][j], dXref[i][j]) <= (1e-6 if dtype == sc.FP32 else 1e-2)


# --------------------------------------------------------------------------- offload / prefetch
def test_offload_prefetch_roundtrip_bit_exact(sc):
    dtype = sc.BF16
    layers = [synth.conv(64, 64, 3, 1, 1)]
    ref, pl = _make(sc, layers, 2, 64, 28, 28, 4, 4, seed=3)
    lv0 = pl.levels[0]
    x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
    keep = x.clone()
    mem = torch.cuda.Stream()
    ready = torch.cuda.Event()
    ready.record()
    hosts = []
    for q in range(16):
        off, nb = sc.splitcnn_patch_bytes(pl.handle, 0, dtype, q)
        h = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
        done = torch.cuda.Event()
        done.record(mem)                       # creates the CUDA handle; the library re-records it
        sc.splitcnn_offload(pl.handle, 0, dtype, q, x, h, ready, mem, done)
        hosts.append((h, done))
    for _, d in hosts:
        torch.cuda.current_stream().wait_event(d)
    x.zero_()
    ready.record()
    for q, (h, _) in enumerate(hosts):
        d = torch.cuda.Event()
        d.record(mem)
        sc.splitcnn_prefetch(pl.handle, 0, dtype, q, h, x, ready, mem, d)
        torch.cuda.current_stream().wait_event(d)
    torch.cuda.synchronize()
    assert torch.equal(x, keep)
    with pytest.raises(sc.SplitCNNError, match="pinned"):
        sc.splitcnn_offload(pl.handle, 0, dtype, 0, x, torch.empty(10 ** 6, dtype=torch.uint8), None, mem, None)


def test_narrow_wgrad_opt_in_parity(sc, monkeypatch):
    """The opt-in 8-channel halo wgrad (SPLITCNN_NARROW_WGRAD) matches the oracle too."""
    monkeypatch.setenv("SPLITCNN_NARROW_WGRAD", "1")
    dtype = sc.BF16
    layers = [synth.conv(3, 64, 3, 1, 1)]
    ref, pl = _make(sc, layers, 2, 3, 30, 26, 2, 2, seed=17)
    lp = ref.layers[0]
    lv0, lv1 = pl.levels
    g = synth.rng(17)
    X = _round(synth.uniform(g, (2, 3, 30, 26)), dtype, sc)
    G = _round(synth.normal(g, (2, 64, 30, 26)), dtype, sc)
    x = _dev(sc, pack_level(X, lv0), dtype)
    dy = _dev(sc, pack_level(G, lv1), dtype)
    ws_b = pl.workspace_size(0, dtype, 2)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dw = torch.zeros((64, 3, 3, 8), dtype=torch.float32, device="cuda")
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, dy, dw, None, 0.0, ws, ws_b)
    dWref, _ = O.conv_bwd_filter(O.split(X, lp.Ih, lp.Iw), O.split(G, lp.Oh, lp.Ow), lp)
    assert normwise(w_lib_to_oihw(_host(dw), 3), dWref) <= TOL[dtype]


# (name, N, cin, cout, H, W, nh, nw): conv3x3 s1 p1 (+bias, ReLU) -> max-pool 2x2 s2, stochastic boundaries
POOL_FUSE_CASES = [
    ("c2_like", 4, 64, 64, 32, 32, 2, 2),          # halo path, 16x16 patches
    ("ragged", 3, 64, 128, 36, 28, 3, 2),          # uneven patches (even extents by R2)
    ("generic_bn256", 2, 128, 256, 24, 20, 2, 2),  # non-halo (BN > 128) tile chooser, 2-CTA
    ("tail_like", 2, 256, 512, 28, 28, 1, 1),      # unsplit tail (1x1 split), Cout 512
]


@pytest.mark.parametrize("case", POOL_FUSE_CASES, ids=[c[0] for c in POOL_FUSE_CASES])
def test_conv_pool_fused_matches_unfused_and_oracle(sc, case):
    """f1: conv(+bias, ReLU) -> max-pool fused in the tcgen05 epilogue equals conv_fwd + pool_fwd BITWISE
    (values and argmax bytes incl. the ReLU bit), and the oracle's pooled values within the bf16 bar."""
    name, N, cin, cout, H, W, nh, nw = case
    dtype = sc.BF16
    layers = [synth.conv(cin, cout, 3, 1, 1, relu=True), synth.maxpool(cout)]
    ref, pl = _make(sc, layers, N, cin, H, W, nh, nw, seed=sum(map(ord, name)))
    assert sc.splitcnn_conv_pool_supported(pl.handle, 0, dtype)
    lv0, lv1, lv2 = pl.levels
    g = synth.rng(7 + len(name))
    X = _round(synth.uniform(g, (N, cin, H, W)), dtype, sc)
    Wt = _round(synth.kaiming(g, cout, cin, 3, 3), dtype, sc)
    b = synth.uniform(g, (cout,), -0.1, 0.1).astype(np.float64)
    x = _dev(sc, pack_level(X, lv0), dtype)
    w = _dev(sc, w_oihw_to_lib(Wt, lv0["Cpad"]), dtype)
    bias = torch.from_numpy(b.astype(np.float32)).cuda()
    y1 = torch.zeros(lv1["total_elems"], dtype=torch.bfloat16, device="cuda")
    yp = torch.full((lv2["total_elems"],), 7.0, dtype=torch.bfloat16, device="cuda")
    ap = torch.full((lv2["total_elems"],), 0x55, dtype=torch.uint8, device="cuda")
    sc.splitcnn_conv_fwd(pl.handle, 0, dtype, x, w, bias, y1, sc.FLAG_RELU)
    sc.splitcnn_pool_fwd(pl.handle, 1, dtype, y1, yp, ap, sc.FLAG_POOL_RELU_MASK)
    yf = torch.full_like(yp, -3.0)
    af = torch.full_like(ap, 0xAA)
    sc.splitcnn_conv_pool_fwd(pl.handle, 0, dtype, x, w, bias, yf, af)
    torch.cuda.synchronize()
    assert torch.equal(yf, yp), "fused pooled values differ from conv_fwd + pool_fwd"
    assert torch.equal(af, ap), "fused argmax bytes differ from conv_fwd + pool_fwd"
    # and the oracle: conv (fp64) -> bf16 rounding -> pool
    lp0, lp1 = ref.layers
    Y = O.conv_fwd(O.split(X, lp0.Ih, lp0.Iw), Wt, b, lp0, True)
    Y = [[synth.to_bf16_f32(y.astype(np.float32)).astype(np.float64) for y in row] for row in Y]
    P, _ = O.pool_fwd(Y, lp1)
    got = unpack_level(_host(yf), lv2)
    err = max(normwise(got[i][j], P[i][j]) for i in range(nh) for j in range(nw))
    assert err <= TOL[dtype], err


# --------------------------------------------------------------------------- residual add, global average pool
@pytest.mark.parametrize("dtype_name", ["bf16", "fp32"])
def test_add_and_gap_parity(sc, dtype_name):
    """splitcnn_add (y = relu(a + b); masked gradient sum) on a patch range of uneven patches, and
    splitcnn_gap_fwd/_bwd (global average pool over the logical H x W) against the oracle definitions."""
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    dtype = sc.BF16 if dtype_name == "bf16" else sc.FP32
    td = _td(sc, dtype)
    N, C, H, W = 3, 24, 9, 11
    pl = SplitPlan([synth.conv(C, C, 1, 1, 0)], N, C, H, W, [0, 4, 9], [0, 3, 7, 11])
    lv = pl.levels[0]
    g = synth.rng(31)
    A, B, M = (_round(synth.normal(g, (N, C, H, W)), dtype, sc) for _ in range(3))
    a, b, m = (_dev(sc, pack_level(T, lv), dtype) for T in (A, B, M))
    y = torch.full_like(a, 7.0)
    sc.splitcnn_add(pl.handle, 0, dtype, a, b, y, None, sc.FLAG_RELU)
    ref = O.residual_add(O.split(A, [0, 4, 9], [0, 3, 7, 11]), O.split(B, [0, 4, 9], [0, 3, 7, 11]), relu=True)
    got = unpack_level(_host(y), lv)
    tol = TOL[dtype]
    assert max(normwise(got[i][j], ref[i][j]) for i in range(2) for j in range(3)) <= tol
    # masked gradient sum on patches [1, 4) only; the rest of y keeps its previous values
    y2 = y.clone()
    sc.splitcnn_add(pl.handle, 0, dtype, a, b, y2, m, 0, 1, 4)
    refm = O.relu_mask(O.residual_add(O.split(A, [0, 4, 9], [0, 3, 7, 11]), O.split(B, [0, 4, 9], [0, 3, 7, 11])),
                       O.split(M, [0, 4, 9], [0, 3, 7, 11]))
    got2 = unpack_level(_host(y2), lv)
    for q in range(6):
        i, j = divmod(q, 3)
        exp = refm[i][j] if 1 <= q < 4 else got[i][j]
        assert normwise(got2[i][j], exp) <= tol, q
    # global average pool over all patches
    pooled = torch.full((N * lv["Cpad"],), 7.0, dtype=td, device="cuda")
    sc.splitcnn_gap_fwd(pl.handle, 0, dtype, a, pooled)
    gp = _host(pooled).reshape(N, lv["Cpad"])
    assert normwise(gp[:, :C], O.global_avg_pool(A)) <= tol
    assert np.all(gp[:, C:] == 0)
    Gp = _round(synth.normal(g, (N, C)), dtype, sc)
    gpad = np.zeros((N, lv["Cpad"]))
    gpad[:, :C] = Gp
    dx = torch.full_like(a, 7.0)
    sc.splitcnn_gap_bwd(pl.handle, 0, dtype, torch.from_numpy(gpad.reshape(-1).astype(np.float32)).to("cuda", td), dx)
    dref = O.split(O.global_avg_pool_bwd(Gp, H, W), [0, 4, 9], [0, 3, 7, 11])
    gd = unpack_level(_host(dx), lv)
    assert max(normwise(gd[i][j], dref[i][j]) for i in range(2) for j in range(3)) <= tol


@pytest.mark.parametrize("dtype_name,cin,cout", [("bf16", 64, 64), ("bf16", 8, 64), ("fp32", 16, 16), ("bf16", 16, 16)])
def test_bwd_filter_empty_patch_range(sc, dtype_name, cin, cout):
    """An empty patch range (p0 == p1, e.g. a rank with no patches) contributes nothing: bwd_filter with
    beta 0 writes dW = db = 0, with beta 1 leaves them unchanged (both the tcgen05 and the FFMA path,
    db requested).  Regression: the db column-sum launch divided by zero on an empty range."""
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    dtype = sc.BF16 if dtype_name == "bf16" else sc.FP32
    l = synth.conv(cin, cout)
    Ob = sc.splitcnn_boundaries_even(16, 2)
    pl = SplitPlan([l], 2, cin, 16, 16, Ob, Ob)
    lv0, lv1 = pl.levels
    x = torch.randn(lv0["total_elems"], dtype=torch.float32, device="cuda").to(_td(sc, dtype))
    dy = torch.randn(lv1["total_elems"], dtype=torch.float32, device="cuda").to(_td(sc, dtype))
    ws_b = max(pl.workspace_size(0, dtype, 2), 16)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    for beta in (1.0, 0.0):
        dw = torch.full((cout, 3, 3, lv0["Cpad"]), 3.0, dtype=torch.float32, device="cuda")
        db = torch.full((cout,), 5.0, dtype=torch.float32, device="cuda")
        for p in (0, 2, 4):
            sc.splitcnn_conv_bwd_filter(pl.handle, 0, dtype, x, dy, dw, db, beta, ws, ws_b, 0, p, p)
        torch.cuda.synchronize()
        assert torch.equal(dw, torch.full_like(dw, 3.0 * beta)) and torch.equal(db, torch.full_like(db, 5.0 * beta))


@pytest.mark.parametrize("layout", ["NCHW", "NHWC"])
def test_split_rows_matches_full_split(sc, layout):
    """splitcnn_split_rows (a rank's own input rows under patch-row sharding) writes bit-exactly the
    patches splitcnn_split writes from the full tensor, for every contiguous block of patch rows of a
    ragged 4x3 split; patches outside [p0, p1) are untouched; a window missing a needed row is refused."""
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    L = sc.NCHW if layout == "NCHW" else sc.NHWC
    l = synth.conv(5, 8)
    N, H, W = 3, 29, 22
    Oh, Ow = [0, 5, 13, 20, 29], [0, 7, 15, 22]
    pl = SplitPlan([l], N, 5, H, W, Oh, Ow)
    lv = pl.levels[0]
    x = torch.randn((N, 5, H, W), dtype=torch.float32, device="cuda").to(torch.bfloat16)
    xl = x if L == sc.NCHW else x.permute(0, 2, 3, 1).contiguous()
    ref = torch.empty(lv["total_elems"], dtype=torch.bfloat16, device="cuda")
    sc.splitcnn_split(pl.handle, 0, sc.BF16, xl, L, ref)
    bh, nw = lv["bh"], lv["n_w"]
    for r0 in range(4):
        for r1 in range(r0 + 1, 5):
            h0, h1 = bh[r0], bh[r1]
            xr = (xl[:, :, h0:h1] if L == sc.NCHW else xl[:, h0:h1]).contiguous()
            got = torch.full_like(ref, 7.0)
            sc.splitcnn_split_rows(pl.handle, 0, sc.BF16, xr, L, h0, h1, got, r0 * nw, r1 * nw)
            lo = N * lv["Cpad"] * bh[r0] * W
            hi = N * lv["Cpad"] * bh[r1] * W
            assert torch.equal(got[lo:hi], ref[lo:hi]), (r0, r1)
            assert bool((got[:lo] == 7).all()) and bool((got[hi:] == 7).all())
    with pytest.raises(Exception):
        sc.splitcnn_split_rows(pl.handle, 0, sc.BF16, xl[:, :, 1:13].contiguous(), L, 1, 13, ref, 0, 2 * nw)


@pytest.mark.parametrize("mode", ["tc", "simt", "fp32"])
@pytest.mark.parametrize("cin,cout,H,nh", [(64, 64, 28, 2), (128, 128, 14, 2), (64, 128, 30, 3)])
def test_conv_fwd_res_parity(sc, mode, cin, cout, H, nh):
    """splitcnn_conv_fwd_res (the ResNet join fused into the conv epilogue): y = ReLU(conv(x) + b + s) per
    patch against the oracle's conv + residual add, bf16 on tcgen05 (one rounding), the conv-then-add path (FORCE_SIMT)
    and fp32; the residual's patch buffers are those of the output level."""
    dtype = sc.FP32 if mode == "fp32" else sc.BF16
    extra = sc.FLAG_FORCE_SIMT if mode == "simt" else 0
    layers = [synth.conv(cin, cout, 3, 1, 1)]
    ref, pl = _make(sc, layers, 2, cin, H, H, nh, nh, seed=cin + H)
    lp = ref.layers[0]
    lv0, lv1 = pl.levels
    g = synth.rng(300 + cin)
    X = _round(synth.uniform(g, (2, cin, H, H)), dtype, sc)
    Wt = _round(synth.kaiming(g, cout, cin, 3, 3), dtype, sc)
    b = synth.uniform(g, (cout,), -0.1, 0.1).astype(np.float64)
    S = _round(synth.uniform(g, (2, cout, H, H)), dtype, sc)
    x = _dev(sc, pack_level(X, lv0), dtype)
    s = _dev(sc, pack_level(S, lv1), dtype)
    w = _dev(sc, w_oihw_to_lib(Wt, lv0["Cpad"]), dtype)
    bias = torch.from_numpy(b.astype(np.float32)).cuda()
    y = torch.full((lv1["total_elems"],), 7.0, dtype=_td(sc, dtype), device="cuda")
    ws_b = max(pl.workspace_size(0, dtype, 0), 16)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    sc.splitcnn_conv_fwd_res(pl.handle, 0, dtype, x, w, bias, s, y, sc.FLAG_RELU | extra, ws, ws_b)
    Yref = O.residual_add(O.conv_fwd(O.split(X, lp.Ih, lp.Iw), Wt, b, lp), O.split(S, lp.Oh, lp.Ow), relu=True)
    got = unpack_level(_host(y), lv1, keep_pad=True)
    assert max(normwise(got[i][j][:, :cout], Yref[i][j]) for i in range(nh) for j in range(nh)) <= TOL[dtype]
    for row in got:
        for blk in row:
            assert np.all(blk[:, cout:] == 0)
