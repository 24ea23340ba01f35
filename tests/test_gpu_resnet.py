"""ResNet-18 split stack: the ResSplitNet executor (chained split plan, residual
joins through splitcnn_add, 1x1 s2 downsample on its own plan, 3x3 s2 p1 max-pool, 7x7 s2 stem)
against the oracle composition tests/oracle_chain.run_resnet."""
import numpy as np
import pytest

import synth
from tests import oracle_chain
from tests.helpers import normwise, unpack_level, w_lib_to_oihw

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_asplos_jinh19_b200 import splitcnn
    return splitcnn


def _run(sc, dtype, N=2, H=64, widths=(64, 128), split=(2, 2), seed=2, s2d=None, exact=False):
    from paper_conf_asplos_jinh19_b200.resnet import ResSplitNet
    chain, blocks = synth.resnet18_blocks(*widths)
    net = ResSplitNet(chain, blocks, N, 3, H, H, split=split, dtype=dtype, s2d_stem=s2d)
    if s2d is not None:
        assert net.s2d == s2d
    g = synth.rng(seed)
    bf = dtype == sc.BF16
    if exact:   # dyadic draws: every fwd / dgrad sum exact in fp32 and fp64 (see test_gpu_stack)
        X = synth.dyadic(g, (N, 3, H, H))
        params = [p for p in synth.exact_layer_params(g, chain) if p is not None]
        params += [p for p in synth.exact_layer_params(g, [b["ds"] for b in blocks if b["ds"] is not None])]
    else:
        X = synth.uniform(g, (N, 3, H, H))
        params = synth.resnet_params(g, chain, blocks)
    if bf:
        X = synth.to_bf16_f32(X)
        params = [(synth.to_bf16_f32(Wt), b) for Wt, b in params]
    net.set_params([(torch.from_numpy(Wt), torch.from_numpy(b)) for Wt, b in params])
    L = net.region.levels[-1]
    G = (synth.dyadic if exact else synth.normal)(g, (N, L["C"], L["H"], L["W"]))
    if bf:
        G = synth.to_bf16_f32(G)
    x = torch.from_numpy(X).to("cuda", net.tdtype)
    dy = torch.from_numpy(np.ascontiguousarray(G.transpose(0, 2, 3, 1))).reshape(-1).to("cuda", net.tdtype)
    out = net.forward(x)
    net.backward(dy)
    torch.cuda.synchronize()
    Oh, Ow = net.boundaries(0)
    ref_out, dWs, dbs = oracle_chain.run_resnet(chain, blocks, N, 3, H, H, Oh, Ow,
                                                [(W.astype(np.float64), b.astype(np.float64)) for W, b in params],
                                                X.astype(np.float64), G.astype(np.float64), round_bf16=bf)
    got = out.float().cpu().numpy().reshape(N, L["H"], L["W"], L["C"]).transpose(0, 3, 1, 2)
    errs = {"out": normwise(got, ref_out)}
    keys = [("r", m) for m, l in enumerate(chain) if l["op"] == "conv"] + [("ds", k) for k in sorted(net.ds_plans)]
    for i, key in enumerate(keys):
        dW = net.grad_oihw(key).double().cpu().numpy()
        errs[f"dW{i}"] = normwise(dW, dWs[i])
        errs[f"db{i}"] = normwise(net.grads[key][1].cpu().numpy(), dbs[i])
    # the block outputs are the merged output of the last level; also check level 2 (pool output)
    return errs


def test_resnet_stack_fp32(sc):
    """fp32 (FFMA) fwd + bwd of the whole stack: output and every dW / db within 1e-4 normwise."""
    errs = _run(sc, sc.FP32)
    assert max(errs.values()) <= 1e-4, errs


def test_resnet_stack_bf16_forward(sc):
    """bf16 tensor-core path, Kaiming draws: the forward output within the bf16 bar 2e-2.  (The
    backward of such a draw is not comparable at 2e-2: a conv output that rounds to the other side of
    a ReLU kink, or a 3x3 max-pool near-tie (R9), re-routes a whole gradient element; the backward is
    checked on dyadic draws below.)"""
    errs = _run(sc, sc.BF16)
    assert errs["out"] <= 2e-2, errs


@pytest.mark.parametrize("s2d", [True, False])
@pytest.mark.parametrize("N,H,seed", [(2, 64, 200), (1, 112, 201), (1, 56, 202)])
def test_resnet_stack_bf16_whole_backward(sc, s2d, N, H, seed):
    """bf16 whole ResNet split stack (s2d or plain 7x7 s2 stem, 3x3 s2 p1 pool, residual joins, 1x1 s2
    downsample; H=56 gives ragged patches), forward and backward, every dW / db within the R13 bf16 bar
    2e-2.  Dyadic draws make every fwd / dgrad sum exact, so both sides take the same decisions; the
    output must agree exactly."""
    errs = _run(sc, sc.BF16, N=N, H=H, seed=seed, s2d=s2d, exact=True)
    assert errs["out"] == 0.0, errs
    assert max(errs.values()) <= 2e-2, errs


def test_s2d_stem_conv_matches_oracle_per_op(sc):
    """Space-to-depth stem (split layout NCHW_S2D + 4x4 s1 conv on 12 channels) vs the oracle's 7x7 s2
    p3 split conv, forward and weight gradient, bf16 within 2e-2 (same products, other order)."""
    from oracle import ops as O
    from oracle import plan as OP
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    from paper_conf_asplos_jinh19_b200.resnet import s2d_stem_layer, s2d_stem_weight, s2d_stem_grad
    g = synth.rng(11)
    N, H, cout = 2, 60, 64
    l = synth.conv(3, cout, k=7, s=2, p=3)
    X = synth.to_bf16_f32(synth.uniform(g, (N, 3, H, H)))
    Wt = synth.to_bf16_f32(synth.kaiming(g, cout, 3, 7, 7))
    b = synth.uniform(g, (cout,), -0.1, 0.1)
    G = synth.to_bf16_f32(synth.normal(g, (N, cout, 30, 30)))
    Oh = [0, 11, 30]
    ref = OP.plan([l], N, 3, H, H, Oh, Oh).layers[0]
    pl = SplitPlan([s2d_stem_layer(l)], N, 12, H // 2, H // 2, Oh, Oh)
    lv0, lv1 = pl.levels
    assert lv0["bh"] == [v // 2 for v in ref.Ih]
    x = torch.from_numpy(X).to("cuda", torch.bfloat16)
    xp = torch.empty(lv0["total_elems"], dtype=torch.bfloat16, device="cuda")
    sc.splitcnn_split(pl.handle, 0, sc.BF16, x, sc.NCHW_S2D, xp)
    from paper_conf_asplos_jinh19_b200.net import pack_weight
    w = pack_weight(s2d_stem_weight(torch.from_numpy(Wt)).cuda(), lv0["Cpad"], torch.bfloat16)
    y = torch.empty(lv1["total_elems"], dtype=torch.bfloat16, device="cuda")
    sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, xp, w, torch.from_numpy(b).cuda(), y, 0)
    Yref = O.conv_fwd(O.split(X.astype(np.float64), ref.Ih, ref.Iw), Wt.astype(np.float64), b.astype(np.float64), ref)
    from tests.helpers import pack_level
    got = unpack_level(y.float().cpu().numpy(), lv1)
    assert max(normwise(got[i][j], Yref[i][j]) for i in range(2) for j in range(2)) <= 2e-2
    dy = torch.from_numpy(pack_level(G.astype(np.float64), lv1).astype(np.float32)).to("cuda", torch.bfloat16)
    ws_b = max(pl.workspace_size(0, sc.BF16, 2), 16)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dw = torch.zeros((cout, 4, 4, lv0["Cpad"]), dtype=torch.float32, device="cuda")
    sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, xp, dy, dw, None, 0.0, ws, ws_b)
    dWref, _ = O.conv_bwd_filter(O.split(X.astype(np.float64), ref.Ih, ref.Iw), O.split(G.astype(np.float64), Oh, Oh), ref)
    assert normwise(s2d_stem_grad(dw, 3).double().cpu().numpy(), dWref) <= 2e-2


def test_resnet_stack_ragged_fp32(sc):
    """Odd input size (ragged patches: a 2x2 split of a 7x7 layer2 output) end to end in fp32."""
    errs = _run(sc, sc.FP32, N=1, H=56, seed=5)
    assert max(errs.values()) <= 1e-4, errs


def test_resnet_stack_ragged_bf16(sc):
    """Odd input size (ragged patches: 2x2 split of a 7x7 layer2 output) through the tensor-core path."""
    errs = _run(sc, sc.BF16, N=1, H=56, seed=5)
    assert errs["out"] <= 2e-2, errs


@pytest.mark.parametrize("dtype_name", ["fp32", "bf16"])
def test_resnet18_full_trunk(sc, dtype_name):
    """Whole trunk (f2): split region -> merge -> unsplit layer3/4 -> global average pool, against
    tests/oracle_chain.run_resnet18_full.  fp32 end to end (pooled output, all 20 dW / db) at 1e-4
    (Kaiming draws); bf16 end to end at the R13 bar 2e-2 on dyadic draws (every fwd / dgrad sum exact,
    so both sides take the same ReLU / pool decisions; layer4 reduces over only 2 x 2 x 2 = 8 pixels,
    where one flipped decision of a Kaiming draw moves a dW by up to 0.34 of its norm)."""
    from paper_conf_asplos_jinh19_b200.resnet import ResNet18Net
    dtype = sc.FP32 if dtype_name == "fp32" else sc.BF16
    bf = dtype == sc.BF16
    rc, rb = synth.resnet18_blocks()
    tc, tb = synth.resnet18_tail_blocks()
    N, H = 2, 64
    net = ResNet18Net(rc, rb, tc, tb, N, 3, H, H, split=(2, 2), dtype=dtype)
    g = synth.rng(13)
    if bf:
        X = synth.dyadic(g, (N, 3, H, H))
        params = []
        for ch, bl in ((rc, rb), (tc, tb)):
            params += [p for p in synth.exact_layer_params(g, ch) if p is not None]
            params += synth.exact_layer_params(g, [b["ds"] for b in bl if b["ds"] is not None])
        G = synth.dyadic(g, (N, 512))
    else:
        X = synth.uniform(g, (N, 3, H, H))
        params = synth.resnet_params(g, rc, rb) + synth.resnet_params(g, tc, tb)
        G = synth.normal(g, (N, 512))
    if bf:
        X = synth.to_bf16_f32(X)
        params = [(synth.to_bf16_f32(Wt), b) for Wt, b in params]
    net.set_params([(torch.from_numpy(Wt), torch.from_numpy(b)) for Wt, b in params])
    if bf:
        G = synth.to_bf16_f32(G)
    pooled = net.forward(torch.from_numpy(X).to("cuda", net.tdtype))
    net.backward(torch.from_numpy(G).reshape(-1).to("cuda", net.tdtype))
    torch.cuda.synchronize()
    Oh, Ow = net.net_r.boundaries(0)
    ref, dWs, dbs = oracle_chain.run_resnet18_full(rc, rb, tc, tb, N, 3, H, H, Oh, Ow,
                                                   [(W.astype(np.float64), b.astype(np.float64)) for W, b in params],
                                                   X.astype(np.float64), G.astype(np.float64), round_bf16=bf)
    errs = {"out": normwise(pooled.float().cpu().numpy().reshape(N, 512), ref)}
    for i in range(len(dWs)):
        dW, db = net.grad_of(i)
        errs[f"dW{i}"] = normwise(dW.double().cpu().numpy(), dWs[i])
        errs[f"db{i}"] = normwise(db.double().cpu().numpy(), dbs[i])
    assert max(errs.values()) <= (2e-2 if bf else 1e-4), errs


def test_resnet_concurrent_wgrad_bitwise(sc):
    """The ResNet executor's weight gradients on the side stream (concurrent with the data gradients, joined
    per block) give bitwise the gradients of the serial backward: the same kernels on the same inputs, only
    the stream placement differs; two steps, so a join that came too late would show as a stale buffer."""
    from paper_conf_asplos_jinh19_b200.resnet import ResSplitNet
    chain, blocks = synth.resnet18_blocks(64, 128)
    N, H = 4, 64
    g = synth.rng(7)
    params = synth.resnet_params(g, chain, blocks)
    params = [(torch.from_numpy(synth.to_bf16_f32(W)), torch.from_numpy(b)) for W, b in params]
    x = torch.from_numpy(synth.to_bf16_f32(synth.uniform(g, (N, 3, H, H)))).to("cuda", torch.bfloat16)
    nets = []
    for conc in (True, False):
        net = ResSplitNet(chain, blocks, N, 3, H, H, split=(2, 2), dtype=sc.BF16, concurrent_wgrad=conc)
        net.set_params(params)
        nets.append(net)
    dy = torch.randn(nets[0].output_numel(), generator=torch.Generator().manual_seed(3)).to("cuda", torch.bfloat16)
    for _ in range(2):
        for net in nets:
            net.forward(x)
            net.backward(dy)
        torch.cuda.synchronize()
        assert torch.equal(nets[0].out, nets[1].out)
        assert torch.equal(nets[0].grad_flat, nets[1].grad_flat)
