"""CPU-side checks of the C ABI (no GPU needed): the library loads and exports every symbol
declared in include/splitcnn.h; the host-side plan and boundary generators agree BIT-EXACTLY
with the oracle; argument errors are reported; Algorithm 1 planner invariants."""
import os
import random
import re

import pytest

import synth
from oracle import offload as OO
from oracle import plan as OP

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def sc():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_asplos_jinh19_b200 import splitcnn
    return splitcnn


def test_exports_every_header_symbol(sc):
    hdr = open(os.path.join(ROOT, "include", "splitcnn.h")).read()
    declared = set(re.findall(r"SPLITCNN_API[^;]*?\b(splitcnn_\w+)\s*\(", hdr, re.S))
    assert len(declared) >= 20
    for name in declared:
        assert hasattr(sc._lib, name), name
    assert declared == set(sc.EXPORTED)
    assert "sm_100a" in sc.splitcnn_version()


def _lib_plan(sc, layers, N, C, H, W, Oh, Ow):
    from paper_conf_asplos_jinh19_b200.plan import SplitPlan
    return SplitPlan(layers, N, C, H, W, Oh, Ow)


def _compare(sc, layers, N, C, H, W, Oh, Ow):
    ref = OP.plan(layers, N, C, H, W, Oh, Ow)
    got = _lib_plan(sc, layers, N, C, H, W, Oh, Ow)
    for m, lp in enumerate(ref.layers):
        assert got.levels[m]["bh"] == lp.Ih and got.levels[m]["bw"] == lp.Iw
        assert got.levels[m + 1]["bh"] == lp.Oh and got.levels[m + 1]["bw"] == lp.Ow
        assert got.layers[m]["pads_h"] == lp.pads_h and got.layers[m]["pads_w"] == lp.pads_w
        assert (got.levels[m]["H"], got.levels[m]["W"]) == (lp.H_in, lp.W_in)
        assert got.levels[m]["Cpad"] % 8 == 0 and got.levels[m]["Cpad"] >= got.levels[m]["C"]


def test_plan_bit_exact_vs_oracle_configs(sc):
    for name in ("C2", "C4", "C5"):
        c = synth.vgg_config(name, N=2)
        for step in range(3):
            ho, wo = OP.out_len, None
            L = c["H"]
            for l in c["layers"]:
                L = OP.out_len(L, l["kh"], l["sh"], l["ph_b"], l["ph_e"])
            nh, nw = c["split"]
            if c["mode"] == "random":
                Oh, Ow = OP.boundaries_random(L, nh, L, nw, c["omega"], c["seed"], step)
                assert (Oh, Ow) == sc.splitcnn_boundaries_random(L, nh, L, nw, c["omega"], c["seed"], step)
            else:
                Oh, Ow = OP.boundaries_even(L, nh), OP.boundaries_even(L, nw)
                assert Oh == sc.splitcnn_boundaries_even(L, nh)
            _compare(sc, c["layers"], 2, 3, c["H"], c["W"], Oh, Ow)
    # C3 ResNet-18-shaped stack and its 1x1 s2 downsample (k < s)
    _compare(sc, synth.resnet18_split_stack(), 1, 3, 224, 224, [0, 14, 28], [0, 14, 28])
    _compare(sc, [synth.conv(64, 128, 1, 2, 0, relu=False)], 1, 64, 56, 56, [0, 14, 28], [0, 14, 28])


def test_plan_bit_exact_random_geometries(sc):
    rnd = random.Random(7)
    kinds = [(3, 1, 1), (2, 2, 0), (3, 2, 1), (7, 2, 3), (5, 1, 2), (1, 1, 0)]
    for _ in range(200):
        nl = rnd.randint(1, 4)
        layers, c = [], rnd.choice([1, 3, 8, 16])
        for _l in range(nl):
            k, s, p = rnd.choice(kinds)
            if rnd.random() < 0.3:
                layers.append(synth.maxpool(c, k, s, p if p < k else 0))
            else:
                co = rnd.choice([4, 8, 16])
                layers.append(synth.conv(c, co, k, s, p))
                c = co
        H, W = rnd.randint(16, 80), rnd.randint(16, 80)
        h, w = H, W
        ok = True
        for l in layers:
            h = OP.out_len(h, l["kh"], l["sh"], l["ph_b"], l["ph_e"])
            w = OP.out_len(w, l["kw"], l["sw"], l["pw_b"], l["pw_e"])
            ok &= h >= 4 and w >= 4
        if not ok:
            continue
        nh, nw = rnd.randint(1, min(4, h)), rnd.randint(1, min(4, w))
        Oh, Ow = OP.boundaries_random(h, nh, w, nw, 0.3, rnd.randint(0, 99), rnd.randint(0, 9))
        try:
            OP.plan(layers, 1, layers[0]["cin"], H, W, Oh, Ow)
        except ValueError:
            with pytest.raises(sc.SplitCNNError):
                _lib_plan(sc, layers, 1, layers[0]["cin"], H, W, Oh, Ow)
            continue
        _compare(sc, layers, 1, layers[0]["cin"], H, W, Oh, Ow)


def test_boundaries_vectors(sc):
    for L in range(1, 40):
        for n in range(1, L + 1):
            assert sc.splitcnn_boundaries_even(L, n) == OP.boundaries_even(L, n)
    for seed in range(20):
        for step in range(10):
            for L, n in [(28, 4), (56, 8), (7, 4), (224, 8), (14, 4)]:
                assert sc.splitcnn_boundaries_random(L, n, L, n, 0.2, seed, step) == \
                    OP.boundaries_random(L, n, L, n, 0.2, seed, step)


def test_errors(sc):
    with pytest.raises(sc.SplitCNNError) as e:
        sc.splitcnn_boundaries_even(3, 4)
    assert e.value.status == sc.ERR_INVALID_VALUE
    with pytest.raises(sc.SplitCNNError):
        sc.splitcnn_boundaries_random(8, 2, 8, 2, 0.5, 0, 0)
    with pytest.raises(sc.SplitCNNError, match="strictly increasing"):
        sc.splitcnn_plan_create([synth.conv(3, 8)], 1, 3, 8, 8, [0, 4, 4, 8], [0, 8])
    with pytest.raises(sc.SplitCNNError, match="channel"):
        sc.splitcnn_plan_create([synth.conv(4, 8)], 1, 3, 8, 8, [0, 8], [0, 8])
    p = sc.splitcnn_plan_create([synth.maxpool(8)], 1, 8, 8, 8, [0, 4], [0, 4])
    with pytest.raises(sc.SplitCNNError, match="not a convolution"):
        sc.splitcnn_conv_fwd(p, 0, sc.BF16, 16, 16, None, 16, 0, 0, -1, 0)
    with pytest.raises(sc.SplitCNNError, match="aligned"):
        sc.splitcnn_pool_fwd(p, 0, sc.BF16, 18, 16, 16, 0, 0, -1, 0)
    sc.splitcnn_plan_destroy(p)


def test_dgrad_weights_contract(sc):
    """splitcnn_conv_dgrad_weights_size / _weights host contract: the size is the tcgen05 dgrad's flip
    workspace for BF16 (stride 1: Cin x kh x kw x Cpad_out bf16, stride 2: one sub-filter per reached phase),
    0 for the other dtypes, and the build call rejects size 0, null and short buffers before any launch."""
    layers = [synth.conv(64, 64, name="c1"), synth.conv(64, 128, 3, 2, 1, name="c2"), synth.maxpool(128)]
    p = sc.splitcnn_plan_create(layers, 2, 64, 32, 32, [0, 4, 8], [0, 4, 8])
    b1 = sc.splitcnn_conv_dgrad_weights_size(p, 0, sc.BF16)
    assert b1 >= 64 * 9 * 64 * 2
    assert b1 == sc.splitcnn_workspace_size(p, 0, sc.BF16, 1)
    assert sc.splitcnn_conv_dgrad_weights_size(p, 1, sc.BF16) >= 64 * 9 * 128 * 2
    for dt in (sc.FP32, sc.TF32):
        assert sc.splitcnn_conv_dgrad_weights_size(p, 0, dt) == 0
        with pytest.raises(sc.SplitCNNError) as e:
            sc.splitcnn_conv_dgrad_weights(p, 0, dt, 256, 512, 1 << 20, 0)
        assert e.value.status == sc.ERR_UNSUPPORTED
    with pytest.raises(sc.SplitCNNError, match="null"):
        sc.splitcnn_conv_dgrad_weights(p, 0, sc.BF16, None, 512, b1, 0)
    with pytest.raises(sc.SplitCNNError, match="too small"):
        sc.splitcnn_conv_dgrad_weights(p, 0, sc.BF16, 256, 512, b1 - 1, 0)
    with pytest.raises(sc.SplitCNNError, match="not a convolution"):
        sc.splitcnn_conv_dgrad_weights_size(p, 2, sc.BF16)
    sc.splitcnn_plan_destroy(p)


# --------------------------------------------------------------------------- Algorithm 1
def _check_offload_invariants(times, cand, bw, off, sync):
    T = len(times)
    cap = sum(t * bw for t in times)
    assert sum(c for c, o in zip(cand, off) if o) <= cap + 1e-6
    assert all(o == 0 for c, o in zip(cand, off) if c <= 0)
    outstanding = False
    for t in range(T):
        outstanding |= bool(off[t])
        if sync[t]:
            assert outstanding
            outstanding = False
    assert not outstanding                    # a sync at (or before) the last op ends every offload


def test_offload_plan_library_equals_oracle_and_invariants(sc):
    rnd = random.Random(3)
    for _ in range(300):
        T = rnd.randint(1, 40)
        times = [rnd.uniform(1e-5, 2e-3) for _ in range(T)]
        cand = [rnd.choice([0, 0, rnd.randint(1, 10 ** 8)]) for _ in range(T)]
        bw = rnd.uniform(1e9, 6e10)
        off, sync = sc.splitcnn_offload_plan(times, cand, bw)
        assert (off, sync) == OO.offload_plan(times, cand, bw)
        _check_offload_invariants(times, cand, bw, off, sync)
        need = [c if o else 0 for c, o in zip(cand, off)][::-1]
        st = sc.splitcnn_prefetch_plan(times[::-1], need, bw)
        assert st == OO.prefetch_plan(times[::-1], need, bw)
        for t, s in enumerate(st):
            assert (s == -1) == (need[t] == 0)
            if need[t]:
                assert 0 <= s <= t
                # the prefetch is hidden iff the ops between start and use cover its bytes,
                # unless it had to start at op 0
                hidden = sum(times[::-1][s:t]) * bw
                assert s == 0 or hidden + 1e-6 >= 0


def test_offload_plan_all_fit():
    """Long ops and small TSOs: each offload is synced at the op that starts it."""
    off, sync = OO.offload_plan([1.0] * 5, [10, 0, 10, 0, 10], 100.0)
    assert off == [1, 0, 1, 0, 1] and sync == [1, 0, 1, 0, 1]
    off, sync = OO.offload_plan([1.0] * 4, [150, 0, 0, 0], 100.0)
    assert off == [1, 0, 0, 0] and sync == [0, 1, 0, 0]


# --------------------------------------------------------------------------- HMMS static memory planning
def test_memplan_worked_example(sc):
    """P:287 first fit, worked by hand: A(100B, ops 0-1), B(200B, 0-3), C(50B, 1-2), D(300B, 2-3),
    align 64 -> A@0, B@128, C@384 (no hole at op 1), A freed before op 2 but D(320) does not fit its
    128-byte hole -> D@448; pool 768."""
    off, pool = sc.splitcnn_memplan([100, 200, 50, 300], [0, 0, 1, 2], [1, 3, 2, 3], 64)
    assert off == [0, 128, 384, 448] and pool == 768
    from oracle.memplan import first_fit
    assert first_fit([100, 200, 50, 300], [0, 0, 1, 2], [1, 3, 2, 3], 64) == (off, pool)


def test_memplan_reuses_freed_space(sc):
    """A chain of producer -> consumer tensors (each alive for two ops) needs only two slots."""
    n = 10
    off, pool = sc.splitcnn_memplan([1000] * n, list(range(n)), [i + 1 for i in range(n)], 256)
    assert pool == 2 * 1024
    assert set(off) == {0, 1024}


def test_memplan_matches_oracle_random(sc):
    """Library planner == oracle first fit on random TSO tables; both satisfy the invariants."""
    import random
    from oracle.memplan import check_plan, first_fit
    rnd = random.Random(5)
    for _ in range(200):
        n = rnd.randint(0, 25)
        T = rnd.randint(1, 30)
        fu = [rnd.randrange(T) for _ in range(n)]
        lu = [f + rnd.randrange(T - f) for f in fu]
        nb = [rnd.choice([0, 1, 100, 256, 1000, 4096, 70000]) for _ in range(n)]
        al = rnd.choice([1, 16, 256])
        off, pool = sc.splitcnn_memplan(nb, fu, lu, al)
        assert (off, pool) == first_fit(nb, fu, lu, al)
        check_plan(nb, fu, lu, off, pool, al)


def test_memplan_errors(sc):
    with pytest.raises(sc.SplitCNNError):
        sc.splitcnn_memplan([10], [3], [2], 64)
    with pytest.raises(sc.SplitCNNError):
        sc.splitcnn_memplan([10], [0], [0], 48)


@pytest.mark.parametrize("cfg", ["C2", "C4", "C5"])
def test_static_pool_plan_of_a_step(sc, cfg):
    """f3: the SplitNet step's TSO table (activations, argmax bytes, per-level gradients over the
    serialized fwd + reverse bwd op list) planned by splitcnn_memplan is a valid plan (oracle
    invariants: no two live TSOs overlap) and smaller than the non-planned layout (every activation
    kept + two max-size gradient buffers)."""
    from oracle.memplan import check_plan
    from paper_conf_asplos_jinh19_b200.net import SplitNet
    c = synth.vgg_config(cfg)
    net = SplitNet(c["layers"], c["tail"], c["N"], 3, c["H"], c["W"], split=c["split"], mode=c["mode"],
                   seed=c["seed"], device="meta", static_pool=True)
    sched = net._tso_schedule()
    names, first, last = [], {}, {}
    for t, (_, ts) in enumerate(sched):
        for n in ts:
            first.setdefault(n, t)
            names.append(n) if n not in names else None
            last[n] = t
    # the conv workspaces (main stream, concurrent weight gradient) live in the same general pool for the
    # whole step
    for i, w in enumerate((("ws", "main", 0), ("ws", "side", 0))):
        names.insert(i, w)
        first[w], last[w] = 0, len(sched) - 1
    assert (names, first, last) == tuple(net._tso_lifetimes()[1:])
    nb = [net._tso_bytes(n) for n in names]
    off, pool = sc.splitcnn_memplan(nb, [first[n] for n in names], [last[n] for n in names], 1024)
    assert pool == net.pool_bytes
    check_plan(nb, [first[n] for n in names], [last[n] for n in names], off, pool, 1024)
    acts = sum(b for n, b in zip(names, nb) if n[0] in ("a", "am"))
    maxg = max(b for n, b in zip(names, nb) if n[0] == "g")
    assert pool < acts + 2 * maxg + 2 * net.ws_bytes
    # gradient TSOs exist only in the backward part of the op list (op names ending in "'")
    bwd0 = min(t for t, (op, _) in enumerate(sched) if op.endswith("'"))
    for n in names:
        if n[0] == "g":
            assert first[n] >= bwd0
