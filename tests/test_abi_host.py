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
