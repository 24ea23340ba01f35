"""Pins for oracle.plan (O1) -- CPU only.  Each test names what fixes the value:
the paper's equations (P:n), the SURVEY 8(c) reading, or brute force."""
import itertools
import json
import os
import random

import pytest

from oracle import plan as P

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")

# layer types of the configs (k, s, p_b, p_e)
LAYER_TYPES = [(3, 1, 1, 1), (2, 2, 0, 0), (7, 2, 3, 3), (3, 2, 1, 1), (1, 2, 0, 0), (1, 1, 0, 0),
               (5, 1, 2, 2), (3, 3, 0, 0)]


def test_even_boundaries_r3():
    for L in range(1, 60):
        for n in range(1, L + 1):
            O = P.boundaries_even(L, n)
            assert O[0] == 0 and O[-1] == L and len(O) == n + 1
            sizes = [O[i + 1] - O[i] for i in range(n)]
            assert max(sizes) - min(sizes) <= 1 and min(sizes) >= 1   # "as evenly as possible"
    with pytest.raises(ValueError):
        P.boundaries_even(3, 4)


def test_printed_p139_is_off_by_one_r1():
    """R1: the begin pad as printed, I_i + p_b - (O_i - 1)s, makes an interior
    patch one output too long; the R1 reading gives exactly O_{i+1} - O_i."""
    k, s, pb, pe, L = 3, 1, 1, 1, 32
    O = [0, 16, 32]
    I = P.compute_input_split_scheme(k, s, pb, O, L)
    printed = I[1] + pb - (O[1] - 1) * s
    pads = P.compute_padding(k, s, pb, pe, O, I)
    assert P.patch_out_len(I[2] - I[1], k, s, printed, pads[1][1]) == 17
    assert P.patch_out_len(I[2] - I[1], k, s, *pads[1]) == 16


@pytest.mark.parametrize("k,s,pb,pe", LAYER_TYPES)
def test_single_layer_sizes_brute_force_pin7(k, s, pb, pe):
    """pin-7: every patch of Eq. 6 produces O_{i+1} - O_i outputs; I partitions
    the input; pads >= 0 unless k < s; I_i within [lb, ub] (Eq. 1-2) when p_b <= k - s."""
    rnd = random.Random(k * 100 + s * 10 + pb)
    for L in range(k, 70):
        Lout = P.out_len(L, k, s, pb, pe)
        if Lout < 1:
            continue
        for n in range(1, min(Lout, 6) + 1):
            for _ in range(4):
                cuts = sorted(rnd.sample(range(1, Lout), n - 1)) if n > 1 else []
                O = [0] + cuts + [Lout]
                I = P.compute_input_split_scheme(k, s, pb, O, L)
                if any(I[i + 1] <= I[i] for i in range(n)):
                    continue
                pads = P.compute_padding(k, s, pb, pe, O, I)
                for i in range(n):
                    assert P.patch_out_len(I[i + 1] - I[i], k, s, *pads[i]) == O[i + 1] - O[i]
                    if k >= s:
                        assert pads[i][0] >= 0 and pads[i][1] >= 0
                    else:
                        assert pads[i][1] >= k - s - pb
                    if i > 0 and pb <= k - s:
                        assert P.lb(O[i], k, s, pb) <= I[i] <= P.ub(O[i], k, s, pb)
                assert sum(O[i + 1] - O[i] for i in range(n)) == Lout


def test_k_equals_s_is_natural_lb_eq_ub():
    """P:128-130 + P:122: lb(I_i) = ub(I_i) iff k = s ("natural and non-intrusive")."""
    for k, s, pb in [(2, 2, 0), (3, 3, 0), (3, 1, 1), (7, 2, 3)]:
        for Oi in range(1, 20):
            assert (P.lb(Oi, k, s, pb) == P.ub(Oi, k, s, pb)) == (k == s)


def test_window_alignment_brute_force():
    """Brute force: in patch i the window of local output oh covers global input rows
    I_i + oh*s - p_{i,b} + r, which are exactly the unsplit window rows of global output
    O_i + oh, namely (O_i + oh)*s - p_b + r (so split only ZEROES taps, never shifts them)."""
    for k, s, pb, pe in LAYER_TYPES:
        L = 40
        Lout = P.out_len(L, k, s, pb, pe)
        O = P.boundaries_even(Lout, 3)
        I = P.compute_input_split_scheme(k, s, pb, O, L)
        pads = P.compute_padding(k, s, pb, pe, O, I)
        for i in range(3):
            for oh in range(O[i + 1] - O[i]):
                for r in range(k):
                    assert I[i] + oh * s - pads[i][0] + r == (O[i] + oh) * s - pb + r


def test_chained_plan_p163():
    """O^{m-1} = I^m through a chain; all pads patch-local for VGG (1,1) convs."""
    from synth import vgg19_layers, split_region
    region, _ = split_region(vgg19_layers(), 8, True)
    pl = P.plan(region, 2, 3, 32, 32, [0, 2, 4], [0, 2, 4])
    for a, b in zip(pl.layers[:-1], pl.layers[1:]):
        assert a.Oh == b.Ih and a.Ow == b.Iw
    assert pl.layers[0].Ih == [0, 16, 32]                    # App. A, C2
    assert [l.Ih for l in pl.layers if l.op == "conv"][2] == [0, 8, 16]
    for l in pl.layers:
        if l.op == "conv":
            assert all(p == (1, 1) for p in l.pads_h)


def test_resnet_appendix_a_pads():
    """App. A (C3): conv1 7x7 s2 p3 on 224 split (0,112): pads (3,2) then (3,3);
    maxpool 3x3 s2 p1 on 112 split (0,56): (1,0) then (1,1); 1x1 s2: (0,-1) then (0,0)."""
    from synth import conv, maxpool
    pl = P.plan([conv(3, 64, 7, 2, 3), maxpool(64, 3, 2, 1)], 1, 3, 224, 224, [0, 28, 56], [0, 28, 56])
    assert pl.layers[0].Ih == [0, 112, 224] and pl.layers[0].pads_h == [(3, 2), (3, 3)]
    assert pl.layers[1].Ih == [0, 56, 112] and pl.layers[1].pads_h == [(1, 0), (1, 1)]
    ds = P.plan([conv(64, 128, 1, 2, 0, relu=False)], 1, 64, 56, 56, [0, 14, 28], [0, 14, 28])
    assert ds.layers[0].pads_h == [(0, -1), (0, 0)]


def test_plan_errors():
    from synth import conv
    with pytest.raises(ValueError):
        P.plan([conv(3, 8)], 1, 3, 8, 8, [0, 4, 4, 8], [0, 8])     # empty patch
    with pytest.raises(ValueError):
        P.plan([conv(3, 8)], 1, 3, 8, 8, [0, 9], [0, 8])           # O_n != L_out
    with pytest.raises(ValueError):
        P.plan([conv(4, 8)], 1, 3, 8, 8, [0, 8], [0, 8])           # channel mismatch


# --------------------------------------------------------------------------- stochastic
def test_stochastic_ranges_pin11():
    """pin-11: s_i in [ceil((i-w)L/N), floor((i+w)L/N)], strictly increasing,
    reproducible per (seed, step); equals R3 when w = 0 and n | L."""
    for L, n in [(28, 4), (14, 4), (56, 4), (224, 8), (32, 2), (7, 4), (3, 2)]:
        for seed in range(5):
            for step in range(5):
                Oh, Ow = P.boundaries_random(L, n, L, n, 0.2, seed, step)
                assert (Oh, Ow) == P.boundaries_random(L, n, L, n, 0.2, seed, step)
                for O in (Oh, Ow):
                    assert O[0] == 0 and O[-1] == L
                    assert all(O[i + 1] > O[i] for i in range(n))
                    for i in range(1, n):
                        lo = -((-(i - 0.2) * L) // n)
                        hi = ((i + 0.2) * L) // n
                        if lo <= hi:
                            assert lo <= O[i] <= hi
        if L % n == 0:
            assert P.boundaries_random(L, n, L, n, 0.0, 1, 1)[0] == P.boundaries_even(L, n)


def test_stochastic_ranges_appendix_a():
    """App. A: at w = 0.2, L=28,n=4 -> [6,8],[13,15],[20,22]; L=56 -> [12,16],[26,30],[40,44]."""
    import math
    def rng(L, n):
        return [(math.ceil((i - 0.2) * L / n), math.floor((i + 0.2) * L / n)) for i in range(1, n)]
    assert rng(28, 4) == [(6, 8), (13, 15), (20, 22)]
    assert rng(14, 4) == [(3, 4), (7, 7), (10, 11)]
    assert rng(56, 4) == [(12, 16), (26, 30), (40, 44)]


def test_stochastic_vectors_r5():
    """R5's own test vectors (they pin oracle <-> library agreement on the RNG spec;
    they do not come from the paper).  tests/golden/r5_vectors.json cites SURVEY pin-11."""
    with open(os.path.join(GOLDEN, "r5_vectors.json")) as f:
        g = json.load(f)
    for v in g["vectors"]:
        Oh, Ow = P.boundaries_random(v["L"], v["n"], v["L"], v["n"], v["omega"], v["seed"], v["step"])
        assert Oh == v["H"] and Ow == v["W"], v
