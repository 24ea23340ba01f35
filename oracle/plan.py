"""O1 -- the Split-CNN plan in plain Python integers (TEST INFRASTRUCTURE ONLY).

Citations are /root/reference/PAPER.md line numbers (P:n) and SURVEY.md 8(c)
readings (R1..R16).

Single layer, one spatial dimension (section 3.1):
    Op(X, k, s, p), p = (p_b, p_e), k >= s
    O = (O_0 .. O_{N-1}) output partition, chosen first
    lb(I_i) = O_i*s - p_b                                         (Eq. 1)
    ub(I_i) = (O_i - 1)*s + k - p_b                               (Eq. 2)
    I_i = s*O_i                                                   (R2)
    p_{i,b} = p_b if i == 0 else I_i + p_b - O_i*s                (P:139 as corrected by R1)
    p_{i,e} = p_e if i == N-1 else (O_{i+1}-1)*s + k - (I_{i+1}+p_b)
Multi-layer: O^{m-1} := I^m, derived backward from the last layer's O (R4).
Boundaries: even O_i = floor(i*L/n) (R3); stochastic with the R5 RNG.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

MASK64 = (1 << 64) - 1


# --------------------------------------------------------------------------- boundaries
def boundaries_even(L: int, n: int) -> list[int]:
    """R3 ("as evenly as possible"): O_i = floor(i*L/n), O_n = L."""
    if n < 1 or n > L:
        raise ValueError(f"need 1 <= n <= L, got n={n}, L={L}")
    return [(i * L) // n for i in range(n + 1)]


class SplitMix64:
    """R5's generator (a fixed, documented stream so every rank draws the same scheme)."""

    def __init__(self, state: int):
        self.state = state & MASK64

    def next(self) -> int:
        self.state = (self.state + 0x9E3779B97F4A7C15) & MASK64
        z = self.state
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
        return z ^ (z >> 31)


def _stochastic_dim(rng: SplitMix64, L: int, n: int, omega: float) -> list[int]:
    """s_0 = 0; for i > 0, s_i ~ DiscreteUniform(ceil((i-w)L/N), floor((i+w)L/N))
    (inclusive bounds; R5).  Empty range -> floor(iL/n), no draw (R5)."""
    O = [0]
    for i in range(1, n):
        lo = math.ceil((i - omega) * L / n)
        hi = math.floor((i + omega) * L / n)
        if lo > hi:
            O.append((i * L) // n)
        else:
            O.append(lo + rng.next() % (hi - lo + 1))
    O.append(L)
    return O


def boundaries_random(Lh: int, nh: int, Lw: int, nw: int, omega: float, seed: int, step: int):
    """One scheme per minibatch (``step``) per spatial dimension, R5:
    state0 = seed XOR (step * 0x9E3779B97F4A7C15); H draws first, then W."""
    if not (0.0 <= omega < 0.5):
        raise ValueError("omega must be in [0, 0.5) (P:171)")
    if nh < 1 or nh > Lh or nw < 1 or nw > Lw:
        raise ValueError("need 1 <= n <= L")
    rng = SplitMix64(seed ^ ((step * 0x9E3779B97F4A7C15) & MASK64))
    Oh = _stochastic_dim(rng, Lh, nh, omega)
    Ow = _stochastic_dim(rng, Lw, nw, omega)
    return Oh, Ow


# --------------------------------------------------------------------------- one layer, one dim
def out_len(L: int, k: int, s: int, pb: int, pe: int) -> int:
    """Output length of the unsplit window op Op(X,k,s,p)."""
    return (L + pb + pe - k) // s + 1


def lb(Oi: int, k: int, s: int, pb: int) -> int:
    """Eq. 1."""
    return Oi * s - pb


def ub(Oi: int, k: int, s: int, pb: int) -> int:
    """Eq. 2."""
    return (Oi - 1) * s + k - pb


def compute_input_split_scheme(k: int, s: int, pb: int, O: list[int], L_in: int) -> list[int]:
    """Eq. 3 with the R2 choice I_i = s*O_i; I_n = L_in closes the partition."""
    return [s * Oi for Oi in O[:-1]] + [L_in]


def compute_padding(k: int, s: int, pb: int, pe: int, O: list[int], I: list[int]):
    """Eq. 5: per-patch (p_{i,b}, p_{i,e}) from P:139 (begin, R1 reading) and P:141 (end)."""
    n = len(O) - 1
    pads = []
    for i in range(n):
        pib = pb if i == 0 else I[i] + pb - O[i] * s                      # P:139 (R1)
        pie = pe if i == n - 1 else (O[i + 1] - 1) * s + k - (I[i + 1] + pb)
        pads.append((pib, pie))
    return pads


# --------------------------------------------------------------------------- the chained plan
@dataclass
class LayerPlan:
    op: str          # "conv" | "maxpool"
    kh: int
    kw: int
    sh: int
    sw: int
    cin: int
    cout: int
    Ih: list[int]    # input split scheme (H), len n_h + 1
    Iw: list[int]
    Oh: list[int]    # output split scheme (H)
    Ow: list[int]
    pads_h: list[tuple[int, int]]  # per patch row: (p_b, p_e)
    pads_w: list[tuple[int, int]]
    H_in: int
    W_in: int
    H_out: int
    W_out: int


@dataclass
class Plan:
    N: int
    layers: list[LayerPlan] = field(default_factory=list)

    @property
    def n_h(self) -> int:
        return len(self.layers[0].Ih) - 1

    @property
    def n_w(self) -> int:
        return len(self.layers[0].Iw) - 1


def plan(layers: list[dict], N: int, C: int, H: int, W: int, O_h: list[int], O_w: list[int]) -> Plan:
    """Build the chained plan.  ``layers`` are dicts with keys op, kh, kw, sh, sw,
    ph_b, ph_e, pw_b, pw_e, cin, cout.  ``O_h``/``O_w`` partition the LAST layer's
    output (R4); every earlier scheme follows from O^{m-1} = I^m."""
    # forward pass over sizes
    Hs, Ws = [H], [W]
    c = C
    for l in layers:
        if l["cin"] != c:
            raise ValueError("channel chain mismatch")
        Hs.append(out_len(Hs[-1], l["kh"], l["sh"], l["ph_b"], l["ph_e"]))
        Ws.append(out_len(Ws[-1], l["kw"], l["sw"], l["pw_b"], l["pw_e"]))
        c = l["cout"]
        if Hs[-1] <= 0 or Ws[-1] <= 0:
            raise ValueError("output size <= 0")
    for O, Lout in ((O_h, Hs[-1]), (O_w, Ws[-1])):
        if O[0] != 0 or O[-1] != Lout:
            raise ValueError("O must start at 0 and end at the output length")
        if any(O[i + 1] <= O[i] for i in range(len(O) - 1)):
            raise ValueError("O must be strictly increasing (no empty patch)")
    out = [None] * len(layers)
    Oh, Ow = list(O_h), list(O_w)
    for m in range(len(layers) - 1, -1, -1):
        l = layers[m]
        Ih = compute_input_split_scheme(l["kh"], l["sh"], l["ph_b"], Oh, Hs[m])
        Iw = compute_input_split_scheme(l["kw"], l["sw"], l["pw_b"], Ow, Ws[m])
        for I in (Ih, Iw):
            if any(I[i + 1] <= I[i] for i in range(len(I) - 1)):
                raise ValueError("empty input patch")
        pads_h = compute_padding(l["kh"], l["sh"], l["ph_b"], l["ph_e"], Oh, Ih)
        pads_w = compute_padding(l["kw"], l["sw"], l["pw_b"], l["pw_e"], Ow, Iw)
        out[m] = LayerPlan(l["op"], l["kh"], l["kw"], l["sh"], l["sw"], l["cin"], l["cout"],
                           Ih, Iw, Oh, Ow, pads_h, pads_w, Hs[m], Ws[m], Hs[m + 1], Ws[m + 1])
        Oh, Ow = Ih, Iw
    return Plan(N, out)


def patch_out_len(Lp: int, k: int, s: int, pb: int, pe: int) -> int:
    """Output extent of Op on one padded patch (Eq. 6)."""
    return (Lp + pb + pe - k) // s + 1
