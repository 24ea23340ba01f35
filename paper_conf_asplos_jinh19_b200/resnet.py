"""ResSplitNet -- the BN-free ResNet-18 split stack through libsplitcnn.

The main branch (conv1 7x7 s2 -> ReLU -> max-pool 3x3 s2 p1 -> layer1 -> layer2) is ONE chained
split plan; each basic block ends in a residual join y = ReLU(conv_b(h) + shortcut(x)).
The join is pointwise, so it is split-invariant and the shortcut shares its sibling's I and O
(summation sharing): the identity shortcut reads the block input's patch buffers as they
are, and the 1x1 s2 downsample gets its own one-layer plan whose output partition is the block
output's, which by I = s*O (R2) gives exactly the block input's partition as its input (asserted).

Backward of a block (x = input level a, h = level a+1, y = level a+2; g = dL/dy, unmasked):
    gz = g * [y > 0]                            (fused into the previous join's add)
    gh = dgrad_b(gz) * [h > 0];  dW_b = wgrad(h, gz)
    gx = dgrad_a(gh) + shortcut^T(gz);  dW_a = wgrad(x, gh)   (+ dW_ds = wgrad(x, gz))
    g' = gx * [x > 0] when x is itself a block output  (splitcnn_add with a mask)
Every step is a libsplitcnn call; PyTorch only allocates memory and provides the stream.
BN (R11) is not part of the split stack.
"""
from __future__ import annotations

import torch

from . import splitcnn as sc
from .net import SplitNet, pack_weight
from .plan import SplitPlan


def s2d_stem_layer(l: dict, cin_pad: int = 0) -> dict:
    """The 7x7 s2 p3 stem on C channels as the equivalent 4x4 s1 conv on the space-to-depth(2) input
    (4C channels, H/2 x W/2): out[t] = sum_{q, phi} Xs2d[t + q - 2][phi] * W[2q + phi - 1] (tap -1 is
    zero), i.e. begin pad 2, end pad 1 -- and under R2 the same patch-local pads (2, k - s - p_b = 1).
    cin_pad > 4C declares zero channels up to cin_pad (64: the level takes the 64-channel halo /
    2-CTA tensor-core kernels instead of the 16-channel per-tap path).  "macs_per_out" keeps the
    algorithmic work of the 7x7 layer for the roofline accounting."""
    return dict(op="conv", kh=4, kw=4, sh=1, sw=1, ph_b=2, ph_e=1, pw_b=2, pw_e=1, cin=max(4 * l["cin"], cin_pad),
                cout=l["cout"], relu=l.get("relu", True), name=l.get("name", "conv1"),
                macs_per_out=l["cin"] * l["kh"] * l["kw"])


def s2d_stem_weight(W: torch.Tensor) -> torch.Tensor:
    """OIHW [Co][C][7][7] -> OIHW [Co][4C][4][4]: W''[o][4c + 2ph + pw][qh][qw] = W[o][c][2qh+ph-1][2qw+pw-1]."""
    co, c, kh, kw = W.shape
    out = torch.zeros((co, 4 * c, 4, 4), dtype=W.dtype, device=W.device)
    for qh in range(4):
        for ph in range(2):
            r = 2 * qh + ph - 1
            if not 0 <= r < kh:
                continue
            for qw in range(4):
                for pw in range(2):
                    s = 2 * qw + pw - 1
                    if 0 <= s < kw:
                        out[:, 2 * ph + pw::4, qh, qw] = W[:, :, r, s]
    return out


def s2d_stem_grad(dWp: torch.Tensor, cin: int) -> torch.Tensor:
    """Packed stem gradient [Co][4][4][Cpad >= 4*cin] -> OIHW [Co][cin][7][7] (adjoint of s2d_stem_weight;
    the zero tap's gradient is dropped)."""
    co = dWp.shape[0]
    out = torch.zeros((co, cin, 7, 7), dtype=dWp.dtype, device=dWp.device)
    for r in range(7):
        qh, ph = (r + 1) // 2, (r + 1) % 2
        for s_ in range(7):
            qw, pw = (s_ + 1) // 2, (s_ + 1) % 2
            out[:, :, r, s_] = dWp[:, qh, qw, 2 * ph + pw:4 * cin:4]
    return out


class ResSplitNet(SplitNet):
    def __init__(self, chain: list[dict], blocks: list[dict], N: int, C: int, H: int, W: int, split=(2, 2),
                 dtype: int = sc.BF16, device="cuda", force_simt: bool = False, s2d_stem: bool | None = None,
                 stem_pad: int = 16, **kw):
        self.blocks = blocks
        self.block_at = {b["a"]: k for k, b in enumerate(blocks)}
        st = chain[0]
        ok = (st["op"] == "conv" and st["kh"] == st["kw"] == 7 and st["sh"] == st["sw"] == 2 and st["ph_b"] == 3
              and H % 2 == 0 and W % 2 == 0 and dtype == sc.BF16 and not force_simt)
        # the stride-2 stem on a 3-channel input is a poor tensor-core shape (8-channel padded, strided
        # TMA rows); read space-to-depth it is a stride-1 4x4 conv on 12 (pad 16) channels, same sums
        self.s2d = ok if s2d_stem is None else (s2d_stem and ok)
        self.stem_cin = st["cin"]
        if self.s2d:
            # stem_pad 16 (default): the 12 real channels in 16 take the narrow-row halo kernels (forward:
            # one x4 MMA issue per kernel row; weight gradient: SW32 MN-major X); 64: the 64-channel halo /
            # 2-CTA kernels on zero channels (5.3x the MMA work of the 7x7 layer, counted as the 7x7 work)
            stem = s2d_stem_layer(st, stem_pad)
            chain = [stem] + list(chain[1:])
            C, H, W = stem["cin"], H // 2, W // 2
        super().__init__(chain, [], N, C, H, W, split=split, mode="even", dtype=dtype, device=device,
                         force_simt=force_simt, fuse_pool=False, **kw)

    # ------------------------------------------------------------------ planning / buffers
    def _alloc(self, grad_buffer=None):
        R = self.region
        self.ds_plans = {}
        for k, b in enumerate(self.blocks):
            if b["ds"] is None:
                continue
            a = b["a"]
            lo, li = R.levels[a + 2], R.levels[a]
            p = SplitPlan([b["ds"]], self.N, li["C"], li["H"], li["W"], lo["bh"], lo["bw"])
            got = p.levels[0]
            assert got["bh"] == li["bh"] and got["bw"] == li["bw"] and got["Cpad"] == li["Cpad"], \
                "downsample input partition differs from the block input's"
            assert p.levels[1]["bh"] == lo["bh"] and p.levels[1]["bw"] == lo["bw"]
            self.ds_plans[k] = p
        super()._alloc(grad_buffer)
        dev, td = self.device, self.tdtype
        # block outputs are relu(z + s) written in place over conv_b's output level
        self.block_out = {b["a"] + 2 for b in self.blocks}
        maxg = self.grad[0].numel()
        self.grad += [torch.zeros(maxg, dtype=td, device=dev), torch.zeros(maxg, dtype=td, device=dev)]
        self.ds_out = {k: torch.zeros(self.region.level_elems(self.blocks[k]["a"] + 2), dtype=td, device=dev)
                       for k in self.ds_plans}
        self.zeros = torch.zeros(self.region.level_elems(self.region.nlayers), dtype=td, device=dev)
        L = self.region.levels[-1]
        self.out = torch.zeros(L["N"] * L["H"] * L["W"] * L["C"], dtype=td, device=dev)   # merged NHWC
        ws = self.ws_bytes
        for p in self.ds_plans.values():
            ws = max(ws, p.workspace_size(0, self.dtype, 1), p.workspace_size(0, self.dtype, 2))
        if ws > self.ws_bytes:
            self.ws = torch.zeros(ws // 4 + 4, dtype=torch.float32, device=dev)
            self.ws_bytes = self.ws.numel() * 4
            self.ws_w = torch.zeros_like(self.ws) if self.concurrent_wgrad else self.ws

    def _ds_layers(self):
        return [(k, self.blocks[k]["ds"], self.ds_plans[k]) for k in sorted(self.ds_plans)]

    def grad_numel(self) -> int:
        n = super().grad_numel()
        for k, l, p in self._ds_layers():
            n += l["cout"] * l["kh"] * l["kw"] * p.levels[0]["Cpad"] + l["cout"]
        return n

    def bind_grads(self, flat: torch.Tensor):
        super().bind_grads(flat)
        off = super().grad_numel()
        for k, l, p in self._ds_layers():
            cpad = p.levels[0]["Cpad"]
            nw = l["cout"] * l["kh"] * l["kw"] * cpad
            self.grads[("ds", k)] = (flat[off:off + nw].view(l["cout"], l["kh"], l["kw"], cpad),
                                     flat[off + nw:off + nw + l["cout"]])
            off += nw + l["cout"]

    def set_params(self, params):
        """params: (W_oihw, b) per chain conv in order, then per downsample conv (synth.resnet_params)."""
        params = list(params)
        nchain = sum(1 for l in self.region_layers if l["op"] == "conv")
        if not hasattr(self, "_ds_params"):
            self._ds_params = {}
            for k, l, p in self._ds_layers():
                self._ds_params[k] = (
                    torch.zeros((l["cout"], l["kh"], l["kw"], p.levels[0]["Cpad"]), dtype=self.tdtype, device=self.device),
                    torch.zeros(l["cout"], dtype=torch.float32, device=self.device))
        if self.s2d:
            W0, b0 = params[0]
            params = [(s2d_stem_weight(torch.as_tensor(W0)), b0)] + params[1:]
        super().set_params(params[:nchain])
        for (k, l, p), (W, b) in zip(self._ds_layers(), params[nchain:]):
            W = torch.as_tensor(W).to(self.device)
            self._ds_params[k][0].copy_(pack_weight(W, p.levels[0]["Cpad"], self.tdtype))
            self._ds_params[k][1].copy_(torch.as_tensor(b, dtype=torch.float32))

    def _conv_keys(self):
        """Conv keys in synth.resnet_params order: chain convs, then downsamples."""
        return [("r", m) for m, l in enumerate(self.region_layers) if l["op"] == "conv"] + \
               [("ds", k) for k in sorted(self.ds_plans)]

    def grad_oihw(self, key) -> torch.Tensor:
        """Weight gradient of conv `key` in OIHW (the stem's s2d gradient mapped back to 7x7)."""
        dW = self.grads[key][0]
        if key == ("r", 0) and self.s2d:
            return s2d_stem_grad(dW, self.stem_cin)
        l = self.region_layers[key[1]] if key[0] == "r" else self.blocks[key[1]]["ds"]
        return dW[..., :l["cin"]].permute(0, 3, 1, 2)

    def _masked(self, key: str, m: int) -> bool:
        """ReLU mask of level m: conv outputs with their own ReLU, and block outputs (ReLU after the add)."""
        if m in getattr(self, "block_out", ()):
            return True
        return super()._masked(key, m)

    # ------------------------------------------------------------------ passes
    def forward(self, x: torch.Tensor, stream=None, x_layout: int = sc.NCHW):
        p0, p1 = self.patch_range
        R, dt, fl = self.region.handle, self.dtype, self.flags_extra
        acts = self.act_r
        self._prep_dgrad(stream)
        self._label = "input"
        if self.s2d:
            self._call("split", 2 * self._bytes(self.region, 0)[0], sc.splitcnn_split_s2d, R, 0, dt, x, self.stem_cin,
                       acts[0], p0, p1, stream)
        else:
            self._call("split", 2 * self._bytes(self.region, 0)[0], sc.splitcnn_split, R, 0, dt, x, x_layout, acts[0],
                       p0, p1, stream)
        m = 0
        L = self.region_layers
        while m < len(L):
            l = L[m]
            self._label = l["name"]
            if m in self.block_at:
                k = self.block_at[m]
                la, lb = L[m], L[m + 1]
                W, b = self.params[("r", m)]
                self._label = la["name"]
                self._call("conv_fwd", self._conv_work(self.region, m, la), sc.splitcnn_conv_fwd, R, m, dt,
                           acts[m], W, b, acts[m + 1], (sc.FLAG_RELU if la["relu"] else 0) | fl, p0, p1, stream)
                if k in self.ds_plans:
                    P, lds = self.ds_plans[k], self.blocks[k]["ds"]
                    W, b = self._ds_params[k]
                    self._label = lds["name"]
                    self._call("conv_fwd", self._conv_work(P, 0, lds), sc.splitcnn_conv_fwd, P.handle, 0, dt,
                               acts[m], W, b, self.ds_out[k], fl, p0, p1, stream)
                    sc_src = self.ds_out[k]
                else:
                    sc_src = acts[m]
                # conv_b with the residual join fused into its epilogue: y = ReLU(conv_b(h) + b + shortcut)
                W, b = self.params[("r", m + 1)]
                self._label = lb["name"]
                self._call("conv_fwd", self._conv_work(self.region, m + 1, lb), sc.splitcnn_conv_fwd_res, R, m + 1, dt,
                           acts[m + 1], W, b, sc_src, acts[m + 2], sc.FLAG_RELU | fl, self.ws, self.ws_bytes, p0, p1,
                           stream)
                m += 2
                continue
            if l["op"] == "conv":
                W, b = self.params[("r", m)]
                self._call("conv_fwd", self._conv_work(self.region, m, l), sc.splitcnn_conv_fwd, R, m, dt, acts[m], W,
                           b, acts[m + 1], (sc.FLAG_RELU if l["relu"] else 0) | fl, p0, p1, stream)
            else:
                flags = sc.FLAG_POOL_RELU_MASK if self._masked("r", m) else 0
                bi, bo = self._bytes(self.region, m)
                self._call("pool_fwd", bi + bo + bo // (2 if dt == sc.BF16 else 4), sc.splitcnn_pool_fwd, R, m, dt,
                           acts[m], acts[m + 1], self.argmax[("r", m)], flags, p0, p1, stream)
            m += 1
        nl = self.region.nlayers
        self._label = "output"
        self._call("merge", 2 * self._bytes(self.region, nl - 1)[1], sc.splitcnn_merge, R, nl, dt, acts[nl], self.out,
                   sc.NHWC, p0, p1, stream)
        return self.out

    def _free(self, *busy):
        for g in self.grad:
            if all(g is not b for b in busy):
                return g
        raise RuntimeError("no free gradient buffer")

    def backward(self, dy: torch.Tensor, stream=None, need_input_grad: bool = False):
        """dy: gradient of the merged NHWC output (same layout as forward()'s result)."""
        p0, p1 = self.patch_range
        R, dt, fl = self.region.handle, self.dtype, self.flags_extra
        acts, L = self.act_r, self.region_layers
        nl = self.region.nlayers
        main = stream if stream is not None else torch.cuda.current_stream(self.device)
        conc = self.concurrent_wgrad
        nev = [0]

        def wgrad(handle, layer, x_act, gsrc, dW, db, wk):
            """A weight gradient: concurrently with the data gradients on the side stream (forked after its dY
            is ready on `main`, own workspace), joined at the end of the block -- or in line."""
            if not conc:
                self._call("conv_wgrad", wk, sc.splitcnn_conv_bwd_filter, handle, layer, dt, x_act, gsrc, dW, db, 0.0,
                           self.ws, self.ws_bytes, fl, p0, p1, stream)
                return
            if self.side is None:
                self.side = torch.cuda.Stream(self.device)
                self.fork_ev = [torch.cuda.Event() for _ in range(64)]
                self.join_ev = [torch.cuda.Event() for _ in range(64)]
            ev = self.fork_ev[nev[0] % 64]
            nev[0] += 1
            ev.record(main)
            self.side.wait_event(ev)
            with torch.cuda.stream(self.side):
                self._call("conv_wgrad", wk, sc.splitcnn_conv_bwd_filter, handle, layer, dt, x_act, gsrc, dW, db, 0.0,
                           self.ws_w, self.ws_bytes, fl, p0, p1, self.side)

        def join():
            """main waits for the side stream's weight gradients (their dY buffers are reused next)."""
            if conc and self.side is not None:
                ev = self.join_ev[nev[0] % 64]
                nev[0] += 1
                ev.record(self.side)
                main.wait_event(ev)

        g = self.grad[0]
        self._label = "output"
        self._call("split", 2 * self._bytes(self.region, nl - 1)[1], sc.splitcnn_split, R, nl, dt, dy, sc.NHWC, g,
                   p0, p1, stream)
        # the last block output is a ReLU output: gz = g * [y > 0]
        nb = self._bytes(self.region, nl - 1)[1]
        self._call("add", 3 * nb, sc.splitcnn_add, R, nl, dt, g, self.zeros, g, acts[nl], 0, p0, p1, stream)
        m = nl - 1
        while m >= 0:
            a = m - 1
            if a in self.block_at:            # m is conv_b of the block starting at a
                k = self.block_at[a]
                la, lb = L[a], L[a + 1]
                gz = g
                gh = self._free(gz)
                W, _ = self.params[("r", a + 1)]
                dW, db = self.grads[("r", a + 1)]
                wk = self._conv_work(self.region, a + 1, lb)
                self._label = lb["name"]
                wgrad(R, a + 1, acts[a + 1], gz, dW, db, wk)
                Wd, fd = self._dgrad_w("r", a + 1, W, fl, main)
                self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, R, a + 1, dt, gz, Wd, gh, acts[a + 1], self.ws,
                           self.ws_bytes, fd, p0, p1, stream)
                gx = self._free(gz, gh)
                W, _ = self.params[("r", a)]
                dW, db = self.grads[("r", a)]
                wk = self._conv_work(self.region, a, la)
                self._label = la["name"]
                wgrad(R, a, acts[a], gh, dW, db, wk)
                Wd, fd = self._dgrad_w("r", a, W, fl, main)
                self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, R, a, dt, gh, Wd, gx, None, self.ws,
                           self.ws_bytes, fd, p0, p1, stream)
                if k in self.ds_plans:
                    P, lds = self.ds_plans[k], self.blocks[k]["ds"]
                    W, _ = self._ds_params[k]
                    dW, db = self.grads[("ds", k)]
                    gs = self._free(gz, gh, gx)
                    wk = self._conv_work(P, 0, lds)
                    self._label = lds["name"]
                    wgrad(P.handle, 0, acts[a], gz, dW, db, wk)
                    self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, P.handle, 0, dt, gz, W, gs, None, self.ws,
                               self.ws_bytes, fl, p0, p1, stream)
                else:
                    gs = gz
                mask = acts[a] if self._masked("r", a) else None
                self._label = f"{la['name'][:-2]}_add"
                nb = self._bytes(self.region, a)[0]
                self._call("add", (4 if mask is not None else 3) * nb, sc.splitcnn_add, R, a, dt, gx, gs, gx, mask, 0,
                           p0, p1, stream)
                join()
                g = gx
                m = a - 1
                continue
            l = L[m]
            self._label = l["name"]
            out = self._free(g)
            last = m == 0 and not need_input_grad
            if l["op"] == "conv":
                W, _ = self.params[("r", m)]
                dW, db = self.grads[("r", m)]
                wk = self._conv_work(self.region, m, l)
                if not last:
                    Wd, fd = self._dgrad_w("r", m, W, fl, main)
                    self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, R, m, dt, g, Wd, out,
                               acts[m] if self._masked("r", m) else None, self.ws, self.ws_bytes, fd, p0, p1, stream)
                self._call("conv_wgrad", wk, sc.splitcnn_conv_bwd_filter, R, m, dt, acts[m], g, dW, db, 0.0, self.ws,
                           self.ws_bytes, fl, p0, p1, stream)
            else:
                flags = sc.FLAG_POOL_RELU_MASK if self._masked("r", m) else 0
                bi, bo = self._bytes(self.region, m)
                self._call("pool_bwd", bi + bo + bo // (2 if dt == sc.BF16 else 4), sc.splitcnn_pool_bwd, R, m, dt, g,
                           self.argmax[("r", m)], out, flags, p0, p1, stream)
            if not last:
                g = out
            m -= 1
        join()
        return g

    # ------------------------------------------------------------------ accounting
    def conv_flops(self) -> int:
        total = super().conv_flops()
        for k, l, p in self._ds_layers():
            lo = p.levels[1]
            total += 3 * 2 * lo["N"] * l["cout"] * lo["H"] * lo["W"] * l["cin"] * l["kh"] * l["kw"]
        return total

    def output_numel(self) -> int:
        return self.out.numel()


class ResBNSplitNet(ResSplitNet):
    """ResNet-18 split stack WITH batch normalisation: every conv (stem, the
    two of each block, the downsample) is conv (no bias) -> whole-tensor BN -> (ReLU), i.e.
        h = ReLU(BN_a(conv_a(x))),  y = ReLU(BN_b(conv_b(h)) + shortcut(x)),  shortcut = x | BN_ds(ds(x)).
    BN statistics are over the logical tensor (all patches) via splitcnn_bn_stats / _bn_fwd; conv
    outputs z are kept (BN backward needs them), BN(+ReLU) outputs live in separate level buffers.
    Under patch sharding (patch_range, dist.DistResNet) every rank sums its own patches and
    `bn_reduce(t)` all-reduces the per-channel [2][C] sums before they are used: the statistics after
    splitcnn_bn_stats, the backward sums (dbeta, dgamma) after splitcnn_bn_bwd_sums -- R11's statistics
    over the whole logical tensor, from per-rank partial sums."""

    def __init__(self, *a, eps: float = 1e-5, bn_reduce=None, **kw):
        self.eps = eps
        self.bn_reduce = bn_reduce          # callable(fp32 tensor): in-place sum over ranks, or None
        super().__init__(*a, **kw)

    def _bn_keys(self):
        keys = [("r", m) for m, l in enumerate(self.region_layers) if l["op"] == "conv"]
        return keys + [("ds", k) for k in sorted(self.ds_plans)]

    def _bn_level(self, key):
        """(plan, level index, logical count) of the conv output that BN `key` normalises."""
        if key[0] == "r":
            P, lv = self.region, key[1] + 1
        else:
            P, lv = self.ds_plans[key[1]], 1
        L = P.levels[lv]
        return P, lv, float(L["N"] * L["H"] * L["W"])

    def _alloc(self, grad_buffer=None):
        super()._alloc(grad_buffer)
        dev, td = self.device, self.tdtype
        R = self.region
        # post-BN activations of every region conv output level (the conv output z stays in act_r)
        self.bn_out = {m + 1: torch.zeros(R.level_elems(m + 1), dtype=td, device=dev)
                       for m, l in enumerate(self.region_layers) if l["op"] == "conv"}
        self.ds_bn = {k: torch.zeros_like(v) for k, v in self.ds_out.items()}
        self.bn_sums, self.bn_mi, self.bn_gamma, self.bn_beta = {}, {}, {}, {}
        ws = 0
        for key in self._bn_keys():
            P, lv, _ = self._bn_level(key)
            C = P.levels[lv]["C"]
            self.bn_sums[key] = torch.zeros(2 * C, dtype=torch.float32, device=dev)
            self.bn_mi[key] = torch.zeros(2 * C, dtype=torch.float32, device=dev)
            self.bn_gamma[key] = torch.ones(C, dtype=torch.float32, device=dev)
            self.bn_beta[key] = torch.zeros(C, dtype=torch.float32, device=dev)
            ws = max(ws, sc.splitcnn_bn_workspace_size(P.handle, lv))
        self.bn_ws = torch.zeros(ws // 4 + 4, dtype=torch.float32, device=dev)
        self.bn_ws_bytes = self.bn_ws.numel() * 4

    def grad_numel(self) -> int:
        n = super().grad_numel()
        for key in self._bn_keys():
            P, lv, _ = self._bn_level(key)
            n += 2 * P.levels[lv]["C"]
        return n

    def bind_grads(self, flat: torch.Tensor):
        super().bind_grads(flat)
        off = super().grad_numel()
        self.bn_grads = {}
        for key in self._bn_keys():
            P, lv, _ = self._bn_level(key)
            C = P.levels[lv]["C"]
            self.bn_grads[key] = flat[off:off + 2 * C]     # [dbeta; dgamma] = the bn_bwd_sums layout
            off += 2 * C

    def set_bn_params(self, bn_params):
        """bn_params: (gamma, beta) per conv in _bn_keys() order (chain convs, then downsamples)."""
        for key, (gm, bt) in zip(self._bn_keys(), bn_params):
            self.bn_gamma[key].copy_(torch.as_tensor(gm, dtype=torch.float32))
            self.bn_beta[key].copy_(torch.as_tensor(bt, dtype=torch.float32))

    def _inp(self, m):
        """The tensor layer m reads: the BN(+ReLU) output for a conv output level, else the level itself."""
        return self.bn_out.get(m, self.act_r[m]) if m > 0 else self.act_r[0]

    # ------------------------------------------------------------------ BN helpers
    def _bn_fwd(self, key, z, y, relu, stream):
        P, lv, cnt = self._bn_level(key)
        p0, p1 = self.patch_range        # a downsample plan shares its block's patch grid
        nb = z.numel() * z.element_size()
        self._call("bn", nb, sc.splitcnn_bn_stats, P.handle, lv, self.dtype, z, self.bn_sums[key], self.bn_ws,
                   self.bn_ws_bytes, p0, p1, stream)
        if self.bn_reduce is not None:
            self.bn_reduce(self.bn_sums[key])
        self._call("bn", 2 * nb, sc.splitcnn_bn_fwd, P.handle, lv, self.dtype, z, self.bn_sums[key], cnt,
                   self.bn_gamma[key], self.bn_beta[key], self.eps, self.bn_mi[key], y,
                   sc.FLAG_RELU if relu else 0, p0, p1, stream)

    def _bn_bwd(self, key, g, z, y_mask, out, stream):
        """out = dL/dz from g = dL/d(BN output) (y_mask: the BN+ReLU output, or None)."""
        P, lv, cnt = self._bn_level(key)
        p0, p1 = self.patch_range
        nb = z.numel() * z.element_size()
        t = self.bn_grads[key]
        self._call("bn", (3 if y_mask is not None else 2) * nb, sc.splitcnn_bn_bwd_sums, P.handle, lv, self.dtype, g,
                   z, y_mask, self.bn_mi[key], t, self.bn_ws, self.bn_ws_bytes, p0, p1, stream)
        if self.bn_reduce is not None:
            self.bn_reduce(t)
        self._call("bn", (4 if y_mask is not None else 3) * nb, sc.splitcnn_bn_bwd, P.handle, lv, self.dtype, g, z,
                   y_mask, self.bn_mi[key], self.bn_gamma[key], t, cnt, out, p0, p1, stream)

    # ------------------------------------------------------------------ passes
    def forward(self, x: torch.Tensor, stream=None, x_layout: int = sc.NCHW):
        p0, p1 = self.patch_range
        R, dt, fl = self.region.handle, self.dtype, self.flags_extra
        acts, L = self.act_r, self.region_layers
        self._label = "input"
        if self.s2d:
            self._call("split", 2 * self._bytes(self.region, 0)[0], sc.splitcnn_split_s2d, R, 0, dt, x, self.stem_cin,
                       acts[0], p0, p1, stream)
        else:
            self._call("split", 2 * self._bytes(self.region, 0)[0], sc.splitcnn_split, R, 0, dt, x, x_layout, acts[0],
                       p0, p1, stream)

        def conv(m, relu):
            W, _ = self.params[("r", m)]
            self._label = L[m]["name"]
            self._call("conv_fwd", self._conv_work(self.region, m, L[m]), sc.splitcnn_conv_fwd, R, m, dt, self._inp(m),
                       W, None, acts[m + 1], fl, p0, p1, stream)
            self._bn_fwd(("r", m), acts[m + 1], self.bn_out[m + 1], relu, stream)

        m = 0
        while m < len(L):
            if m in self.block_at:
                k = self.block_at[m]
                conv(m, True)
                conv(m + 1, False)
                if k in self.ds_plans:
                    P, lds = self.ds_plans[k], self.blocks[k]["ds"]
                    W, _ = self._ds_params[k]
                    self._label = lds["name"]
                    self._call("conv_fwd", self._conv_work(P, 0, lds), sc.splitcnn_conv_fwd, P.handle, 0, dt,
                               self._inp(m), W, None, self.ds_out[k], fl, p0, p1, stream)
                    self._bn_fwd(("ds", k), self.ds_out[k], self.ds_bn[k], False, stream)
                    s = self.ds_bn[k]
                else:
                    s = self._inp(m)
                self._label = f"{L[m]['name'][:-2]}_add"
                y = self.bn_out[m + 2]
                self._call("add", 3 * y.numel() * y.element_size(), sc.splitcnn_add, R, m + 2, dt, y, s, y, None,
                           sc.FLAG_RELU, p0, p1, stream)
                m += 2
                continue
            if L[m]["op"] == "conv":
                conv(m, True)
            else:
                self._label = L[m]["name"]
                bi, bo = self._bytes(self.region, m)
                self._call("pool_fwd", bi + bo + bo // (2 if dt == sc.BF16 else 4), sc.splitcnn_pool_fwd, R, m, dt,
                           self._inp(m), acts[m + 1], self.argmax[("r", m)], sc.FLAG_POOL_RELU_MASK, p0, p1, stream)
            m += 1
        nl = self.region.nlayers
        self._label = "output"
        self._call("merge", 2 * self._bytes(self.region, nl - 1)[1], sc.splitcnn_merge, R, nl, dt, self._inp(nl),
                   self.out, sc.NHWC, p0, p1, stream)
        return self.out

    def backward(self, dy: torch.Tensor, stream=None, need_input_grad: bool = False):
        p0, p1 = self.patch_range
        R, dt, fl = self.region.handle, self.dtype, self.flags_extra
        acts, L = self.act_r, self.region_layers
        nl = self.region.nlayers
        g = self.grad[0]
        self._label = "output"
        self._call("split", 2 * self._bytes(self.region, nl - 1)[1], sc.splitcnn_split, R, nl, dt, dy, sc.NHWC, g,
                   p0, p1, stream)
        nb = self._bytes(self.region, nl - 1)[1]
        self._call("add", 3 * nb, sc.splitcnn_add, R, nl, dt, g, self.zeros, g, self._inp(nl), 0, p0, p1, stream)

        def conv_bwd(m, gz, want_dx):
            """conv m backward from gz = dL/dz_m: wgrad, and dgrad into a free buffer (unmasked)."""
            W, _ = self.params[("r", m)]
            dW, _ = self.grads[("r", m)]
            wk = self._conv_work(self.region, m, L[m])
            self._label = L[m]["name"]
            out = None
            if want_dx:
                out = self._free(gz, *busy)
                self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, R, m, dt, gz, W, out, None, self.ws,
                           self.ws_bytes, fl, p0, p1, stream)
            self._call("conv_wgrad", wk, sc.splitcnn_conv_bwd_filter, R, m, dt, self._inp(m), gz, dW, None, 0.0,
                       self.ws, self.ws_bytes, fl, p0, p1, stream)
            return out

        busy = []
        m = nl - 1
        while m >= 0:
            a = m - 1
            if a in self.block_at:
                k = self.block_at[a]
                gz = g                                           # dL/d(BN_b out + shortcut), masked
                busy = [gz]
                gzb = self._free(gz)
                self._label = L[a + 1]["name"]
                self._bn_bwd(("r", a + 1), gz, acts[a + 2], None, gzb, stream)
                busy = [gz, gzb]
                gh = conv_bwd(a + 1, gzb, True)                  # dL/dh (h = BN_a+ReLU output), unmasked
                busy = [gz, gh]
                gza = gzb                                        # gzb is consumed: reuse its buffer
                self._label = L[a]["name"]
                self._bn_bwd(("r", a), gh, acts[a + 1], self.bn_out[a + 1], gza, stream)
                busy = [gz, gza]
                gx = conv_bwd(a, gza, True)
                busy = [gz, gx]
                if k in self.ds_plans:
                    P, lds = self.ds_plans[k], self.blocks[k]["ds"]
                    W, _ = self._ds_params[k]
                    dW, _ = self.grads[("ds", k)]
                    gzd = self._free(gz, gx)
                    self._label = lds["name"]
                    self._bn_bwd(("ds", k), gz, self.ds_out[k], None, gzd, stream)
                    gs = self._free(gz, gx, gzd)
                    wk = self._conv_work(P, 0, lds)
                    self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, P.handle, 0, dt, gzd, W, gs, None, self.ws,
                               self.ws_bytes, fl, p0, p1, stream)
                    self._call("conv_wgrad", wk, sc.splitcnn_conv_bwd_filter, P.handle, 0, dt, self._inp(a), gzd, dW,
                               None, 0.0, self.ws, self.ws_bytes, fl, p0, p1, stream)
                else:
                    gs = gz
                mask = self._inp(a) if a in self.block_out else None
                self._label = f"{L[a]['name'][:-2]}_add"
                nb = self._bytes(self.region, a)[0]
                self._call("add", (4 if mask is not None else 3) * nb, sc.splitcnn_add, R, a, dt, gx, gs, gx, mask, 0,
                           p0, p1, stream)
                g = gx
                m = a - 1
                continue
            l = L[m]
            busy = [g]
            if l["op"] == "conv":                                # the stem: g = dL/d(BN+ReLU out), masked
                gz = self._free(g)
                self._label = l["name"]
                self._bn_bwd(("r", m), g, acts[m + 1], None, gz, stream)
                busy = [gz]
                last = m == 0 and not need_input_grad
                out = conv_bwd(m, gz, not last)
                g = out if out is not None else gz
            else:
                out = self._free(g)
                self._label = l["name"]
                bi, bo = self._bytes(self.region, m)
                self._call("pool_bwd", bi + bo + bo // (2 if dt == sc.BF16 else 4), sc.splitcnn_pool_bwd, R, m, dt, g,
                           self.argmax[("r", m)], out, sc.FLAG_POOL_RELU_MASK, p0, p1, stream)
                g = out
            m -= 1
        return g


class ResNet18Net:
    """The whole ResNet-18 trunk: the split region (stem .. layer2, split per the
    config) -> merge at the join (Eq. 7) -> the unsplit tail (layer3, layer4: the same block executor
    on a 1x1 split) -> global average pool.  BN-free by default, `bn=True` puts whole-tensor BN after
    every conv.  forward(x NCHW) -> [N][C] pooled features; backward(dY [N][C]).  No FC head (the
    benchmark drives backward with a synthetic dY)."""

    def __init__(self, region_chain, region_blocks, tail_chain, tail_blocks, N, C, H, W, split=(2, 2), bn=False,
                 dtype: int = sc.BF16, device="cuda"):
        cls = ResBNSplitNet if bn else ResSplitNet
        self.net_r = cls(region_chain, region_blocks, N, C, H, W, split=split, dtype=dtype, device=device)
        L = self.net_r.region.levels[-1]
        self.net_t = cls(tail_chain, tail_blocks, N, L["C"], L["H"], L["W"], split=(1, 1), dtype=dtype, device=device)
        self.dtype, self.tdtype, self.device = dtype, self.net_r.tdtype, self.net_r.device
        self.N = N
        Lt = self.net_t.region.levels[-1]
        self.C_out = Lt["C"]
        self.pooled = torch.zeros(N * Lt["Cpad"], dtype=self.tdtype, device=self.device)
        self.g_out = torch.zeros(Lt["total_elems"], dtype=self.tdtype, device=self.device)
        self.step_index = 0
        self.input_grad = False
        n_r, n_t = self.net_r.grad_numel(), self.net_t.grad_numel()
        self.bind_grads(torch.zeros(n_r + n_t, dtype=torch.float32, device=self.device))

    def bind_grads(self, flat):
        n_r = self.net_r.grad_numel()
        self.grad_flat = flat
        self.net_r.bind_grads(flat[:n_r])
        self.net_t.bind_grads(flat[n_r:])

    @property
    def timers(self):
        return self.net_r.timers

    @timers.setter
    def timers(self, v):
        self.net_r.timers = v
        self.net_t.timers = v

    def set_params(self, params):
        params = list(params)
        n_r = sum(1 for l in self.net_r.region_layers if l["op"] == "conv") + len(self.net_r.ds_plans)
        self.net_r.set_params(params[:n_r])
        self.net_t.set_params(params[n_r:])

    def set_bn_params(self, bn_params):
        if not hasattr(self.net_r, "_bn_keys"):
            return                               # BN-free trunk
        bn_params = list(bn_params)
        n_r = len(self.net_r._bn_keys())
        self.net_r.set_bn_params(bn_params[:n_r])
        self.net_t.set_bn_params(bn_params[n_r:])

    def output_numel(self) -> int:
        return self.pooled.numel()

    def forward(self, x, stream=None):
        y = self.net_r.forward(x, stream)                          # merged NHWC join tensor
        z = self.net_t.forward(y, stream, sc.NHWC)                 # merged NHWC tail output
        T = self.net_t.region
        self.net_t._label = "gap"
        self.net_t._call("gap", z.numel() * z.element_size(), sc.splitcnn_gap_fwd, T.handle, T.nlayers, self.dtype, z,
                         self.pooled, stream)
        return self.pooled

    def backward(self, dy, stream=None, need_input_grad: bool = False):
        T = self.net_t.region
        self.net_t._label = "gap"
        self.net_t._call("gap", self.g_out.numel() * self.g_out.element_size(), sc.splitcnn_gap_bwd, T.handle,
                         T.nlayers, self.dtype, dy, self.g_out, stream)
        g = self.net_t.backward(self.g_out, stream, need_input_grad=True)    # tail level 0 = merged NHWC
        return self.net_r.backward(g, stream, need_input_grad)

    def step(self, x, dy, stream=None):
        self.forward(x, stream)
        self.backward(dy, stream, self.input_grad)
        self.step_index += 1

    def conv_flops(self) -> int:
        return self.net_r.conv_flops() + self.net_t.conv_flops()

    def grad_of(self, i):
        """OIHW weight gradient of conv i in resnet_params order (region chain, region ds, tail chain, tail ds)."""
        keys = [(self.net_r, k) for k in self.net_r._conv_keys()] + [(self.net_t, k) for k in self.net_t._conv_keys()]
        net, key = keys[i]
        return net.grad_oihw(key), net.grads[key][1]
