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


class ResSplitNet(SplitNet):
    def __init__(self, chain: list[dict], blocks: list[dict], N: int, C: int, H: int, W: int, split=(2, 2),
                 dtype: int = sc.BF16, device="cuda", force_simt: bool = False, **kw):
        self.blocks = blocks
        self.block_at = {b["a"]: k for k, b in enumerate(blocks)}
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
        super().set_params(params[:nchain])
        for (k, l, p), (W, b) in zip(self._ds_layers(), params[nchain:]):
            W = torch.as_tensor(W).to(self.device)
            self._ds_params[k][0].copy_(pack_weight(W, p.levels[0]["Cpad"], self.tdtype))
            self._ds_params[k][1].copy_(torch.as_tensor(b, dtype=torch.float32))

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
        self._label = "input"
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
                for mm, ll in ((m, la), (m + 1, lb)):
                    W, b = self.params[("r", mm)]
                    self._label = ll["name"]
                    self._call("conv_fwd", self._conv_work(self.region, mm, ll), sc.splitcnn_conv_fwd, R, mm, dt,
                               acts[mm], W, b, acts[mm + 1], (sc.FLAG_RELU if ll["relu"] else 0) | fl, p0, p1, stream)
                if k in self.ds_plans:
                    P, lds = self.ds_plans[k], self.blocks[k]["ds"]
                    W, b = self._ds_params[k]
                    self._label = lds["name"]
                    self._call("conv_fwd", self._conv_work(P, 0, lds), sc.splitcnn_conv_fwd, P.handle, 0, dt,
                               acts[m], W, b, self.ds_out[k], fl, p0, p1, stream)
                    sc_src = self.ds_out[k]
                else:
                    sc_src = acts[m]
                self._label = f"{la['name'][:-2]}_add"
                nb = self._bytes(self.region, m + 1)[1]
                self._call("add", 3 * nb, sc.splitcnn_add, R, m + 2, dt, acts[m + 2], sc_src, acts[m + 2], None,
                           sc.FLAG_RELU, p0, p1, stream)
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
                self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, R, a + 1, dt, gz, W, gh, acts[a + 1], self.ws,
                           self.ws_bytes, fl, p0, p1, stream)
                self._call("conv_wgrad", wk, sc.splitcnn_conv_bwd_filter, R, a + 1, dt, acts[a + 1], gz, dW, db, 0.0,
                           self.ws, self.ws_bytes, fl, p0, p1, stream)
                gx = self._free(gz, gh)
                W, _ = self.params[("r", a)]
                dW, db = self.grads[("r", a)]
                wk = self._conv_work(self.region, a, la)
                self._label = la["name"]
                self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, R, a, dt, gh, W, gx, None, self.ws,
                           self.ws_bytes, fl, p0, p1, stream)
                self._call("conv_wgrad", wk, sc.splitcnn_conv_bwd_filter, R, a, dt, acts[a], gh, dW, db, 0.0,
                           self.ws, self.ws_bytes, fl, p0, p1, stream)
                if k in self.ds_plans:
                    P, lds = self.ds_plans[k], self.blocks[k]["ds"]
                    W, _ = self._ds_params[k]
                    dW, db = self.grads[("ds", k)]
                    gs = self._free(gz, gh, gx)
                    wk = self._conv_work(P, 0, lds)
                    self._label = lds["name"]
                    self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, P.handle, 0, dt, gz, W, gs, None, self.ws,
                               self.ws_bytes, fl, p0, p1, stream)
                    self._call("conv_wgrad", wk, sc.splitcnn_conv_bwd_filter, P.handle, 0, dt, acts[a], gz, dW, db,
                               0.0, self.ws, self.ws_bytes, fl, p0, p1, stream)
                else:
                    gs = gz
                mask = acts[a] if self._masked("r", a) else None
                self._label = f"{la['name'][:-2]}_add"
                nb = self._bytes(self.region, a)[0]
                self._call("add", (4 if mask is not None else 3) * nb, sc.splitcnn_add, R, a, dt, gx, gs, gx, mask, 0,
                           p0, p1, stream)
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
                    self._call("conv_dgrad", wk, sc.splitcnn_conv_bwd_data, R, m, dt, g, W, out,
                               acts[m] if self._masked("r", m) else None, self.ws, self.ws_bytes, fl, p0, p1, stream)
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
