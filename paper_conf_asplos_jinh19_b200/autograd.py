"""torch.nn front end: a Split-CNN conv stack as a differentiable module (SURVEY §1 layer L4).

    stack = SplitStack(region_layers, tail_layers, N, C, H, W, split=(8, 8))
    y = stack(x)                 # NCHW input -> the executor's output buffer (NHWC / patch buffers)
    (y * g).sum().backward()     # x.grad (if requested) and every weight / bias .grad

The module owns its parameters in the library layout (weights [Cout][kh][kw][Cpad_in] in the compute
dtype, biases fp32) and binds them to the executor's parameter slots, so an optimizer updating them
in place is seen by the next step.  forward / backward are the executor's passes (every step is a
libsplitcnn call); autograd only routes tensors.  Gradients come from the executor's fp32 buffer and
are handed to autograd in the parameters' dtype.

Per-op front end on patch buffers of one SplitPlan (level m -> m + 1), for composing a split stack
by hand: SplitConv2d(plan, m) (conv fwd [+ReLU] / dgrad / wgrad) and SplitMaxPool2d(plan, m).
"""
from __future__ import annotations

import torch

from . import splitcnn as sc
from .net import SplitNet


class _SplitStackFn(torch.autograd.Function):
    @staticmethod
    def forward(ctx, module, x, *params):
        net = module.net
        net.replan(net.step_index)
        out = net.forward(x.contiguous())
        ctx.module = module
        ctx.x_shape = x.shape
        return out.clone()          # executor buffers are reused by the next step

    @staticmethod
    def backward(ctx, dy):
        module = ctx.module
        net = module.net
        need_dx = ctx.needs_input_grad[1]
        g = net.backward(dy.contiguous().to(net.tdtype), need_input_grad=need_dx)
        net.step_index += 1
        dx = None
        if need_dx:
            # g is the gradient of the first level (patch buffers): back to the NCHW input layout
            full = torch.empty(ctx.x_shape, dtype=net.tdtype, device=dy.device)
            sc.splitcnn_merge(net.region.handle, 0, net.dtype, g, full, sc.NCHW)
            dx = full
        grads = []
        for key in module.keys:
            dW, db = net.grads[key]
            grads += [dW.to(module.weight(key).dtype), db.clone()]
        return (None, dx, *grads)


class SplitStack(torch.nn.Module):
    def __init__(self, region: list[dict], tail: list[dict], N: int, C: int, H: int, W: int, **kw):
        super().__init__()
        self.net = SplitNet(region, tail, N, C, H, W, **kw)
        self.keys = sorted(self.net.params, key=lambda k: (k[0] != "r", k[1]))
        for i, key in enumerate(self.keys):
            Wt, b = self.net.params[key]
            self.register_parameter(f"w{i}", torch.nn.Parameter(Wt, requires_grad=True))
            self.register_parameter(f"b{i}", torch.nn.Parameter(b, requires_grad=True))
            self.net.params[key] = (getattr(self, f"w{i}"), getattr(self, f"b{i}"))   # same storage

    def weight(self, key):
        return getattr(self, f"w{self.keys.index(key)}")

    def set_params(self, params):
        """(W_oihw, b) per conv, region then tail order (as SplitNet.set_params)."""
        with torch.no_grad():
            self.net.set_params(params)

    def forward(self, x):
        flat = [p for key in self.keys for p in (self.weight(key), getattr(self, f"b{self.keys.index(key)}"))]
        return _SplitStackFn.apply(self, x, *flat)


# --------------------------------------------------------------------------- per-op autograd front end
class _SplitConvFn(torch.autograd.Function):
    """One split convolution on patch buffers (level `layer` -> level `layer` + 1 of `plan`)."""

    @staticmethod
    def forward(ctx, x, w, b, plan, layer, dtype, relu, ws):
        lo = plan.levels[layer + 1]
        y = torch.empty(lo["total_elems"], dtype=x.dtype, device=x.device)
        sc.splitcnn_conv_fwd(plan.handle, layer, dtype, x, w, b, y, sc.FLAG_RELU if relu else 0)
        ctx.save_for_backward(x, w, y if relu else None)
        ctx.plan, ctx.layer, ctx.dtype, ctx.relu, ctx.ws = plan, layer, dtype, relu, ws
        return y

    @staticmethod
    def backward(ctx, gy):
        x, w, y = ctx.saved_tensors
        plan, layer, dtype, ws = ctx.plan, ctx.layer, ctx.dtype, ctx.ws
        gy = gy.contiguous()
        if ctx.relu:      # ReLU backward on the output: dY * [y > 0] (the library's masked sum with zeros)
            gz = torch.empty_like(gy)
            sc.splitcnn_add(plan.handle, layer + 1, dtype, gy, torch.zeros_like(gy), gz, y)
            gy = gz
        dx = None
        if ctx.needs_input_grad[0]:
            dx = torch.empty_like(x)
            sc.splitcnn_conv_bwd_data(plan.handle, layer, dtype, gy, w, dx, None, ws, ws.numel())
        dw = torch.zeros(w.shape, dtype=torch.float32, device=w.device)
        db = torch.zeros(w.shape[0], dtype=torch.float32, device=w.device)
        sc.splitcnn_conv_bwd_filter(plan.handle, layer, dtype, x, gy, dw, db, 0.0, ws, ws.numel())
        return dx, dw.to(w.dtype), db, None, None, None, None, None


class _SplitPoolFn(torch.autograd.Function):
    @staticmethod
    def forward(ctx, x, plan, layer, dtype):
        lo = plan.levels[layer + 1]
        y = torch.empty(lo["total_elems"], dtype=x.dtype, device=x.device)
        a = torch.empty(lo["total_elems"], dtype=torch.uint8, device=x.device)
        sc.splitcnn_pool_fwd(plan.handle, layer, dtype, x, y, a, 0)
        ctx.save_for_backward(a)
        ctx.plan, ctx.layer, ctx.dtype, ctx.n_in = plan, layer, dtype, x.numel()
        ctx.mark_non_differentiable(a)
        return y

    @staticmethod
    def backward(ctx, gy):
        (a,) = ctx.saved_tensors
        dx = torch.empty(ctx.n_in, dtype=gy.dtype, device=gy.device)
        sc.splitcnn_pool_bwd(ctx.plan.handle, ctx.layer, ctx.dtype, gy.contiguous(), a, dx, 0)
        return dx, None, None, None


class SplitConv2d(torch.nn.Module):
    """Split convolution of layer `layer` of a SplitPlan, on patch buffers (library weight layout
    [Cout][kh][kw][Cpad_in]); forward / backward are splitcnn_conv_fwd / _bwd_data / _bwd_filter."""

    def __init__(self, plan, layer: int, dtype: int = sc.BF16, relu: bool = True, device="cuda"):
        super().__init__()
        l, lv = plan.layer_dicts[layer], plan.levels[layer]
        td = torch.bfloat16 if dtype == sc.BF16 else torch.float32
        self.plan, self.layer, self.dtype, self.relu = plan, layer, dtype, relu
        self.weight = torch.nn.Parameter(torch.zeros((l["cout"], l["kh"], l["kw"], lv["Cpad"]), dtype=td, device=device))
        self.bias = torch.nn.Parameter(torch.zeros(l["cout"], dtype=torch.float32, device=device))
        nbytes = max(plan.workspace_size(layer, dtype, 1), plan.workspace_size(layer, dtype, 2), 16)
        self.register_buffer("ws", torch.empty(nbytes, dtype=torch.uint8, device=device), persistent=False)

    def forward(self, x):
        return _SplitConvFn.apply(x, self.weight, self.bias, self.plan, self.layer, self.dtype, self.relu, self.ws)


class SplitMaxPool2d(torch.nn.Module):
    def __init__(self, plan, layer: int, dtype: int = sc.BF16):
        super().__init__()
        self.plan, self.layer, self.dtype = plan, layer, dtype

    def forward(self, x):
        return _SplitPoolFn.apply(x, self.plan, self.layer, self.dtype)
