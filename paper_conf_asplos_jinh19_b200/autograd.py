"""torch.nn front end: a Split-CNN conv stack as a differentiable module (SURVEY §1 layer L4).

    stack = SplitStack(region_layers, tail_layers, N, C, H, W, split=(8, 8))
    y = stack(x)                 # NCHW input -> the executor's output buffer (NHWC / patch buffers)
    (y * g).sum().backward()     # x.grad (if requested) and every weight / bias .grad

The module owns its parameters in the library layout (weights [Cout][kh][kw][Cpad_in] in the compute
dtype, biases fp32) and binds them to the executor's parameter slots, so an optimizer updating them
in place is seen by the next step.  forward / backward are the executor's passes (every step is a
libsplitcnn call); autograd only routes tensors.  Gradients come from the executor's fp32 buffer and
are handed to autograd in the parameters' dtype.
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
