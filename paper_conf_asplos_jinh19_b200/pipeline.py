"""Host-fed training steps with the copies overlapped: the public end-to-end API.

    pipe = HostPipeline(net)                    # net: SplitNet / ResSplitNet / DistSplitNet-like
    for xh, dyh in batches:                     # pinned host tensors
        pipe.submit(xh, dyh, grads_host)        # H2D of this step's inputs, the step, D2H of its grads
    pipe.synchronize()

Step i's inputs are copied host->device on an H2D stream into one of two device buffers while step
i-1 still computes; step i's weight / bias gradients (the executor's flat fp32 buffer, of which there
are also two, alternated per step) are copied device->host on a D2H stream while step i+1 computes.
Events order every reuse: a device input buffer is refilled only after the step that read it, a
gradient buffer is rewritten only after its D2H finished.  Results are bitwise those of
net.step on the same inputs (the same kernels in the same order on the compute stream).
"""
from __future__ import annotations

import torch


class HostPipeline:
    def __init__(self, net, x_like: torch.Tensor | None = None, dy_numel: int | None = None, graphs: bool = False):
        self.net = net
        self.graphs = [None, None] if graphs else None   # one CUDA graph per buffer parity (fixed pointers)
        dev = net.device
        self.compute = torch.cuda.current_stream(dev)
        self.h2d = torch.cuda.Stream(dev)
        self.d2h = torch.cuda.Stream(dev)
        self.x = None if x_like is None else [torch.empty_like(x_like, device=dev) for _ in range(2)]
        n = dy_numel if dy_numel is not None else net.output_numel()
        self.dy = [torch.empty(n, dtype=net.tdtype, device=dev) for _ in range(2)]
        self.g = [net.grad_flat, torch.zeros_like(net.grad_flat)]
        ev = lambda: [torch.cuda.Event() for _ in range(2)]
        self.in_ready, self.in_free, self.g_ready, self.g_free = ev(), ev(), ev(), ev()
        self.used = [False, False]
        self.i = 0

    def submit(self, xh: torch.Tensor, dyh: torch.Tensor, grads_host: torch.Tensor | None = None):
        b = self.i & 1
        if self.x is None:
            self.x = [torch.empty(xh.shape, dtype=xh.dtype, device=self.net.device) for _ in range(2)]
        with torch.cuda.stream(self.h2d):
            if self.used[b]:
                self.h2d.wait_event(self.in_free[b])      # the step that last read these buffers is done
            self.x[b].copy_(xh, non_blocking=True)
            self.dy[b].copy_(dyh.reshape(-1), non_blocking=True)
            self.in_ready[b].record(self.h2d)
        self.compute.wait_event(self.in_ready[b])
        if self.used[b]:
            self.compute.wait_event(self.g_free[b])       # this gradient buffer's D2H has finished
        self.net.bind_grads(self.g[b])
        if self.graphs is not None:
            if self.graphs[b] is None:
                self.graphs[b] = self._capture(b)
            self.graphs[b].replay()
        else:
            self.net.step(self.x[b], self.dy[b], self.compute)
        self.in_free[b].record(self.compute)
        self.g_ready[b].record(self.compute)
        if grads_host is not None:
            # a sharded executor reads back only its slice of the (allreduced) gradient
            lo, hi = self.net.grad_slice() if hasattr(self.net, "grad_slice") else (0, self.g[b].numel())
            with torch.cuda.stream(self.d2h):
                self.d2h.wait_event(self.g_ready[b])
                grads_host.copy_(self.g[b][lo:hi], non_blocking=True)
                self.g_free[b].record(self.d2h)
        else:
            self.g_free[b].record(self.compute)
        self.used[b] = True
        self.i += 1
        return self.g[b]

    def _capture(self, b):
        """Capture one step on buffers (x[b], dy[b], g[b]) as a CUDA graph (a static plan: even split)."""
        side = torch.cuda.Stream(self.net.device)
        side.wait_stream(self.compute)
        with torch.cuda.stream(side):
            self.net.step(self.x[b], self.dy[b])           # warm-up outside the capture
        self.compute.wait_stream(side)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            self.net.step(self.x[b], self.dy[b])
        return g

    def synchronize(self):
        self.compute.synchronize()
        self.h2d.synchronize()
        self.d2h.synchronize()
