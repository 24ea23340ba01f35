"""Patch-granular activation offload / prefetch (the HMMS idea, section 4.3).

Four moments per offloaded tensor-storage object, here a level's patch buffers:
  1. start of offload  : right when the op that reads it as input starts (its producer has finished),
                         one `splitcnn_offload` (D2H cudaMemcpyAsync) per patch on an idle memory stream;
  2. end of offload    : at the op Algorithm 1 picks (balance >= 0 or last op) the compute stream waits on
                         the copies' events and the device buffer is freed (returned to the allocator);
  3. start of prefetch : at the backward op the reverse pass picks, a device buffer is allocated
                         and `splitcnn_prefetch` (H2D) runs per patch on a memory stream;
  4. end of prefetch   : the compute stream waits on those events right before the first backward use.
Planning: per-op times are profiled as the mean of 20 repetitions (CUDA events instead of
high_resolution_clock), the host-link bandwidth is MEASURED with pinned copies, and
`splitcnn_offload_plan` / `splitcnn_prefetch_plan` (Algorithm 1 + its reverse pass) decide.
Levels that only feed a max-pool are not needed in backward (the pool keeps its argmax) and are freed
right after the pool (the reference-count release of P:197-203, restricted to the split region).
"""
from __future__ import annotations

import torch

from . import splitcnn as sc
from .net import SplitNet


def measure_host_bandwidth(nbytes: int = 256 << 20, reps: int = 5) -> tuple[float, float]:
    """Pinned D2H and H2D bandwidth in bytes/s (the 'nvlink_bandwidth' of Algorithm 1, here PCIe)."""
    dev = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    host = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    out = []
    for d2h in (True, False):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        (host.copy_(dev, non_blocking=True) if d2h else dev.copy_(host, non_blocking=True))
        torch.cuda.synchronize()
        e0.record()
        for _ in range(reps):
            (host.copy_(dev, non_blocking=True) if d2h else dev.copy_(host, non_blocking=True))
        e1.record()
        torch.cuda.synchronize()
        out.append(nbytes * reps / (e0.elapsed_time(e1) / 1e3))
    return out[0], out[1]


class OffloadSplitNet(SplitNet):
    """SplitNet whose split-region activations are offloaded / prefetched per Algorithm 1."""

    def __init__(self, *args, offload: bool = True, **kw):
        # fused conv -> pool pairs are ONE forward op of the planner's serialized list (their conv
        # output level is never materialised); the backward list stays one op per layer
        super().__init__(*args, **kw)
        self.offload_enabled = offload
        L = self.region.nlayers
        # levels needed in backward: inputs of region convs (wgrad input, ReLU mask of the dgrad)
        self.needed = [m < L and self.region_layers[m]["op"] == "conv" for m in range(L + 1)]
        self.needed[L] = True                         # the join / tail input
        self.level_bytes = [a.numel() * a.element_size() for a in self.act_r]
        self.host = {}
        self.plan_ready = False
        self.d2h = [torch.cuda.Stream(), torch.cuda.Stream()]   # R15: two memory streams each way
        self.h2d = [torch.cuda.Stream(), torch.cuda.Stream()]
        self.stats = {}

    # ------------------------------------------------------------------ op indexing
    def _all_ops(self):
        ops = [("r", m) for m in range(len(self.region_layers))]
        if self.tail:
            ops += [("t", m) for m in range(len(self.tail_layers))]
        return ops

    def _fwd_ops(self):
        """Serialized forward ops: a fused conv -> pool pair (key, m) is one op (its pool half m+1 skipped)."""
        skip = {(k, m + 1) for k, m in self.fused}
        return [op for op in self._all_ops() if op not in skip]

    def _bwd_ops(self):
        return list(reversed(self._all_ops()))

    # ------------------------------------------------------------------ profiling + planning
    def profile_and_plan(self, x, dy, reps: int = 20, bw: float | None = None):
        """Profiling stage: mean of `reps` timed executions per op; then Algorithm 1."""
        saved = self.offload_enabled
        self.offload_enabled = False
        if self.static_pool and getattr(self, "_bwd_view", None) is not None:
            torch.cuda.synchronize()
            self._fwd_view = self._bwd_view = None
            self._alloc_static()                        # back to the plain plan while profiling
        self.timers = []
        for _ in range(reps):
            self.forward(x)
            self.backward(dy)
        torch.cuda.synchronize()
        fwd_t, bwd_t = {}, {}
        ops = self._fwd_ops()
        # per-op mean times from the events recorded around every library call (split/merge ignored)
        for kind, e0, e1, _work, label in self.timers:
            if kind in ("conv_fwd", "pool_fwd"):
                d = fwd_t
            elif kind in ("conv_dgrad", "conv_wgrad", "pool_bwd"):
                d = bwd_t
            else:
                continue
            d[label] = d.get(label, 0.0) + e0.elapsed_time(e1) / 1e3 / reps
        self.timers = None
        self.offload_enabled = saved
        nm = lambda k, m: (self.region_layers if k == "r" else self.tail_layers)[m].get("name", f"{k}{m}")
        op_t = [fwd_t.get(nm(k, m), 0.0) for k, m in ops]
        op_bt = [bwd_t.get(nm(k, m), 0.0) for k, m in self._bwd_ops()]
        if bw is None:
            d2h, h2d = measure_host_bandwidth()
            bw = min(d2h, h2d)
        self.bw = bw
        cand = [0] * len(ops)
        for t, (k, m) in enumerate(ops):
            if k == "r" and self.needed[m]:
                cand[t] = self.level_bytes[m]
        off, sync = sc.splitcnn_offload_plan(op_t, cand, bw)
        self.offload_at = {ops[t]: bool(off[t]) for t in range(len(ops))}
        self.sync_at = {ops[t]: bool(sync[t]) for t in range(len(ops))}
        # reverse pass: an offloaded level m is first needed by the backward op of region conv m
        bops = self._bwd_ops()
        need = [0] * len(bops)
        for u, (k, m) in enumerate(bops):
            if k == "r" and self.offload_at.get(("r", m)):
                need[u] = self.level_bytes[m]
        start = sc.splitcnn_prefetch_plan(op_bt, need, bw)
        self.prefetch_at = {}
        for u, (k, m) in enumerate(bops):
            if need[u]:
                self.prefetch_at.setdefault(bops[start[u]], []).append(m)
        self.stats = dict(op_time_fwd_s=op_t, op_time_bwd_s=op_bt, bw_bytes_per_s=bw,
                          offloaded_levels=[m for (k, m), v in self.offload_at.items() if v],
                          offloaded_bytes=sum(c for c, o in zip(cand, off) if o),
                          candidate_bytes=sum(cand), cap_bytes=sum(op_t) * bw)
        self._alloc_host_pool()
        self.plan_ready = True
        self._pending = []
        self._inflight = {}
        self._rr = 0
        if self.static_pool:
            self._alloc_static_offload()
        return self.stats

    def _alloc_host_pool(self):
        """HMMS host general-purpose pool: ONE pinned allocation holds every offloaded level,
        placed by the same first-fit planner over the host TSOs' lives -- from the forward op whose D2H
        starts it to the backward op that first reads the prefetched level (serialized step order)."""
        lvls = self.stats["offloaded_levels"]
        if not lvls:
            self.host, self.host_pool_bytes = {}, 0
            return
        fops, bops = self._fwd_ops(), self._bwd_ops()
        fidx = {op: t for t, op in enumerate(fops)}
        bidx = {op: len(fops) + u for u, op in enumerate(bops)}
        first = [fidx[("r", m)] for m in lvls]
        last = [bidx[("r", m)] for m in lvls]
        sizes = [self.level_bytes[m] for m in lvls]
        offs, pool = sc.splitcnn_memplan(sizes, first, last, 4096)
        if getattr(self, "host_pool_bytes", -1) != pool:
            self.host_pool = torch.empty(max(pool, 4096), dtype=torch.uint8, pin_memory=True)
            self.host_pool_bytes = pool
        self.host = {m: self.host_pool[o:o + b] for m, o, b in zip(lvls, offs, sizes)}

    def _alloc_static_offload(self):
        """HMMS static planning WITH the offload schedule (memory is held 'only for the minimum
        duration required mandated both by the reference counter and the previously computed offloading
        and prefetching scheme'): an offloaded level becomes two TSOs -- its forward life (producer op
        .. the Algorithm-1 sync op that ends its D2H) and its backward life (the op whose prefetch
        starts its H2D .. its last backward use) -- so the arena reuses its space in between."""
        torch.cuda.synchronize()
        sched, names, first, last = self._tso_lifetimes()
        idx = {op: t for t, (op, _) in enumerate(sched)}
        fname = lambda k, m: f"{k}{m}+pool" if (k, m) in self.fused else f"{k}{m}"
        pending, freed_at = [], {}
        for k, m in self._fwd_ops():                       # replay the forward hooks' bookkeeping
            if self.offload_at.get((k, m)):
                pending.append(m)
            if self.sync_at.get((k, m)) and pending:
                for lvl in pending:
                    freed_at[lvl] = idx[fname(k, m)]
                pending = []
        pre_at = {lvl: idx[f"{k}{m}'"] for (k, m), lvls in self.prefetch_at.items() for lvl in lvls}
        names2, first2, last2 = [], {}, {}
        for n in names:
            lvl = n[2]
            if n[0] == "a" and n[1] == "r" and lvl in freed_at and lvl in pre_at:
                nf, nb = ("aF", "r", lvl), ("aB", "r", lvl)
                names2 += [nf, nb]
                first2[nf], last2[nf] = first[n], max(first[n], freed_at[lvl])
                first2[nb], last2[nb] = pre_at[lvl], last[n]
            else:
                names2.append(n)
                first2[n], last2[n] = first[n], last[n]
        self._alloc_static((names2, first2, last2))
        self._fwd_view = {m: self.act_r[m] for m in range(len(self.act_r))}
        self._bwd_view = {n[2]: v for n, v in self.static_views.items() if n[0] == "aB"}

    # ------------------------------------------------------------------ hooks
    def _ensure(self, m):
        if self.act_r[m] is None and getattr(self, "_fwd_view", None) is not None:
            self.act_r[m] = self._fwd_view[m]             # static arena: the level's (forward) view
            return
        if self.act_r[m] is None:
            self.act_r[m] = torch.empty(self.level_bytes[m] // (2 if self.dtype == sc.BF16 else 4),
                                        dtype=self.tdtype, device=self.device)

    def forward(self, x, stream=None, x_layout: int = sc.NCHW):
        if getattr(self, "_bwd_view", None) and not self.offload_enabled:
            raise RuntimeError("the offload-aware static plan needs offload_enabled (re-run profile_and_plan)")
        self._ensure(0)
        if not (self.offload_enabled and self.plan_ready):
            for m in range(len(self.act_r)):
                self._ensure(m)
        return super().forward(x, stream, x_layout)

    def hook_before_fwd(self, key, m):
        if key == "r":
            self._ensure(m + 1)      # allocate a level right before the op that produces it
            if (key, m) in self.fused:
                self._ensure(m + 2)  # a fused pair produces the pool output level
        if not (self.offload_enabled and self.plan_ready) or not self.offload_at.get((key, m)):
            return
        # moment 1: the input level of op m is final -> D2H per patch on an idle memory stream
        ready = torch.cuda.Event()
        ready.record()
        mem = self.d2h[self._rr % 2]
        self._rr += 1
        nq = self.region.npatch
        host = self.host[m]
        for q in range(nq):
            off, nb = sc.splitcnn_patch_bytes(self.region.handle, m, self.dtype, q)
            sc.splitcnn_offload(self.region.handle, m, self.dtype, q, self.act_r[m], host.data_ptr() + off,
                                ready if q == 0 else None, mem, None)
        # torch creates an event's CUDA handle lazily at its first record(): record it here, on `mem`
        done = torch.cuda.Event()
        done.record(mem)
        self._pending.append((m, done, mem))

    def hook_after_fwd(self, key, m):
        if not (self.offload_enabled and self.plan_ready):
            return
        if key == "r" and m + 1 < len(self.act_r) and not self.needed[m] and m > 0:
            # a level read only by this max-pool: release it (not needed in backward)
            if self.region_layers[m]["op"] == "maxpool":
                self.act_r[m] = None
        if self.sync_at.get((key, m)) and self._pending:
            # moment 2: the compute stream waits for the outstanding offloads, then frees them
            cur = torch.cuda.current_stream()
            for lvl, done, mem in self._pending:
                cur.wait_event(done)
                if getattr(self, "_fwd_view", None) is None:
                    self.act_r[lvl].record_stream(mem)
                self.act_r[lvl] = None
            self._pending = []

    def hook_before_bwd(self, key, m):
        if not (self.offload_enabled and self.plan_ready):
            return
        cur = torch.cuda.current_stream()
        for lvl in self.prefetch_at.get((key, m), []):
            # moment 3: allocate (static arena: the level's backward view) and start H2D per patch
            if getattr(self, "_bwd_view", None) is not None and lvl in self._bwd_view:
                self.act_r[lvl] = self._bwd_view[lvl]
            self._ensure(lvl)
            ready = torch.cuda.Event()
            ready.record()
            mem = self.h2d[self._rr % 2]
            self._rr += 1
            nq = self.region.npatch
            for q in range(nq):
                off, nb = sc.splitcnn_patch_bytes(self.region.handle, lvl, self.dtype, q)
                sc.splitcnn_prefetch(self.region.handle, lvl, self.dtype, q, self.host[lvl].data_ptr() + off,
                                     self.act_r[lvl], ready if q == 0 else None, mem, None)
            done = torch.cuda.Event()
            done.record(mem)
            if getattr(self, "_fwd_view", None) is None:
                self.act_r[lvl].record_stream(mem)
            self._inflight[lvl] = done
        if key == "r" and m in self._inflight:
            # moment 4: the compute stream waits right before the first backward use
            cur.wait_event(self._inflight.pop(m))

    def hook_after_bwd(self, key, m):
        # a region conv's input level is dead after its backward until the next forward rewrites it
        if self.offload_enabled and self.plan_ready and key == "r" and self.region_layers[m]["op"] == "conv":
            self.act_r[m] = None
