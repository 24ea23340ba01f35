"""SplitNet -- executes a Split-CNN conv stack (split region + unsplit tail) through libsplitcnn.

A step is one pass of the hot path: split (Eq. 4) -> per-patch conv / max-pool
forward (Eq. 6) through the chained split region -> merge at the join (Eq. 7) -> the
unsplit tail (a 1x1 "split", i.e. ordinary layers) -> backward in reverse order: pool backward,
conv data gradient (ReLU mask fused), conv weight gradient summed over patches and batch.
PyTorch only allocates device memory and provides the stream; every step runs in libsplitcnn.
"""
from __future__ import annotations

import torch

from . import splitcnn as sc
from .plan import SplitPlan

TORCH_DTYPE = {sc.BF16: torch.bfloat16, sc.FP32: torch.float32, sc.TF32: torch.float32}


def pack_weight(W_oihw: torch.Tensor, cpad_in: int, dtype) -> torch.Tensor:
    """OIHW -> the library layout [Cout][kh][kw][Cpad_in] (zero channel padding); parameter setup."""
    co, ci, kh, kw = W_oihw.shape
    out = torch.zeros((co, kh, kw, cpad_in), dtype=dtype, device=W_oihw.device)
    out[..., :ci] = W_oihw.permute(0, 2, 3, 1).to(dtype)
    return out


def unpack_grad(dW: torch.Tensor, cin: int) -> torch.Tensor:
    """[Cout][kh][kw][Cpad_in] -> OIHW."""
    return dW[..., :cin].permute(0, 3, 1, 2)


class SplitNet:
    def __init__(self, region: list[dict], tail: list[dict], N: int, C: int, H: int, W: int,
                 split=(2, 2), mode: str = "even", omega: float = 0.2, seed: int = 0,
                 dtype: int = sc.BF16, device="cuda", patch_range=None, force_simt: bool = False,
                 grad_buffer: torch.Tensor | None = None, input_relu: bool = False, fuse_pool: bool = True,
                 static_pool: bool = False, input_grad: bool = False, mask_output_grad: bool = True,
                 concurrent_wgrad: bool = True, schedule: str = "layer", group_rows: int = 1,
                 prep_dgrad_weights: bool = False):
        self.region_layers, self.tail_layers = region, tail
        self.N, self.C, self.H, self.W = N, C, H, W
        self.split, self.mode, self.omega, self.seed = split, mode, omega, seed
        self.dtype, self.tdtype, self.device = dtype, TORCH_DTYPE[dtype], torch.device(device)
        self.flags_extra = sc.FLAG_FORCE_SIMT if force_simt else 0
        self.input_relu = input_relu   # level 0 is a ReLU output (e.g. a tail fed by a ReLU conv)
        self.fuse_pool = fuse_pool and dtype == sc.BF16 and not force_simt
        self.step_index = 0
        self.static_pool = static_pool   # HMMS static memory plan: one arena, first-fit offsets
        self.input_grad = input_grad  # step(): also compute dX of the first layer (C1's single-layer pass)
        # dY is the gradient of the stack output; False when the caller already applied the output's ReLU
        # mask (a region whose gradient comes back from a tail that masks its input, dist.py)
        self.mask_output_grad = mask_output_grad
        # a layer's weight gradient and its data gradient both read only dY: the weight gradient runs on a
        # side stream (its own workspace) concurrently with the data gradient, joined before the next layer
        self.concurrent_wgrad = concurrent_wgrad
        # prep_dgrad_weights: the data gradients' flipped weights (splitcnn_conv_dgrad_weights) built once per
        # step on a side stream during the forward pass instead of inside every conv_bwd_data call.  Off by
        # default: the flips share the SMs with the forward convs and cost more there than the ~5 us each
        # costs on the backward's path (same-box A/B, C2 0.995 -> 1.03 ms, C5 28.5 -> 28.8 ms:
        # profiles/r2i/ab_prep_resnet_conc.txt)
        self.prep_dgrad_weights = prep_dgrad_weights and not force_simt
        self.prep_stream, self._prep_pending, self._prep_valid = None, False, False
        # "layer": every layer over all patches, layer after layer; "patch": patch-major (depth-first,
        # chained patches never communicate, so any schedule is valid): `group_rows` patch rows
        # run through the whole split region before the next group, forward and backward
        if schedule not in ("layer", "patch") or (schedule == "patch" and static_pool):
            raise ValueError("schedule: 'layer', or 'patch' without static_pool")
        self.schedule, self.group_rows = schedule, group_rows
        self.timers = None       # list -> every library call is bracketed by CUDA events (bench.py)
        self.wgrad_hook = None   # callable(key, m) after each layer's weight-gradient call is enqueued
        self._label = ""
        self.region = self._make_region_plan(0)
        self.patch_range = patch_range or (0, self.region.npatch)
        L = self.region.levels[-1]
        self.tail = SplitPlan(tail, N, L["C"], L["H"], L["W"], [0, _out_len(tail, L["H"], 0)],
                              [0, _out_len(tail, L["W"], 1)]) if tail else None
        self._alloc(grad_buffer)

    # ------------------------------------------------------------------ planning
    def _region_output_hw(self):
        h, w = self.H, self.W
        for l in self.region_layers:
            h = (h + l["ph_b"] + l["ph_e"] - l["kh"]) // l["sh"] + 1
            w = (w + l["pw_b"] + l["pw_e"] - l["kw"]) // l["sw"] + 1
        return h, w

    def boundaries(self, step: int):
        ho, wo = self._region_output_hw()
        nh, nw = self.split
        if self.mode == "random":                      # a new scheme per minibatch
            return sc.splitcnn_boundaries_random(ho, nh, wo, nw, self.omega, self.seed, step)
        return sc.splitcnn_boundaries_even(ho, nh), sc.splitcnn_boundaries_even(wo, nw)

    def _make_region_plan(self, step: int) -> SplitPlan:
        Oh, Ow = self.boundaries(step)
        return SplitPlan(self.region_layers, self.N, self.C, self.H, self.W, Oh, Ow)

    def replan(self, step: int):
        """Stochastic splitting: redraw the boundaries; buffer sizes do not depend on them."""
        if self.mode == "random":
            self.region = self._make_region_plan(step)

    # ------------------------------------------------------------------ buffers
    def _stages(self):
        st = [(self.region, m, l) for m, l in enumerate(self.region_layers)]
        if self.tail:
            st += [(self.tail, m, l) for m, l in enumerate(self.tail_layers)]
        return st

    def grad_numel(self) -> int:
        """fp32 elements of all weight + bias gradients (for a caller-provided flat buffer)."""
        n = 0
        for layers, plan in ((self.region_layers, self.region), (self.tail_layers, self.tail)):
            for m, l in enumerate(layers):
                if l["op"] == "conv":
                    n += l["cout"] * l["kh"] * l["kw"] * plan.levels[m]["Cpad"] + l["cout"]
        return n

    def _fusable(self, key: str, plan, layers, m: int) -> bool:
        """conv m (+ReLU) and the 2x2/s2 max-pool m+1 run as ONE fused call (conv_pool_fwd)."""
        return (self.fuse_pool and m + 1 < len(layers) and layers[m]["op"] == "conv" and layers[m].get("relu", True)
                and layers[m + 1]["op"] == "maxpool"
                and sc.splitcnn_conv_pool_supported(plan.handle, m, self.dtype))

    def _alloc(self, grad_buffer=None):
        dev, td = self.device, self.tdtype
        # the conv output of a fused conv -> pool pair is never materialised (the pool's argmax
        # carries everything the backward pass needs): its level gets no buffer
        self.fused = set()
        for key, plan, layers in (("r", self.region, self.region_layers), ("t", self.tail, self.tail_layers)):
            if plan is None:
                continue
            for m in range(len(layers)):
                if self._fusable(key, plan, layers, m):
                    self.fused.add((key, m))
        skip_r = {m + 1 for k, m in self.fused if k == "r"}
        skip_t = {m + 1 for k, m in self.fused if k == "t"}
        self.ws_bytes = self._ws_size()
        self.side = None          # created on first use (a meta-device executor only plans)
        if self.static_pool:
            self._alloc_static()      # activations, argmax bytes and gradients: views of one planned arena
        else:
            self.act_r = [torch.zeros(0 if m in skip_r else self.region.level_elems(m), dtype=td, device=dev)
                          for m in range(self.region.nlayers + 1)]
            self.act_t = ([torch.zeros(0 if m in skip_t else self.tail.level_elems(m), dtype=td, device=dev)
                           for m in range(self.tail.nlayers + 1)] if self.tail else [])
            self.argmax = {}
            for plan, key in ((self.region, "r"), (self.tail, "t")):
                if plan is None:
                    continue
                for m, l in enumerate(plan.layers):
                    if l["op"] == "maxpool":
                        self.argmax[(key, m)] = torch.zeros(plan.level_elems(m + 1), dtype=torch.uint8, device=dev)
            region_levels = range(self.region.nlayers + 1)
            if self.schedule == "patch":
                # patch-major: the region's gradient levels live one patch group at a time in two compact
                # ping-pong buffers; the full-size ones are needed only by the tail and the join
                self.groups = self._patch_groups()
                gmax = max(self._group_span(m, q0, q1)[1] for m in region_levels for q0, q1 in self.groups)
                self.ggrad = [torch.zeros(gmax, dtype=td, device=dev), torch.zeros(gmax, dtype=td, device=dev)]
                region_levels = [self.region.nlayers]
            maxg = max([self.region.level_elems(m) for m in region_levels] +
                       ([self.tail.level_elems(m) for m in range(self.tail.nlayers + 1)] if self.tail else []))
            self.gbuf = None
            self.grad = [torch.zeros(maxg, dtype=td, device=dev), torch.zeros(maxg, dtype=td, device=dev)]
            self.ws = torch.zeros(self.ws_bytes // 4, dtype=torch.float32, device=dev)
            self.ws_w = torch.zeros_like(self.ws) if self.concurrent_wgrad else self.ws     # the side stream's
        self._alloc_params(grad_buffer)

    def _ws_size(self) -> int:
        """Scratch bytes of the largest conv call (library workspace_size over ops 0..2), 256-aligned."""
        ws = 16
        for plan in (self.region, self.tail):
            if plan is None:
                continue
            for m, l in enumerate(plan.layers):
                if l["op"] == "conv":
                    ws = max(ws, *(plan.workspace_size(m, self.dtype, op) for op in (0, 1, 2)))
        return (ws + 255) // 256 * 256

    def _alloc_params(self, grad_buffer=None):
        """HMMS device PARAMETER pool: every conv's weights [Cout][kh][kw][Cpad] (compute dtype) and
        bias (fp32), and the flat fp32 weight / bias gradient buffer, as views of ONE contiguous
        allocation (parameters are small tensors: one pool avoids fragmenting the general pool)."""
        dev, td = self.device, self.tdtype
        es = 2 if self.dtype == sc.BF16 else 4
        al = lambda b: (b + 255) // 256 * 256
        shapes = []
        for key, layers, plan in (("r", self.region_layers, self.region), ("t", self.tail_layers, self.tail)):
            for m, l in enumerate(layers):
                if l["op"] == "conv":
                    wp = (sc.splitcnn_conv_dgrad_weights_size(plan.handle, m, self.dtype)
                          if self.prep_dgrad_weights and self._has_dgrad(key, m) else 0)
                    shapes.append(((key, m), (l["cout"], l["kh"], l["kw"], plan.levels[m]["Cpad"]), l["cout"], wp))
        nbytes = sum(al(4 * co) + al(es * sh[0] * sh[1] * sh[2] * sh[3]) + al(wp) for _, sh, co, wp in shapes)
        gbytes = 0 if grad_buffer is not None else al(4 * self.grad_numel())
        self.param_pool = torch.zeros(nbytes + gbytes, dtype=torch.uint8, device=dev)
        self.params, self.wprep, off = {}, {}, 0
        for key, sh, co, wp in shapes:
            nw = es * sh[0] * sh[1] * sh[2] * sh[3]
            W = self.param_pool[off:off + nw].view(td).view(sh)
            off += al(nw)
            b = self.param_pool[off:off + 4 * co].view(torch.float32)
            off += al(4 * co)
            self.params[key] = (W, b)
            if wp:        # the layer's dgrad-ready weights (parameter pool: they live as long as the weights)
                self.wprep[key] = self.param_pool[off:off + wp]
                off += al(wp)
        if grad_buffer is None:
            grad_buffer = self.param_pool[off:off + 4 * self.grad_numel()].view(torch.float32)
        self.bind_grads(grad_buffer)

    # ------------------------------------------------------------------ HMMS static memory plan
    def _tso_schedule(self):
        """Serialized op list of one step (forward ops in topological order, then the backward
        ops in reverse) as the TSOs each op touches: [(op, [tso names])].  TSOs: ('a', key, m)
        activation level, ('am', key, m) argmax bytes, ('g', key, m) gradient of level m."""
        ops = [("split", [("a", "r", 0)])]
        for key, layers in (("r", self.region_layers), ("t", self.tail_layers)):
            if key == "t":
                if not self.tail:
                    break
                ops.append(("merge", [("a", "r", len(self.region_layers)), ("a", "t", 0)]))
            skip = False
            for m, l in enumerate(layers):
                if skip:
                    skip = False
                    continue
                if (key, m) in self.fused:
                    ops.append((f"{key}{m}+pool", [("a", key, m), ("a", key, m + 2), ("am", key, m + 1)]))
                    skip = True
                elif l["op"] == "conv":
                    ops.append((f"{key}{m}", [("a", key, m), ("a", key, m + 1)]))
                else:
                    ops.append((f"{key}{m}", [("a", key, m), ("a", key, m + 1), ("am", key, m)]))
        out_key = ("a", "t", len(self.tail_layers)) if self.tail else ("a", "r", len(self.region_layers))
        if self._top_masked():
            tk = "t" if self.tail else "r"
            ops.append(("topmask'", [out_key, ("g", tk, len(self.tail_layers if self.tail else self.region_layers))]))
        for key, layers in (("t", self.tail_layers), ("r", self.region_layers)):
            if key == "t" and not self.tail:
                continue
            for m in range(len(layers) - 1, -1, -1):
                top = m == len(layers) - 1 and (key == "t" or not self.tail)
                gin = [] if top and not self._top_masked() else [("g", key, m + 1)]   # else dY is the caller's
                last = key == "r" and m == 0 and not self.input_grad
                gout = [] if last else [("g", key, m)]
                if layers[m]["op"] == "conv":
                    ops.append((f"{key}{m}'", gin + [("a", key, m)] + gout))
                else:
                    ops.append((f"{key}{m}'", gin + [("am", key, m)] + gout))
            if key == "t":
                ops.append(("join'", [("g", "t", 0), ("g", "r", len(self.region_layers))]))
        ops.append(("end", [out_key]))                    # the step's output stays readable
        return ops

    def _tso_bytes(self, name):
        kind, key, m = name
        if kind == "ws":
            return self.ws_bytes
        if kind in ("aF", "aB"):                           # the two halves of an offloaded level
            kind = "a"
        plan = self.region if key == "r" else self.tail
        es = 2 if self.dtype == sc.BF16 else 4
        if kind == "am":
            return plan.level_elems(m + 1)
        if kind == "a" and (key, m - 1) in self.fused:
            return 0                                       # a fused pair's conv output is never stored
        return plan.level_elems(m) * es

    def _tso_lifetimes(self):
        """(schedule, TSO names in first-use order, first use, last use) of one step.  The conv workspaces
        (the main stream's and the concurrent weight gradient's) are TSOs of the same general pool that
        live through the whole step (the device general pool also provides the conv workspace)."""
        sched = self._tso_schedule()
        names, first, last = [], {}, {}
        for w in (("ws", "main", 0), ("ws", "side", 0)) if self.concurrent_wgrad else (("ws", "main", 0),):
            names.append(w)
            first[w], last[w] = 0, len(sched) - 1
        for t, (_, ts) in enumerate(sched):
            for n in ts:
                if n not in first:
                    first[n] = t
                    names.append(n)
                last[n] = t
        return sched, names, first, last

    def _alloc_static(self, lifetimes=None):
        """Place every activation, argmax and gradient TSO of the step in ONE device arena with the
        library's first-fit static planner (splitcnn_memplan): each lives only from the op
        that first touches it to the op that last does, so backward gradients reuse the space of
        activations whose last use has passed.  `lifetimes` (names, first, last) overrides the plain
        schedule scan (the offload executor splits offloaded levels into two TSOs)."""
        names, first, last = lifetimes if lifetimes is not None else self._tso_lifetimes()[1:]
        nbytes = [self._tso_bytes(n) for n in names]
        offs, pool = sc.splitcnn_memplan(nbytes, [first[n] for n in names], [last[n] for n in names], 1024)
        self.arena = torch.empty(max(pool, 1024), dtype=torch.uint8, device=self.device)
        self.pool_bytes = pool
        self.pool_naive_bytes = sum(nbytes)
        td = self.tdtype
        views = {}
        for n, o, b in zip(names, offs, nbytes):
            v = self.arena[o:o + b]
            views[n] = v if n[0] == "am" else v.view(torch.float32) if n[0] == "ws" else v.view(td)
        empty = torch.zeros(0, dtype=td, device=self.device)
        self.static_views = views
        self.ws = views[("ws", "main", 0)]
        self.ws_w = views.get(("ws", "side", 0), self.ws)
        self.act_r = [views.get(("a", "r", m), views.get(("aF", "r", m), empty)) for m in range(self.region.nlayers + 1)]
        self.act_t = ([views.get(("a", "t", m), empty) for m in range(self.tail.nlayers + 1)] if self.tail else [])
        self.argmax = {(n[1], n[2]): v for n, v in views.items() if n[0] == "am"}
        self.gbuf = {(n[1], n[2]): v for n, v in views.items() if n[0] == "g"}
        self.grad = None

    def _gout(self, key, m, g):
        """Buffer for the gradient of level m: its planned TSO, or the ping-pong buffer g is not."""
        if self.gbuf is not None:
            return self.gbuf[(key, m)]
        return self.grad[0] if g is not self.grad[0] else self.grad[1]

    def bind_grads(self, flat: torch.Tensor):
        """All weight / bias gradients become views of one flat fp32 buffer (one allreduce per step)."""
        self.grad_flat = flat
        self.grads = {}
        off = 0
        for key, layers, plan in (("r", self.region_layers, self.region), ("t", self.tail_layers, self.tail)):
            for m, l in enumerate(layers):
                if l["op"] == "conv":
                    cpad = plan.levels[m]["Cpad"]
                    nw = l["cout"] * l["kh"] * l["kw"] * cpad
                    dW = flat[off:off + nw].view(l["cout"], l["kh"], l["kw"], cpad)
                    db = flat[off + nw:off + nw + l["cout"]]
                    off += nw + l["cout"]
                    self.grads[(key, m)] = (dW, db)

    def set_params(self, params):
        """params: list (region + tail order, convs only) of (W_oihw, b) torch/numpy arrays."""
        it = iter(params)
        self._prep_valid = False     # new weights: the next forward rebuilds the dgrad-ready copies
        for key, layers, plan in (("r", self.region_layers, self.region), ("t", self.tail_layers, self.tail)):
            for m, l in enumerate(layers):
                if l["op"] == "conv":
                    W, b = next(it)
                    W = torch.as_tensor(W).to(self.device)
                    self.params[(key, m)][0].copy_(pack_weight(W, plan.levels[m]["Cpad"], self.tdtype))
                    self.params[(key, m)][1].copy_(torch.as_tensor(b, dtype=torch.float32))

    # ------------------------------------------------------------------ instrumentation
    def _call(self, kind: str, work: float, fn, *args):
        """Run one library call; when self.timers is a list, bracket it with CUDA events on the
        launching stream and record (kind, start, end, algorithmic work)."""
        if self.timers is None:
            return fn(*args)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn(*args)
        e1.record()
        self.timers.append((kind, e0, e1, work, self._label))

    def _conv_work(self, plan, m, l):
        """Algorithmic FLOPs of one pass (a re-expressed layer, e.g. the space-to-depth stem, carries the
        MACs per output of the layer it implements in "macs_per_out")."""
        lo = plan.levels[m + 1]
        macs = l.get("macs_per_out", l["cin"] * l["kh"] * l["kw"])
        return 2.0 * lo["N"] * l["cout"] * lo["H"] * lo["W"] * macs

    def _frac(self, plan, m, p0, p1) -> float:
        """Share of layer m's work (its output level's elements) in patches [p0, p1): the accounting of a
        call over a patch range (a rank's rows, a patch-major group)."""
        lv = plan.levels[m + 1]
        n = lv["n_h"] * lv["n_w"]
        if p0 == 0 and p1 >= n:
            return 1.0
        def off(q):
            if q >= n:
                return lv["total_elems"]
            i, j = divmod(q, lv["n_w"])
            return lv["N"] * lv["Cpad"] * (lv["bh"][i] * lv["W"] + (lv["bh"][i + 1] - lv["bh"][i]) * lv["bw"][j])
        return (off(p1) - off(p0)) / lv["total_elems"]

    def _bytes(self, plan, m):
        es = 2 if self.dtype == sc.BF16 else 4
        li, lo = plan.levels[m], plan.levels[m + 1]
        return es * li["N"] * li["C"] * li["H"] * li["W"], es * lo["N"] * lo["C"] * lo["H"] * lo["W"]

    # ------------------------------------------------------------------ masks
    def _masked(self, key: str, m: int) -> bool:
        """Level m is the output of a conv with fused ReLU -> its gradient producer applies the mask."""
        if key == "r":
            if m == 0:
                return self.input_relu
            return self.region_layers[m - 1]["op"] == "conv" and self.region_layers[m - 1].get("relu", True)
        if m > 0:
            return self.tail_layers[m - 1]["op"] == "conv" and self.tail_layers[m - 1].get("relu", True)
        return self._masked("r", len(self.region_layers))

    def _top_masked(self) -> bool:
        """The stack ends in a conv with a fused ReLU: dY (the gradient of the stack OUTPUT) reaches the
        conv's pre-activation only where the output is > 0, one ReLU-backward call."""
        layers = self.tail_layers if self.tail else self.region_layers
        return self.mask_output_grad and bool(layers) and layers[-1]["op"] == "conv" and layers[-1].get("relu", True)

    # ------------------------------------------------------------------ patch-major schedule
    def _patch_groups(self):
        """Contiguous groups of `group_rows` patch rows inside the patch range: [(p0, p1)]."""
        lv = self.region.levels[0]
        nw = lv["n_w"]
        p0, p1 = self.patch_range
        r0, r1 = p0 // nw, (p1 - 1) // nw + 1
        return [(max(p0, r * nw), min(p1, min(r + self.group_rows, r1) * nw)) for r in range(r0, r1, self.group_rows)]

    def _group_span(self, m, q0, q1):
        """(element offset, element count) of patches [q0, q1) in region level m (patches are contiguous)."""
        lv = self.region.levels[m]
        N, Cp, W = lv["N"], lv["Cpad"], lv["W"]
        def off(q):
            if q >= lv["n_h"] * lv["n_w"]:
                return lv["total_elems"]
            i, j = divmod(q, lv["n_w"])
            return N * Cp * (lv["bh"][i] * W + (lv["bh"][i + 1] - lv["bh"][i]) * lv["bw"][j])
        return off(q0), off(q1) - off(q0)

    def _run_bwd_patch_major(self, g, stream, need_input_grad):
        """Region backward one patch group at a time (its whole layer chain), the group's gradient levels in
        two compact buffers addressed as if they were full levels (base = buffer - offset of the group's
        first patch: the library reaches a patch at base + its level offset).  Weight gradients accumulate
        over the groups (beta = 1 after the first); the allreduce hook fires on the last group."""
        es = 2 if self.dtype == sc.BF16 else 4
        out = None
        for k, (q0, q1) in enumerate(self.groups):
            state = {"cur": None}

            def outbuf(m, gin, q0=q0, state=state):
                i = 1 if state["cur"] == 0 else 0
                state["cur"] = i
                return self.ggrad[i].data_ptr() - self._group_span(m, q0, q0 + 1)[0] * es
            out = self._run_bwd("r", self.region, self.region_layers, self.act_r, g, q0, q1, stream, need_input_grad,
                                beta=0.0 if k == 0 else 1.0, hook=k == len(self.groups) - 1, outbuf=outbuf)
        return out

    # ------------------------------------------------------------------ passes
    def input_rows(self):
        """Input rows [h0, h1) the patch range reads (all rows for the whole grid)."""
        lv = self.region.levels[0]
        p0, p1 = self.patch_range
        return lv["bh"][p0 // lv["n_w"]], lv["bh"][(p1 - 1) // lv["n_w"] + 1]

    def forward(self, x: torch.Tensor, stream=None, x_layout: int = sc.NCHW):
        """x: full tensor (dtype) on the device, NCHW or NHWC -- or only the input_rows() window of it
        (NCHW [N][C][h1-h0][W]: a rank's own rows under patch-row sharding).  Returns the output level."""
        p0, p1 = self.patch_range
        R, dt, fl = self.region.handle, self.dtype, self.flags_extra
        self._prep_dgrad(stream)
        b_in = 2 * self._bytes(self.region, 0)[0]
        h0, h1 = self.input_rows()
        if x.dim() == 4 and x_layout == sc.NCHW and x.shape[2] == h1 - h0 and h1 - h0 != self.H:
            self._call("split", b_in * (h1 - h0) // self.H, sc.splitcnn_split_rows, R, 0, dt, x, x_layout, h0, h1,
                       self.act_r[0], p0, p1, stream)
        else:
            self._call("split", b_in, sc.splitcnn_split, R, 0, dt, x, x_layout, self.act_r[0], p0, p1, stream)
        if self.schedule == "patch":       # depth-first: each patch group through the whole region
            for q0, q1 in self.groups:
                self._run_fwd("r", self.region, self.region_layers, self.act_r, q0, q1, stream)
        else:
            self._run_fwd("r", self.region, self.region_layers, self.act_r, p0, p1, stream)
        if self.tail:
            b_j = 2 * self._bytes(self.region, self.region.nlayers - 1)[1]
            self._call("merge", b_j, sc.splitcnn_merge, R, self.region.nlayers, dt, self.act_r[-1], self.act_t[0],
                       sc.NHWC, p0, p1, stream)
            self._run_fwd("t", self.tail, self.tail_layers, self.act_t, 0, 1, stream)
            return self.act_t[-1]
        return self.act_r[-1]

    def _has_dgrad(self, key, m) -> bool:
        """Whether the backward runs conv (key, m)'s data gradient (not the region's first layer unless the
        input gradient is asked for)."""
        return not (key == "r" and m == 0 and not self.input_grad)

    def _prep_dgrad(self, stream):
        """Fork a side stream off the forward and build every layer's dgrad-ready weights there; the backward
        waits for it before its first data gradient (a captured step records the fork as a parallel branch)."""
        if not self.wprep:
            return
        main = stream if stream is not None else torch.cuda.current_stream(self.device)
        if self.prep_stream is None:
            self.prep_stream = torch.cuda.Stream(self.device)
            self.prep_fork, self.prep_join = torch.cuda.Event(), torch.cuda.Event()
        self.prep_fork.record(main)
        self.prep_stream.wait_event(self.prep_fork)
        with torch.cuda.stream(self.prep_stream):
            for (key, m), wt in self.wprep.items():
                plan = self.region if key == "r" else self.tail
                W = self.params[(key, m)][0]
                self._label = (self.region_layers if key == "r" else self.tail_layers)[m].get("name", f"{key}{m}")
                self._call("dgrad_weights", 2 * W.numel() * W.element_size(), sc.splitcnn_conv_dgrad_weights,
                           plan.handle, m, self.dtype, W, wt, wt.numel(), self.prep_stream)
        self.prep_join.record(self.prep_stream)
        self._prep_pending = self._prep_valid = True

    def _dgrad_w(self, key, m, W, flags, main):
        """(weights, flags) for conv (key, m)'s data gradient: the prepared copy (+ FLAG_DGRAD_WEIGHTS, after
        waiting once per backward for the forward's preparation branch) where there is one."""
        if (key, m) not in self.wprep or not self._prep_valid:
            return W, flags
        if self._prep_pending:
            main.wait_event(self.prep_join)
            self._prep_pending = False
        return self.wprep[(key, m)], flags | sc.FLAG_DGRAD_WEIGHTS

    # hooks (no-ops here; the offload executor overrides them)
    def hook_before_fwd(self, key, m):
        pass

    def hook_after_fwd(self, key, m):
        pass

    def hook_before_bwd(self, key, m):
        pass

    def hook_after_bwd(self, key, m):
        pass

    def _run_fwd(self, key, plan, layers, acts, p0, p1, stream):
        skip = False
        for m, l in enumerate(layers):
            if skip:          # the pool half of a fused pair
                skip = False
                continue
            self._label = l.get("name", f"{key}{m}")
            self.hook_before_fwd(key, m)
            if (key, m) in self.fused:
                W, b = self.params[(key, m)]
                self._call("conv_fwd", self._conv_work(plan, m, l) * self._frac(plan, m, p0, p1), sc.splitcnn_conv_pool_fwd, plan.handle, m,
                           self.dtype, acts[m], W, b, acts[m + 2], self.argmax[(key, m + 1)],
                           sc.FLAG_RELU | sc.FLAG_POOL_RELU_MASK | self.flags_extra, p0, p1, stream)
                self.hook_after_fwd(key, m)
                skip = True
                continue
            if l["op"] == "conv":
                W, b = self.params[(key, m)]
                flags = (sc.FLAG_RELU if l.get("relu", True) else 0) | self.flags_extra
                self._call("conv_fwd", self._conv_work(plan, m, l) * self._frac(plan, m, p0, p1), sc.splitcnn_conv_fwd_ws, plan.handle, m, self.dtype,
                           acts[m], W, b, acts[m + 1], flags, self.ws, self.ws_bytes, p0, p1, stream)
            else:
                flags = sc.FLAG_POOL_RELU_MASK if self._masked(key, m) else 0
                bi, bo = self._bytes(plan, m)
                work = (bi + bo + bo // (2 if self.dtype == sc.BF16 else 4)) * self._frac(plan, m, p0, p1)
                self._call("pool_fwd", work, sc.splitcnn_pool_fwd, plan.handle, m, self.dtype, acts[m], acts[m + 1],
                           self.argmax[(key, m)], flags, p0, p1, stream)
            self.hook_after_fwd(key, m)

    def backward(self, dy: torch.Tensor, stream=None, need_input_grad: bool = False):
        """dy: gradient w.r.t. the output level buffer (same layout).  Fills self.grads."""
        p0, p1 = self.patch_range
        g = dy
        if self._top_masked():
            key, plan, acts, q0, q1 = (("t", self.tail, self.act_t, 0, 1) if self.tail else
                                       ("r", self.region, self.act_r, p0, p1))
            gm = self._gout(key, plan.nlayers, g)
            es = 2 if self.dtype == sc.BF16 else 4
            self._call("relu_bwd", 3 * es * dy.numel(), sc.splitcnn_add, plan.handle, plan.nlayers, self.dtype, dy, None,
                       gm, acts[-1], 0, q0, q1, stream)
            g = gm
        if self.tail:
            g = self._run_bwd("t", self.tail, self.tail_layers, self.act_t, g, 0, 1, stream, True)
            gi = self._gout("r", self.region.nlayers, g)
            b_j = 2 * self._bytes(self.region, self.region.nlayers - 1)[1]
            self._call("split", b_j, sc.splitcnn_split, self.region.handle, self.region.nlayers, self.dtype, g,
                       sc.NHWC, gi, p0, p1, stream)
            g = gi
        if self.schedule == "patch":
            return self._run_bwd_patch_major(g, stream, need_input_grad)
        return self._run_bwd("r", self.region, self.region_layers, self.act_r, g, p0, p1, stream, need_input_grad)

    def _run_bwd(self, key, plan, layers, acts, g, p0, p1, stream, need_input_grad, beta=0.0, hook=True, outbuf=None):
        for m in range(len(layers) - 1, -1, -1):
            l = layers[m]
            self._label = l.get("name", f"{key}{m}")
            self.hook_before_bwd(key, m)
            last = (m == 0 and not need_input_grad) and key == "r"
            if last and (self.gbuf is not None or outbuf is not None):
                out = None
            else:
                out = outbuf(m, g) if outbuf is not None else self._gout(key, m, g)
            if l["op"] == "conv":
                W, _ = self.params[(key, m)]
                dW, db = self.grads[(key, m)]
                work = self._conv_work(plan, m, l) * self._frac(plan, m, p0, p1)
                fork = self.concurrent_wgrad and not last
                main = stream if stream is not None else torch.cuda.current_stream(self.device)
                if fork and self.side is None:
                    self.side = torch.cuda.Stream(self.device)
                    self.fork_ev = [torch.cuda.Event() for _ in range(64)]
                    self.join_ev = [torch.cuda.Event() for _ in range(64)]
                if fork:      # the weight gradient on the side stream, after dY (= g) is ready
                    ev = self.fork_ev[m % 64]
                    ev.record(main)
                    self.side.wait_event(ev)
                    with torch.cuda.stream(self.side):
                        self._call("conv_wgrad", work, sc.splitcnn_conv_bwd_filter, plan.handle, m, self.dtype, acts[m],
                                   g, dW, db, beta, self.ws_w, self.ws_bytes, self.flags_extra, p0, p1, self.side)
                        if self.wgrad_hook is not None and hook:
                            self.wgrad_hook(key, m)
                        self.join_ev[m % 64].record(self.side)
                if not last:
                    relu_src = acts[m] if self._masked(key, m) else None
                    wt, fl = self._dgrad_w(key, m, W, self.flags_extra, main)
                    self._call("conv_dgrad", work, sc.splitcnn_conv_bwd_data, plan.handle, m, self.dtype, g, wt, out,
                               relu_src, self.ws, self.ws_bytes, fl, p0, p1, stream)
                if fork:      # join: the next layer may overwrite g's buffer
                    main.wait_event(self.join_ev[m % 64])
                else:
                    self._call("conv_wgrad", work, sc.splitcnn_conv_bwd_filter, plan.handle, m, self.dtype, acts[m], g,
                               dW, db, beta, self.ws, self.ws_bytes, self.flags_extra, p0, p1, stream)
                    if self.wgrad_hook is not None and hook:      # e.g. dist.GradBuckets: start this layer's allreduce
                        self.wgrad_hook(key, m)
            else:
                flags = sc.FLAG_POOL_RELU_MASK if self._masked(key, m) else 0
                bi, bo = self._bytes(plan, m)
                work = (bi + bo + bo // (2 if self.dtype == sc.BF16 else 4)) * self._frac(plan, m, p0, p1)
                self._call("pool_bwd", work, sc.splitcnn_pool_bwd, plan.handle, m, self.dtype, g,
                           self.argmax[(key, m)], out, flags, p0, p1, stream)
            if not last:
                g = out
            self.hook_after_bwd(key, m)
        return g

    def step(self, x, dy, stream=None):
        self.replan(self.step_index)
        self.forward(x, stream)
        self.backward(dy, stream, need_input_grad=self.input_grad)
        self.step_index += 1

    # ------------------------------------------------------------------ accounting
    def conv_flops(self) -> int:
        """Algorithmic FLOPs of one fwd+bwd step: 2*N*Cout*Ho*Wo*Cin*kh*kw per pass;
        fwd + wgrad for every conv, + dgrad for every conv except the first."""
        total = 0
        first = True
        for plan, layers in ((self.region, self.region_layers), (self.tail, self.tail_layers)):
            if plan is None:
                continue
            for m, l in enumerate(layers):
                if l["op"] != "conv":
                    continue
                lo = plan.levels[m + 1]
                f = 2 * lo["N"] * l["cout"] * lo["H"] * lo["W"] * l.get("macs_per_out", l["cin"] * l["kh"] * l["kw"])
                total += f * (2 if first and not self.input_grad else 3)
                first = False
        return total

    def output_numel(self) -> int:
        return (self.act_t[-1] if self.tail else self.act_r[-1]).numel()


def _out_len(layers, L, dim):
    for l in layers:
        k, s = (l["kh"], l["sh"]) if dim == 0 else (l["kw"], l["sw"])
        pb, pe = (l["ph_b"], l["ph_e"]) if dim == 0 else (l["pw_b"], l["pw_e"])
        L = (L + pb + pe - k) // s + 1
    return L
