"""Patch-parallel Split-CNN across the GPUs of one node.

Patches of a chained split region never communicate, so the region is sharded by contiguous
PATCH ROWS: rank r owns patch range [p0, p1) and runs every region layer on it for the whole batch
(weights replicated), reading only its own input rows (splitcnn_split_rows).  The unsplit tail runs
BATCH-parallel, so at the join the region output is re-sharded (patch-sharded -> batch-sharded) and
its gradient is sent back in backward.  The only reduction is the weight/bias-gradient sum (the wgrad
allreduce of SURVEY 8(a) a10 / P:409-415), BUCKETED per layer and started as soon as a bucket's
weight gradients are enqueued, so it runs on NCCL's stream while the rest of the backward computes:
the step costs max(T_backward, 2|G|/alpha B) rather than their sum (the paper's pipelined model,
P:413-415).

Join exchange without packing copies: in a patch buffer `[N][Hp][Wp][C]` the images of one batch
shard are a CONTIGUOUS slice, and on the receiving side the same slice is a whole patch buffer of a
plan built for the shard's batch size.  So every message is a plain view: (patch q, shard k) goes
from the owner of q to rank k.  Messages between a pair of ranks are posted in ascending q on both
sides, which fixes their matching order.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import splitcnn as sc
from .net import SplitNet, _out_len
from .plan import SplitPlan


# ------------------------------------------------------------------ pure index logic (CPU-testable)
def patch_row_ranges(n_h: int, n_w: int, world: int):
    """Contiguous blocks of patch rows per rank -> [(p0, p1)] in row-major patch index."""
    if world > n_h:
        raise ValueError(f"{world} ranks but only {n_h} patch rows to shard")
    out = []
    for r in range(world):
        r0, r1 = (r * n_h) // world, ((r + 1) * n_h) // world
        out.append((r0 * n_w, r1 * n_w))
    return out


def batch_ranges(N: int, world: int):
    if N % world:
        raise ValueError("global batch must divide across ranks")
    b = N // world
    return [(k * b, (k + 1) * b) for k in range(world)]


def patch_geometry(level: dict):
    """[(offset, elems_per_image)] of every patch buffer of a level (full batch)."""
    N, Cp, W = level["N"], level["Cpad"], level["W"]
    bh, bw = level["bh"], level["bw"]
    out = []
    for i in range(level["n_h"]):
        hp = bh[i + 1] - bh[i]
        for j in range(level["n_w"]):
            wp = bw[j + 1] - bw[j]
            out.append((N * Cp * (bh[i] * W + hp * bw[j]), hp * wp * Cp))
    return out


def join_messages(level_full: dict, level_shard: dict, owners, rank: int, world: int, nb: int):
    """Messages of the forward join exchange seen from `rank`:
    sends: (dst, patch, full-buffer offset, count); recvs: (src, patch, shard-buffer offset, count).
    The backward exchange is the same list with the roles swapped."""
    gf, gs = patch_geometry(level_full), patch_geometry(level_shard)
    sends, recvs = [], []
    for q, (off_f, per_img) in enumerate(gf):
        owner = next(r for r, (a, b) in enumerate(owners) if a <= q < b)
        cnt = nb * per_img
        if owner == rank:
            for k in range(world):
                sends.append((k, q, off_f + k * cnt, cnt))
        recvs.append((owner, q, gs[q][0], cnt))
    return sends, recvs


def _host_staged(t: torch.Tensor, group=None) -> bool:
    """gloo cannot read or write device memory: CUDA tensors are then staged through the host (the
    multi-process test runs several ranks on one GPU over gloo, since NCCL refuses that)."""
    return t.is_cuda and dist.get_backend(group) == "gloo"


def all_reduce_sum(t: torch.Tensor, group=None, async_op: bool = False):
    """In-place sum over ranks (NCCL on device memory; gloo through a host copy)."""
    if _host_staged(t, group):
        h = t.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
        t.copy_(h)
        return None
    return dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group, async_op=async_op)


def exchange(src_flat: torch.Tensor, dst_flat: torch.Tensor, sends, recvs, rank: int):
    """Post all sends / receives as tensor views (no packing); self-messages are local copies."""
    if _host_staged(src_flat):
        hs, hd = src_flat.cpu(), torch.empty(dst_flat.shape, dtype=dst_flat.dtype)
        exchange(hs, hd, sends, recvs, rank)
        for src, q, off, cnt in recvs:
            dst_flat[off:off + cnt].copy_(hd[off:off + cnt])
        return
    ops = []
    local = {}
    for dst, q, off, cnt in sends:
        if dst == rank:
            local[q] = src_flat[off:off + cnt]
        else:
            ops.append(dist.P2POp(dist.isend, src_flat[off:off + cnt], dst))
    for src, q, off, cnt in recvs:
        if src == rank:
            dst_flat[off:off + cnt].copy_(local[q])
        else:
            ops.append(dist.P2POp(dist.irecv, dst_flat[off:off + cnt], src))
    if ops:
        for w in dist.batch_isend_irecv(ops):
            w.wait()


def reverse(sends, recvs):
    """Backward join exchange: every forward message travels back."""
    rsends = [(src, q, off, cnt) for src, q, off, cnt in recvs]
    rrecvs = [(dst, q, off, cnt) for dst, q, off, cnt in sends]
    return rsends, rrecvs


# ------------------------------------------------------------------ bucketed, overlapped wgrad allreduce
class GradBuckets:
    """The flat fp32 gradient buffer cut into buckets of consecutive layers in BACKWARD completion order
    (layers are laid out in forward order, so a bucket is one contiguous slice).  mark_ready(key) is
    called right after a layer's weight-gradient call is enqueued; when every layer of a bucket is
    ready, the bucket's all_reduce(SUM) is issued asynchronously (NCCL orders it after the enqueued
    work of the current stream and runs it on its own stream, overlapping the remaining backward).
    wait() makes the current stream wait for every issued bucket; the summed gradient is then in place.

    segments: [(key, offset, numel)] in the order the backward finishes them."""

    def __init__(self, flat: torch.Tensor, segments, bucket_bytes: int = 8 << 20, group=None):
        self.flat, self.group = flat, group
        self.buckets = []          # [lo, hi, keys]
        self.of = {}
        cur = None
        for key, off, n in segments:
            if cur is not None and off + n == cur[0] and (cur[1] - cur[0]) * flat.element_size() < bucket_bytes:
                cur[0] = off
                cur[2].append(key)
            else:
                cur = [off, off + n, [key]]
                self.buckets.append(cur)
            self.of[key] = len(self.buckets) - 1
        self.pending = [len(b[2]) for b in self.buckets]
        self.works = []

    def rebind(self, flat: torch.Tensor):
        self.flat = flat

    def mark_ready(self, key):
        b = self.of[key]
        self.pending[b] -= 1
        if self.pending[b] == 0:
            lo, hi, _ = self.buckets[b]
            w = all_reduce_sum(self.flat[lo:hi], group=self.group, async_op=True)
            if w is not None:
                self.works.append(w)

    def wait(self):
        assert all(p == 0 for p in self.pending), "a bucket was never completed"
        for w in self.works:
            w.wait()
        self.works = []
        self.pending = [len(b[2]) for b in self.buckets]


def grad_segments(net, prefix: str, base: int = 0):
    """[(key, offset, numel)] of a SplitNet's (dW, db) slices in the flat buffer, in backward order."""
    segs = []
    off = base
    for key, layers, plan in (("r", net.region_layers, net.region), ("t", net.tail_layers, net.tail)):
        for m, l in enumerate(layers):
            if l["op"] == "conv":
                n = l["cout"] * l["kh"] * l["kw"] * plan.levels[m]["Cpad"] + l["cout"]
                segs.append(((prefix + key, m), off, n))
                off += n
    return segs[::-1]


# ------------------------------------------------------------------ the distributed executor
class DistSplitNet:
    def __init__(self, c: dict, world: int, rank: int, dtype: int = sc.BF16, device="cuda",
                 bucket_bytes: int = 8 << 20):
        self.world, self.rank, self.dtype = world, rank, dtype
        self.device = torch.device(device)
        N, H, W = c["N"], c["H"], c["W"]
        self.N = N
        nb = N // world
        self.nb = nb
        # region: full batch, patch range of this rank
        probe = SplitNet(c["layers"], [], 1, 3, H, W, split=c["split"], mode=c["mode"], omega=c.get("omega", 0.2),
                         seed=c["seed"], dtype=dtype, device=device)
        lv = probe.region.levels[0]
        self.owners = patch_row_ranges(lv["n_h"], lv["n_w"], world)
        del probe
        self.region_net = SplitNet(c["layers"], [], N, 3, H, W, split=c["split"], mode=c["mode"],
                                   omega=c.get("omega", 0.2), seed=c["seed"], dtype=dtype, device=device,
                                   patch_range=self.owners[rank], mask_output_grad=False)
        L = self.region_net.region.levels[-1]
        self.C_join, self.H_join, self.W_join = L["C"], L["H"], L["W"]
        tail = c["tail"]
        last = c["layers"][-1]
        self.tail_net = SplitNet(tail, [], nb, L["C"], L["H"], L["W"], split=(1, 1), dtype=dtype, device=device,
                                 input_relu=last["op"] == "conv" and last.get("relu", True))
        self.tdtype = self.region_net.tdtype
        self.bucket_bytes = bucket_bytes
        n_rg, n_tl = self.region_net.grad_numel(), self.tail_net.grad_numel()
        self.bind_grads(torch.zeros(n_rg + n_tl, dtype=torch.float32, device=device))
        self._set_join_plan(0)
        self.step_index = 0

    @property
    def timers(self):
        return self.region_net.timers

    @timers.setter
    def timers(self, v):
        self.region_net.timers = v
        self.tail_net.timers = v

    def bind_grads(self, flat: torch.Tensor):
        """All region + tail weight / bias gradients as views of one flat fp32 buffer, cut into allreduce
        buckets (tail layers finish first in backward, then the region's)."""
        n_rg = self.region_net.grad_numel()
        self.grad_flat = flat
        self.region_net.bind_grads(flat[:n_rg])
        self.tail_net.bind_grads(flat[n_rg:])
        if getattr(self, "buckets", None) is None:
            segs = grad_segments(self.tail_net, "t", n_rg) + grad_segments(self.region_net, "r", 0)
            self.buckets = GradBuckets(flat, segs, self.bucket_bytes)
            self.tail_net.wgrad_hook = lambda key, m: self.buckets.mark_ready(("t" + key, m))
            self.region_net.wgrad_hook = lambda key, m: self.buckets.mark_ready(("r" + key, m))
        self.buckets.rebind(flat)

    def input_rows(self):
        """Rows [h0, h1) of the input this rank reads (its patch rows at level 0)."""
        return self.region_net.input_rows()

    def grad_slice(self):
        """[lo, hi) of the flat gradient this rank reads back to the host (1/world of it; every rank
        holds the whole sum after the allreduce, so the host gets all of it once across ranks)."""
        n = self.grad_flat.numel()
        return (n * self.rank) // self.world, (n * (self.rank + 1)) // self.world

    def _set_join_plan(self, step: int):
        rn = self.region_net
        Oh, Ow = rn.boundaries(step)
        self.join_shard = SplitPlan(rn.region_layers, self.nb, 3, rn.H, rn.W, Oh, Ow)
        self.staging = getattr(self, "staging", None)
        n = self.join_shard.level_elems(self.join_shard.nlayers)
        if self.staging is None or self.staging.numel() != n:
            self.staging = torch.zeros(n, dtype=self.tdtype, device=rn.device)
        lf = rn.region.levels[-1]
        ls = self.join_shard.levels[-1]
        self.msgs = join_messages(lf, ls, self.owners, self.rank, self.world, self.nb)

    @property
    def grads(self):
        g = dict(self.region_net.grads)
        g.update({("t", k[1]): v for k, v in self.tail_net.grads.items()})
        return g

    def set_params(self, params):
        nr = sum(1 for l in self.region_net.region_layers if l["op"] == "conv")
        self.region_net.set_params(params[:nr])
        self.tail_net.set_params(params[nr:])

    def output_numel(self) -> int:
        return self.tail_net.output_numel()

    def step(self, x, dy, stream=None):
        """x: the full input or only this rank's input_rows() window ([N][C][h1-h0][W]); dy: the gradient
        of this rank's batch shard of the tail output."""
        rn, tn = self.region_net, self.tail_net
        if rn.mode == "random":
            rn.replan(self.step_index)
            self._set_join_plan(self.step_index)
        # region forward on this rank's patches (full batch)
        rn.forward(x, stream)
        # join: patch-sharded -> batch-sharded, merge into the tail's NHWC input
        sends, recvs = self.msgs
        exchange(rn.act_r[-1], self.staging, sends, recvs, self.rank)
        Lj = self.join_shard.nlayers
        sc.splitcnn_merge(self.join_shard.handle, Lj, self.dtype, self.staging, tn.act_r[0], sc.NHWC, 0, -1, stream)
        tn._run_fwd("r", tn.region, tn.region_layers, tn.act_r, 0, 1, stream)
        # tail backward (batch shard) down to the join gradient
        g = tn.backward(dy, stream, need_input_grad=True)
        sc.splitcnn_split(self.join_shard.handle, Lj, self.dtype, g, sc.NHWC, self.staging, 0, -1, stream)
        rs, rr = reverse(sends, recvs)
        g_region = rn.grad[0]
        exchange(self.staging, g_region, rs, rr, self.rank)
        rn.backward(g_region, stream)
        # the wgrad allreduce (sum over ranks of the per-rank partial sums): the buckets were issued as
        # their layers' weight gradients were enqueued; the step ends when the last one has landed
        self.buckets.wait()
        self.step_index += 1


class DistResNet:
    """Patch-row sharded ResNet-18 split stack (C3).  Rank r runs every region layer on
    its own patch rows (ResSplitNet / ResBNSplitNet with patch_range; the 1x1 downsamples share the
    block's patch grid); the output stays patch-sharded (each rank merges only its rows and reads only
    their rows of dY).  With BN, every BN's per-channel [2][C] sums are all-reduced before use -- the
    statistics in forward, (dbeta, dgamma) in backward -- so BN is the unsplit whole-tensor BN (R11)
    under sharding: 2C floats per BN per pass, the only exchange inside the region besides the
    weight-gradient sum, which is one allreduce of the conv gradients after the backward (the BN
    parameter gradients are already global)."""

    def __init__(self, c: dict, world: int, rank: int, dtype: int = sc.BF16, bn: bool = False, device="cuda",
                 group=None, stem_pad: int = 16):
        from .resnet import ResBNSplitNet, ResSplitNet
        self.world, self.rank, self.dtype, self.group = world, rank, dtype, group
        nh, nw = c["split"]
        self.owners = patch_row_ranges(nh, nw, world)
        kw = dict(split=c["split"], dtype=dtype, device=device, patch_range=self.owners[rank], stem_pad=stem_pad)
        if bn:
            kw["bn_reduce"] = lambda t: all_reduce_sum(t, group=group)
        cls = ResBNSplitNet if bn else ResSplitNet
        self.net = cls(c["layers"], c["blocks"], c["N"], 3, c["H"], c["W"], **kw)
        self.n_conv = ResSplitNet.grad_numel(self.net)          # conv (dW, db) part of the flat buffer
        self.tdtype, self.device = self.net.tdtype, self.net.device
        self.input_grad = False

    @property
    def timers(self):
        return self.net.timers

    @timers.setter
    def timers(self, v):
        self.net.timers = v

    @property
    def grad_flat(self):
        return self.net.grad_flat

    @property
    def grads(self):
        return self.net.grads

    def bind_grads(self, flat):
        self.net.bind_grads(flat)

    def grad_slice(self):
        n = self.grad_flat.numel()
        return (n * self.rank) // self.world, (n * (self.rank + 1)) // self.world

    def set_params(self, params):
        self.net.set_params(params)

    def set_bn_params(self, bn_params):
        self.net.set_bn_params(bn_params)

    def output_numel(self) -> int:
        return self.net.output_numel()

    def step(self, x, dy, stream=None):
        self.net.forward(x, stream)
        self.net.backward(dy, stream)
        all_reduce_sum(self.net.grad_flat[:self.n_conv], group=self.group)
