"""Multi-process CPU tests (gloo, world_size 2 and 4) of the communication of one patch-parallel step
(dist.py): the join exchange (patch-sharded region output -> batch-sharded tail input, and its
gradient back) as plain tensor views with no packing, and the bucketed wgrad allreduce (GradBuckets:
buckets issued asynchronously as layers finish in backward order) whose result must be the oracle's
O10 sum of the per-rank partial gradients.  Runs on CPU: the plan is host code, the exchange plumbing."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth
from tests.helpers import pack_level


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import __graft_entry__
        __graft_entry__.build()
        from paper_conf_asplos_jinh19_b200 import dist as D
        from paper_conf_asplos_jinh19_b200.plan import SplitPlan
        layers = [synth.conv(3, 8), synth.maxpool(8), synth.conv(8, 16)]
        N, H, W = 4, 32, 24
        Oh, Ow = [0, 3, 8, 12, 16], [0, 5, 12]           # uneven: 4 patch rows x 2 columns at the output
        full = SplitPlan(layers, N, 3, H, W, Oh, Ow)
        shard = SplitPlan(layers, N // world, 3, H, W, Oh, Ow)
        lf, ls = full.levels[-1], shard.levels[-1]
        owners = D.patch_row_ranges(lf["n_h"], lf["n_w"], world)
        sends, recvs = D.join_messages(lf, ls, owners, rank, world, N // world)
        g = synth.rng(7)
        X = synth.uniform(g, (N, 16, lf["H"], lf["W"])).astype(np.float64)
        G = synth.uniform(g, (N, 16, lf["H"], lf["W"])).astype(np.float64)
        src = torch.from_numpy(pack_level(X, lf))
        # poison the patches this rank does not own: they must never be read
        p0, p1 = owners[rank]
        for qq, (off, per) in enumerate(D.patch_geometry(lf)):
            if not (p0 <= qq < p1):
                src[off:off + N * per] = float("nan")
        staging = torch.zeros(ls["total_elems"], dtype=torch.float64)
        D.exchange(src, staging, sends, recvs, rank)
        nb = N // world
        want = pack_level(X[rank * nb:(rank + 1) * nb], ls)
        ok_fwd = bool(np.array_equal(staging.numpy(), want))
        # backward: each rank holds the gradient of its batch shard; owners receive their patches
        gstage = torch.from_numpy(pack_level(G[rank * nb:(rank + 1) * nb], ls))
        greg = torch.full((lf["total_elems"],), float("nan"), dtype=torch.float64)
        rs, rr = D.reverse(sends, recvs)
        D.exchange(gstage, greg, rs, rr, rank)
        ref = pack_level(G, lf)
        ok_bwd = True
        for qq, (off, per) in enumerate(D.patch_geometry(lf)):
            if p0 <= qq < p1:
                ok_bwd &= bool(np.array_equal(greg[off:off + N * per].numpy(), ref[off:off + N * per]))
        # bucketed wgrad allreduce: per-rank partial gradients (dyadic, so any summation order is exact),
        # layers completed in backward order, buckets issued asynchronously as they fill
        from oracle import ops as OO
        sizes = [1728 + 8, 36864 + 64, 73728 + 128, 147456 + 128, 4608 + 512, 9 + 1]   # (dW + db) per layer
        offs = np.cumsum([0] + sizes)
        segs = [((("r", m)), int(offs[m]), sizes[m]) for m in range(len(sizes))][::-1]
        parts = [synth.dyadic(synth.rng(100 + r), (int(offs[-1]),)).astype(np.float64) for r in range(world)]
        flat = torch.from_numpy(parts[rank].copy())
        B = D.GradBuckets(flat, segs, bucket_bytes=300_000)
        cover = sorted((lo, hi) for lo, hi, _ in B.buckets)
        ok_buckets = (cover[0][0] == 0 and cover[-1][1] == offs[-1] and len(B.buckets) < len(sizes)
                      and all(a[1] == b[0] for a, b in zip(cover, cover[1:])))
        for step in range(2):          # twice: the pending counters re-arm after wait()
            flat.copy_(torch.from_numpy(parts[rank]))
            for key, _, _ in segs:
                B.mark_ready(key)
            B.wait()
            ok_buckets &= bool(np.array_equal(flat.numpy(), OO.allreduce_sum(parts)))
        q.put((rank, ok_fwd, ok_bwd, ok_buckets))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_step_communication_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=180)
    res = sorted(q.get(timeout=5) for _ in range(world))
    assert res == [(r, True, True, True) for r in range(world)], res


def test_grad_buckets_layout():
    """Buckets are contiguous slices of consecutive layers in backward order, merged up to the byte cap."""
    from paper_conf_asplos_jinh19_b200 import dist as D
    flat = torch.zeros(100, dtype=torch.float32)
    segs = [(("t", 3), 90, 10), (("t", 1), 60, 30), (("r", 2), 20, 40), (("r", 0), 0, 20)][::1]
    B = D.GradBuckets(flat, segs, bucket_bytes=4 * 35)
    assert [(lo, hi, keys) for lo, hi, keys in B.buckets] == [(60, 100, [("t", 3), ("t", 1)]),
                                                              (20, 60, [("r", 2)]), (0, 20, [("r", 0)])]
    B = D.GradBuckets(flat, segs, bucket_bytes=1 << 20)
    assert len(B.buckets) == 1 and B.buckets[0][:2] == [0, 100]


def test_patch_and_batch_ranges():
    from paper_conf_asplos_jinh19_b200 import dist as D
    assert D.patch_row_ranges(8, 8, 8) == [(8 * r, 8 * r + 8) for r in range(8)]
    assert D.patch_row_ranges(8, 8, 2) == [(0, 32), (32, 64)]
    assert D.patch_row_ranges(3, 2, 2) == [(0, 2), (2, 6)]
    with pytest.raises(ValueError):
        D.patch_row_ranges(2, 2, 4)
    assert D.batch_ranges(256, 8)[3] == (96, 128)
    with pytest.raises(ValueError):
        D.batch_ranges(10, 4)
