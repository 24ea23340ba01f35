"""Probe: does the gloo backend move CUDA tensors (all_reduce, batch_isend_irecv) between two processes
that share one GPU?  (NCCL refuses two ranks on one device.)"""
import os
import socket
import sys

import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def work(rank, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    torch.cuda.set_device(0)
    try:
        t = torch.full((1000,), float(rank + 1), device="cuda")
        w = dist.all_reduce(t, async_op=True)
        w.wait()
        ok1 = bool((t == 3).all())
        a = torch.full((64,), float(rank), device="cuda")
        b = torch.empty(64, device="cuda")
        ops = [dist.P2POp(dist.isend, a, 1 - rank), dist.P2POp(dist.irecv, b, 1 - rank)]
        for r in dist.batch_isend_irecv(ops):
            r.wait()
        ok2 = bool((b == 1 - rank).all())
        q.put((rank, ok1, ok2))
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e)[:300]))
    dist.destroy_process_group()


if __name__ == "__main__":
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=work, args=(r, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(120)
    print([q.get(timeout=5) for _ in range(2)])
    sys.stdout.flush()
