"""bench.py -- VGG-19 Split-CNN fwd+bwd images/s on B200 (BASELINE.json metric).

One STEP = one pass of the whole hot path over one synthetic batch: split ->
per-patch conv(+bias+ReLU) / max-pool forward through the split region -> merge at the join ->
unsplit tail -> backward (pool bwd, conv dgrad with fused ReLU mask, conv wgrad summed over
patches and batch) [-> wgrad allreduce across ranks when N > 1].

Default workload: C5 (VGG-19 224x224, global batch 256, 8x8 split at depth 50%).  Inputs are
resident in HBM and far larger than L2 (126 MB), so no explicit L2 flush is needed.

    python bench.py [--gpus N --steps K --warmup W --config C5|C2|C4 --impl ours|reference]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "VGG-19 split-CNN fwd+bwd images/sec"
UNIT = "images/s"


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index, self.rows, self.proc = index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        self.proc.wait()
        self.th.join(timeout=2)
        sm = [float(r[0]) for r in self.rows if r and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) > 1 and r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in self.rows for k in range(4) if len(r) > 2 + k and r[2 + k] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(sm)}


# --------------------------------------------------------------------------- workloads
def workload(name: str, N: int | None = None):
    import synth
    c = synth.vgg_config(name, N=N)
    return c


def make_inputs(c, dtype_t, device, world=1, rank=0):
    """Seeded synthetic inputs: X ~ U[-1,1), W ~ Kaiming, b ~ U[-.1,.1), dY ~ N(0,1)."""
    import torch
    import synth
    g = synth.rng(c["seed"])
    if c.get("resnet"):
        params = synth.resnet_params(g, c["layers"], c["blocks"])
        if c.get("full"):
            params += synth.resnet_params(g, *synth.resnet18_tail_blocks())
    else:
        params = [p for p in synth.layer_params(g, c["layers"] + c["tail"]) if p is not None]
    gen = torch.Generator(device="cpu").manual_seed(c["seed"])
    N = c["N"]
    x = (torch.rand((N, c.get("C", 3), c["H"], c["W"]), generator=gen) * 2 - 1).to(dtype_t)
    return params, x, gen


# --------------------------------------------------------------------------- ours
def _nets(net):
    """The SplitNet executors inside an executor (the dist executor holds a region and a tail net)."""
    return [n for n in (getattr(net, "region_net", None), getattr(net, "tail_net", None), getattr(net, "net_r", None),
                        getattr(net, "net_t", None), getattr(net, "net", None)) if n is not None] or [net]


def run_ours(args):
    import torch
    import torch.distributed as dist
    from paper_conf_asplos_jinh19_b200 import splitcnn as sc
    from paper_conf_asplos_jinh19_b200.net import SplitNet

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.gpus != world:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}: launch N ranks (bench.py self-launches "
                         f"them when WORLD_SIZE is unset)")
    if torch.cuda.device_count() < world or local >= torch.cuda.device_count():
        raise SystemExit(f"{world} ranks but only {torch.cuda.device_count()} visible GPUs")
    torch.cuda.set_device(local)
    if world > 1 or args.force_dist:
        if "RANK" not in os.environ:            # --force-dist at one rank without a launcher
            import socket
            so = socket.socket()
            so.bind(("127.0.0.1", 0))
            os.environ.update(RANK="0", WORLD_SIZE="1", MASTER_ADDR="127.0.0.1", MASTER_PORT=str(so.getsockname()[1]))
            so.close()
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    c = workload(args.config)
    if getattr(args, "full", False) and c.get("resnet"):
        c["full"] = True
    if args.dtype is None:
        args.dtype = c.get("dtype", "bf16")
    dtype = {"bf16": sc.BF16, "fp32": sc.FP32, "tf32": sc.TF32}[args.dtype]
    use_offload = args.offload if args.offload is not None else (args.config == "C4")
    if c.get("resnet"):
        from paper_conf_asplos_jinh19_b200.resnet import ResBNSplitNet, ResSplitNet
        if world > 1 or args.force_dist:
            if args.full:
                raise SystemExit("C3 --full (unsplit tail) runs on one GPU; the split stack shards (DistResNet)")
            from paper_conf_asplos_jinh19_b200.dist import DistResNet
            net = DistResNet(c, world, rank, dtype, bn=args.bn, stem_pad=args.stem_pad)
        elif args.full:          # the whole trunk: split region -> unsplit layer3/4 -> global average pool (f2)
            import synth
            from paper_conf_asplos_jinh19_b200.resnet import ResNet18Net
            tc, tb = synth.resnet18_tail_blocks()
            net = ResNet18Net(c["layers"], c["blocks"], tc, tb, c["N"], 3, c["H"], c["W"], split=c["split"],
                              bn=args.bn, dtype=dtype)
        else:
            cls = ResBNSplitNet if args.bn else ResSplitNet
            net = cls(c["layers"], c["blocks"], c["N"], 3, c["H"], c["W"], split=c["split"], dtype=dtype,
                      stem_pad=args.stem_pad)
        use_offload = False
    elif world > 1 or args.force_dist:
        from paper_conf_asplos_jinh19_b200.dist import DistSplitNet
        net = DistSplitNet(c, world, rank, dtype)
        use_offload = False
    elif use_offload:
        from paper_conf_asplos_jinh19_b200.offload import OffloadSplitNet
        net = OffloadSplitNet(c["layers"], c["tail"], c["N"], 3, c["H"], c["W"], split=c["split"], mode=c["mode"],
                              omega=c.get("omega", 0.2), seed=c["seed"], dtype=dtype, static_pool=args.static_pool)
    else:
        net = SplitNet(c["layers"], c["tail"], c["N"], c.get("C", 3), c["H"], c["W"], split=c["split"], mode=c["mode"],
                       omega=c.get("omega", 0.2), seed=c["seed"], dtype=dtype,
                       static_pool=args.static_pool and args.schedule == "layer", input_grad=args.config == "C1",
                       schedule=args.schedule, group_rows=args.group_rows, prep_dgrad_weights=args.prep_dgrad)
    net.input_grad = args.config == "C1"      # C1 = one layer's fwd + dgrad + wgrad
    if args.serial_wgrad:                     # weight gradients on the main stream (A/B of the overlap)
        for n in _nets(net):
            n.concurrent_wgrad = False
    params, x_host, gen = make_inputs(c, net.tdtype, "cuda")
    net.set_params([(torch.from_numpy(W), torch.from_numpy(b)) for W, b in params])
    if getattr(net, "set_bn_params", None) is not None:
        import synth
        net.set_bn_params(synth.bn_params(synth.rng(c["seed"] + 100), [W.shape[0] for W, _ in params]))
    out_numel = net.output_numel()
    if c.get("resnet"):      # the ResNet region output stays patch-sharded: every rank reads the whole dY
        dy_host = torch.randn(out_numel, generator=gen).to(net.tdtype)
    else:                    # the VGG tail is batch-sharded: this rank's batch shard of dY
        dy_all = torch.randn(out_numel * world, generator=gen).to(net.tdtype)
        dy_host = dy_all[rank * out_numel:(rank + 1) * out_numel]
    if world > 1 and hasattr(net, "input_rows"):   # a rank reads only its own patch rows' input (as its loader would)
        h0, h1 = net.input_rows()
        x_host = x_host[:, :, h0:h1].contiguous()
    x = x_host.cuda()
    dy = dy_host.cuda()
    stream = torch.cuda.current_stream()

    def step():
        net.step(x, dy)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        step()
    barrier()
    offload_info = None
    if use_offload:
        # without offload first (same net, offload disabled): the degradation reference
        net.offload_enabled = False
        torch.cuda.reset_peak_memory_stats()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        barrier()
        e0.record(stream)
        for _ in range(args.steps):
            step()
        e1.record(stream)
        barrier()
        ms_plain = e0.elapsed_time(e1) / args.steps
        peak_plain = torch.cuda.max_memory_allocated()
        stats = net.profile_and_plan(x, dy, reps=20)
        net.offload_enabled = True
        for _ in range(2):
            step()
        barrier()
        torch.cuda.reset_peak_memory_stats()
        offload_info = {"plan": "Algorithm 1 + reverse pass (splitcnn_offload_plan / _prefetch_plan)",
                        "host_link_gbs": round(stats["bw_bytes_per_s"] / 1e9, 1),
                        "offloaded_levels": stats["offloaded_levels"],
                        "offloaded_gb": round(stats["offloaded_bytes"] / 1e9, 3),
                        "candidate_gb": round(stats["candidate_bytes"] / 1e9, 3),
                        "cap_gb": round(stats["cap_bytes"] / 1e9, 3),
                        "no_offload_ms_per_step": round(ms_plain, 3),
                        "no_offload_peak_gb": round(peak_plain / 1e9, 2)}
    # default: one CUDA graph per step wherever the plan is static (even split; C4 draws new boundaries
    # every step) on one process: C1/C2 are launch-bound, C3 gains 5 % (2.97 vs 3.12 ms), C5 is neutral
    # device-side and gains on the e2e path (profiles/r2_ab_graph.txt)
    use_graph = args.graph if args.graph is not None else (
        args.config in ("C1", "C2", "C3", "C5") and world == 1 and not args.force_dist)
    graph = None
    if use_graph:
        # capture one whole step (every library call enqueues on the current stream, the db side stream
        # joins back) and replay it
        side = torch.cuda.Stream()
        side.wait_stream(stream)
        with torch.cuda.stream(side):
            step()
        stream.wait_stream(side)
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        l0 = sc.splitcnn_kernel_launches()
        with torch.cuda.graph(graph):
            step()
        launches_per_step = sc.splitcnn_kernel_launches() - l0
        torch.cuda.synchronize()
        for _ in range(3):
            graph.replay()
        step = graph.replay                   # noqa: F811 (the timed step is the graph replay)
    launches0 = sc.splitcnn_kernel_launches()
    clocks = ClockSampler(local)
    clocks.start()
    net.timers = None             # the timed steps carry no per-call events (breakdown: separate pass below)
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    flush_l2 = c["H"] < 224          # small working sets: flush L2 between timed steps, time each step
    if flush_l2:
        l2buf = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")     # 256 MB > 126 MB L2
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    barrier()
    t0.record(stream)
    for i in range(args.steps):
        if flush_l2:
            l2buf.zero_()
            evs[i][0].record(stream)
        step()
        if flush_l2:
            evs[i][1].record(stream)
    t1.record(stream)
    barrier()
    clk = clocks.stop()
    launches = (launches_per_step * args.steps) if graph else sc.splitcnn_kernel_launches() - launches0
    ms = sum(a.elapsed_time(b) for a, b in evs) if flush_l2 else t0.elapsed_time(t1)
    # per-kind breakdown (roofline) from an eager pass with CUDA events around every library call; the
    # weight gradients run on the main stream here, so every kernel is timed alone (not while it shares the
    # GPU with its layer's concurrent data gradient)
    conc = [(n, n.concurrent_wgrad) for n in _nets(net)]
    for n, _ in conc:
        n.concurrent_wgrad = False
    # the device must not wait on the host between calls, or a small kernel's interval would include the
    # host's launch latency: each step is queued behind a spin kernel that lasts ~2x the host's issue time
    # of one step (measured), so its events record back-to-back device execution
    torch.cuda.synchronize()
    h0 = time.perf_counter()
    net.step(x, dy)
    host_s = time.perf_counter() - h0
    torch.cuda.synchronize()
    spin_cycles = int(min(0.05, 2.0 * host_s) * 2.0e9)
    net.timers = []
    for _ in range(args.steps):
        if flush_l2:
            l2buf.zero_()
        torch.cuda._sleep(spin_cycles)
        net.step(x, dy)
    barrier()
    for n, v in conc:
        n.concurrent_wgrad = v
    if world > 1:
        tt = torch.tensor([ms], device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = tt.item()
    # per-kind device time from the events recorded around every library call
    kinds, per_layer = {}, {}
    for kind, e0, e1, work, label in net.timers:
        dt_ms = e0.elapsed_time(e1)
        k = kinds.setdefault(kind, [0.0, 0.0, 0])
        k[0] += dt_ms
        k[1] += work
        k[2] += 1
        pl = per_layer.setdefault(f"{label}:{kind}", [0.0, 0.0])
        pl[0] += dt_ms
        pl[1] += work
    net.timers = None
    ms_step = ms / args.steps
    global_batch = c["N"]
    if offload_info is not None:
        offload_info["offload_peak_gb"] = round(torch.cuda.max_memory_allocated() / 1e9, 2)
        offload_info["degradation_pct"] = round(100 * (ms_step / offload_info["no_offload_ms_per_step"] - 1), 2)
    value = global_batch / (ms_step / 1e3)

    # e2e: the same step through the public API with host buffers: every step copies its inputs (x, dY)
    # from pinned host memory and reads back its result (all weight / bias gradients) -- through
    # HostPipeline, which overlaps step i+1's H2D and step i's D2H with compute (double buffers, events)
    from paper_conf_asplos_jinh19_b200.pipeline import HostPipeline
    xh = x_host.pin_memory()
    dyh = dy.cpu().pin_memory()
    g_lo, g_hi = net.grad_slice() if hasattr(net, "grad_slice") else (0, net.grad_flat.numel())
    gh = torch.empty(g_hi - g_lo, dtype=net.grad_flat.dtype, pin_memory=True)
    h2d = xh.numel() * xh.element_size() + dyh.numel() * dyh.element_size()
    d2h = gh.numel() * gh.element_size()
    ke = max(1, min(args.steps, 10))
    pipe = HostPipeline(net, x, dy.numel(), graphs=graph is not None)
    for _ in range(3):
        pipe.submit(xh, dyh, gh)
    pipe.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    e0.record(stream)
    for _ in range(ke):
        pipe.submit(xh, dyh, gh)
    pipe.d2h.synchronize()
    stream.wait_stream(pipe.d2h)
    e1.record(stream)
    barrier()
    ms_e2e = e0.elapsed_time(e1) / ke
    if world > 1:
        tt = torch.tensor([ms_e2e], device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms_e2e = tt.item()

    peaks, src = _peaks()
    conv_ms = sum(kinds[k][0] for k in kinds if k.startswith("conv"))
    conv_flop = sum(kinds[k][1] for k in kinds if k.startswith("conv"))
    conv_launch_count = sum(kinds[k][2] for k in kinds if k.startswith("conv"))
    achieved = conv_flop / (conv_ms / 1e3) / 1e12 if conv_ms > 0 else 0.0
    peak = peaks.get("bf16_tflops_sustained", peaks["bf16_tflops"])
    peak_note = f"{src} bf16_tflops_sustained"
    if args.dtype == "tf32":      # the measured bf16 peak x the nominal dense tf32 / bf16 ratio (1.1 / 2.25)
        peak, peak_note = peak * 1.1 / 2.25, peak_note + " x 1.1/2.25 (nominal tf32/bf16)"
    elif args.dtype == "fp32":    # 3xTF32 (and 6 bf16 split products for wgrad): a third of the tf32 peak
        peak, peak_note = peak * 1.1 / 2.25 / 3, peak_note + " x 1.1/2.25 / 3 (3xTF32)"
    hbm_ms = sum(kinds[k][0] for k in kinds if not k.startswith("conv"))
    hbm_bytes = sum(kinds[k][1] for k in kinds if not k.startswith("conv"))
    traffic = None
    tp = os.path.join(ROOT, "profiles", f"traffic_{args.config}.json")
    if os.path.exists(tp):
        traffic = json.load(open(tp)).get("conv_bytes_per_launch")
    line = {
        "metric": METRIC, "value": round(value, 2), "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_step, 4), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None,          # the global batch is fixed as N grows
        "dtype": args.dtype, "data": "synthetic (seeded PCG64 / torch.Generator; random-init weights)",
        "config": {"workload": f"{args.config}: {c['desc']}" + (" + unsplit layer3/4 + GAP (full trunk)" if c.get("full") else "")
                               + (" + whole-tensor BN" if args.bn else ""),
                   "global_batch": global_batch,
                   "image": [c["H"], c["W"]], "split": list(c["split"]), "split_mode": c["mode"],
                   "split_convs": sum(1 for l in c["layers"] if l["op"] == "conv"),
                   "parallelism": f"patch{world}" if world > 1 else "1gpu",
                   "l2": "inputs/activations >> 126 MB L2 (no flush needed)" if c["H"] >= 224 else
                         "L2 flushed (256 MB write) before every timed step; each step timed by its own events",
                   "cuda_graph": bool(graph),
                   "schedule": args.schedule + (f" ({args.group_rows} patch rows per group)" if args.schedule == "patch" else "")},
        "e2e": {"value": round(global_batch / (ms_e2e / 1e3), 2), "unit": UNIT, "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": d2h},
        "gpu_launches": launches,
        "roofline": {"bound": "tensor", "kernel": "split conv (fwd+dgrad+wgrad, all layers)",
                     "achieved": round(achieved, 2), "peak": peak, "unit": "TFLOP/s",
                     "frac": round(achieved / peak, 4), "traffic": traffic,
                     "peak_source": peak_note,
                     "conv_share_of_step": round(conv_ms / max(ms, 1e-9), 4),
                     "conv_launches_timed": conv_launch_count,
                     "timing": "CUDA events around every library call, a separate eager pass with the weight "
                               "gradients serial, each step queued behind a spin kernel (device-bound intervals)"
                               + (", L2 flushed before each step" if flush_l2 else "")},
        "hbm_ops": {"kinds": sorted(k for k in kinds if not k.startswith("conv")),
                    "achieved_gbs": round(hbm_bytes / (hbm_ms / 1e3) / 1e9, 1) if hbm_ms > 0 else None,
                    "peak_gbs": peaks["hbm_gbs"], "share_of_step": round(hbm_ms / max(ms, 1e-9), 4)},
        "per_kind_ms_per_step": {k: round(v[0] / args.steps, 4) for k, v in kinds.items()},
        "clocks": clk,
    }
    if offload_info is not None:
        line["offload"] = offload_info
    line["memory"] = {"peak_allocated_gb": round(torch.cuda.max_memory_allocated() / 1e9, 3),
                      "static_pool": bool(getattr(net, "static_pool", False))}
    if getattr(net, "static_pool", False):
        line["memory"]["pool_gb"] = round(net.pool_bytes / 1e9, 3)
        line["memory"]["tso_sum_gb"] = round(net.pool_naive_bytes / 1e9, 3)
    if args.per_layer:
        line["per_layer"] = {k: {"ms": round(v[0] / args.steps, 4),
                                 "tflops" if ":conv" in k else "gbs": round(v[1] / (v[0] / 1e3) / (1e12 if ":conv" in k else 1e9), 1)}
                             for k, v in per_layer.items()}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(args.config, budget_tiles=args.cpu_tiles, full=bool(c.get("full")))
    if rank == 0:
        print(json.dumps(line), flush=True)
    if dist.is_initialized():
        dist.destroy_process_group()


# --------------------------------------------------------------------------- oracle timing
def oracle_sample_time(config: str, tiles: int, full: bool = False):
    """Time the ORACLE (as it stands) on a bounded sample of one step and scale to images/s.

    Sample: 1 image; for every layer-op of the step (conv fwd / dgrad / wgrad, pool fwd / bwd) the
    oracle runs on `tiles` output tiles, each 1/64 of the layer's output plane (region layers: one
    of the plan's patches of a 8x8 even split of that level; tail layers: a 1/8 x 1/8 crop with the
    layer's own padding).  Work is linear in output pixels, so time/image = sum over ops of
    t(sample) * (output pixels of the op) / (sample output pixels)."""
    import numpy as np
    import synth
    from oracle import ops as O
    from oracle import plan as OP

    c = workload(config, N=1)
    g = synth.rng(c["seed"])
    layers = c["layers"] + c["tail"]
    if full and c.get("resnet"):                  # + the unsplit layer3/4 (their downsamples via blocks)
        tc, tb = synth.resnet18_tail_blocks()
        off = len(layers)
        layers = layers + tc
        c = dict(c, blocks=list(c["blocks"]) + [dict(a=b["a"] + off, ds=b["ds"]) for b in tb])
    params = synth.layer_params(g, layers)
    ops, h = [], c["H"]
    for m, (l, prm) in enumerate(zip(layers, params)):
        ops.append((l, prm, h))
        for b in c.get("blocks", ()):      # ResNet: the 1x1 downsample reads the block input
            if b["a"] == m and b["ds"] is not None:
                ops.append((b["ds"], synth.layer_params(g, [b["ds"]])[0], h))
        h = OP.out_len(h, l["kh"], l["sh"], l["ph_b"], l["ph_e"])
    total = 0.0
    sample_px = 0
    first_conv = config != "C1"     # C1 times its dgrad too
    for l, prm, h in ops:
        ho = OP.out_len(h, l["kh"], l["sh"], l["ph_b"], l["ph_e"])
        # a tile = a patch of an 8x8 even split of this layer's output (>= 1 px)
        n = min(8, ho)
        Ob = OP.boundaries_even(ho, n)
        lp = OP.plan([l], 1, l["cin"], h, h, Ob, Ob).layers[0]
        t_layer = 0.0
        px_s = 0
        for t in range(tiles):
            i, j = (t // n) % n, t % n
            hp, wp = lp.Ih[i + 1] - lp.Ih[i], lp.Iw[j + 1] - lp.Iw[j]
            X = g.uniform(-1, 1, (1, l["cin"], hp, wp))
            if l["op"] == "conv":
                W, b = prm
                t0 = time.perf_counter()
                Y = O.conv_fwd_patch(X, W, b, l["sh"], l["sw"], lp.pads_h[i], lp.pads_w[j], True)
                if not first_conv:    # the step computes no input gradient for the first conv
                    O.conv_bwd_data_patch(Y, W, hp, wp, l["sh"], l["sw"], lp.pads_h[i], lp.pads_w[j], X)
                O.conv_bwd_filter_patch(X, Y, l["kh"], l["kw"], l["sh"], l["sw"], lp.pads_h[i], lp.pads_w[j])
                t_layer += time.perf_counter() - t0
            else:
                t0 = time.perf_counter()
                Y, A = O.pool_fwd_patch(X, l["kh"], l["kw"], l["sh"], l["sw"], lp.pads_h[i], lp.pads_w[j])
                O.pool_bwd_patch(Y, A, hp, wp, l["kh"], l["kw"], l["sh"], l["sw"], lp.pads_h[i], lp.pads_w[j])
                t_layer += time.perf_counter() - t0
            px_s += (lp.Oh[i + 1] - lp.Oh[i]) * (lp.Ow[j + 1] - lp.Ow[j])
        total += t_layer * (ho * ho) / px_s
        first_conv = first_conv and l["op"] != "conv"
        sample_px += px_s
    return total, f"1 image, {tiles} of 64 output tiles per layer-op (fwd+dgrad+wgrad / pool fwd+bwd), scaled by output pixels"


def cpu_baseline(config: str, budget_tiles: int = 4, full: bool = False):
    import os as _os
    t_img, sample = oracle_sample_time(config, budget_tiles, full)
    cores = len(_os.sched_getaffinity(0))
    return {"value": round(1.0 / t_img, 5), "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
            "seconds_per_image_est": round(t_img, 2)}


def run_reference(args):
    """--impl reference: the oracle (test infrastructure) timed as it stands on the host cores."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    c = workload(args.config)
    tiles = 4      # 4 of 64 output tiles of every layer-op per step (~2 s of oracle work): a stable estimate
    for _ in range(args.warmup):
        oracle_sample_time(args.config, tiles)
    vals, t0 = [], time.perf_counter()
    for _ in range(args.steps):
        t_img, sample = oracle_sample_time(args.config, tiles)
        vals.append(t_img * c["N"])
    ms_step = 1e3 * statistics.mean(vals)
    value = c["N"] / (ms_step / 1e3)
    cores = len(os.sched_getaffinity(0))
    line = {"impl": "reference", "metric": METRIC, "value": round(value, 6), "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 1), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{args.config}: {c['desc']}", "global_batch": c["N"]},
            "cpu_baseline": {"kind": "oracle", "cores": cores, "sample": sample, "value": round(value, 6)},
            "e2e": {"value": round(value, 6), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "wall_s": round(time.perf_counter() - t0, 1)}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C5", choices=["C1", "C2", "C3", "C4", "C5"])
    ap.add_argument("--dtype", default=None, choices=["bf16", "fp32", "tf32"])
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--cpu-tiles", type=int, default=12)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--per-layer", action="store_true")
    ap.add_argument("--prep-dgrad", action="store_true",
                    help="VGG executor: build the dgrad-ready weights on a side stream during the forward (A/B; measured slower)")
    ap.add_argument("--serial-wgrad", action="store_true",
                    help="weight gradients on the main stream instead of concurrently with the data gradients")
    ap.add_argument("--graph", dest="graph", action="store_true", default=None,
                    help="time CUDA-graph replays of the step (default for C1, C2)")
    ap.add_argument("--no-graph", dest="graph", action="store_false")
    ap.add_argument("--static-pool", dest="static_pool", action="store_true", default=True,
                    help="HMMS static memory plan: all activations / gradients in one first-fit arena (f3; default)")
    ap.add_argument("--no-static-pool", dest="static_pool", action="store_false")
    ap.add_argument("--force-dist", action="store_true",
                    help="run the multi-GPU executor (DistSplitNet, NCCL) even at one rank (exercises the N>1 path)")
    ap.add_argument("--full", action="store_true", help="C3: the whole ResNet-18 trunk (split region + tail + GAP)")
    ap.add_argument("--bn", action="store_true", help="C3 with whole-tensor BN after every conv (R11, f2)")
    ap.add_argument("--schedule", default="layer", choices=["layer", "patch"],
                    help="patch: patch-major (depth-first) region schedule, --group-rows patch rows per group")
    ap.add_argument("--group-rows", type=int, default=1)
    ap.add_argument("--stem-pad", type=int, default=16, choices=[16, 64],
                    help="C3: channels of the space-to-depth stem level (12 real; 16 = narrow-row halo kernels, "
                         "64 = 64-channel halo / 2-CTA kernels on zero channels)")
    ap.add_argument("--offload", dest="offload", action="store_true", default=None)
    ap.add_argument("--no-offload", dest="offload", action="store_false")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "ours" and args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # one process per GPU: re-launch this command under torch.distributed.run (127.0.0.1 rendezvous)
        import socket
        import torch
        if torch.cuda.device_count() < args.gpus:
            raise SystemExit(f"--gpus {args.gpus} but only {torch.cuda.device_count()} visible GPUs")
        s = socket.socket()
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
        s.close()
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
        raise SystemExit(subprocess.call(cmd))
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
