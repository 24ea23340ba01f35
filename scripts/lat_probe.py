"""Device latency of small split convs (50 calls captured in a CUDA graph, CUDA events around one replay):
the fixed cost of one conv_tc launch vs the C2 tail layers' shapes."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_jinh19_b200 import splitcnn as sc
from paper_conf_asplos_jinh19_b200.plan import SplitPlan

def run(C, H, split, N, label):
    l = synth.conv(C, C, name="c")
    O = sc.splitcnn_boundaries_even(H, split)
    pl = SplitPlan([l], N, C, H, H, O, O)
    lv0, lv1 = pl.levels
    x = torch.randn(lv0["total_elems"], device="cuda").to(torch.bfloat16)
    y = torch.empty(lv1["total_elems"], device="cuda", dtype=torch.bfloat16)
    w = (torch.randn(C, 3, 3, lv0["Cpad"], device="cuda") * 0.05).to(torch.bfloat16)
    b = torch.zeros(C, device="cuda")
    ws_b = max(pl.workspace_size(0, sc.BF16, 1), pl.workspace_size(0, sc.BF16, 2))
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    fl = 2.0 * N * C * H * H * C * 9
    def t(fn, n=50):   # device time per call: n calls captured in one CUDA graph (no host issue cost)
        for _ in range(3): fn()
        torch.cuda.synchronize()
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            gr = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gr, stream=s):
                for _ in range(n): fn()
        gr.replay(); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); gr.replay(); e1.record(); torch.cuda.synchronize()
        return e0.elapsed_time(e1) / n * 1000
    f = t(lambda: sc.splitcnn_conv_fwd(pl.handle, 0, sc.BF16, x, w, b, y, sc.FLAG_RELU))
    d = t(lambda: sc.splitcnn_conv_bwd_data(pl.handle, 0, sc.BF16, y, w, x, x, ws, ws_b))
    g = t(lambda: sc.splitcnn_conv_bwd_filter(pl.handle, 0, sc.BF16, x, y, torch.empty((C, 3, 3, lv0["Cpad"]), device="cuda"), None, 0.0, ws, ws_b))
    print(f"{label:28s} C={C} H={H} split={split} N={N}: fwd {f:6.1f} us ({fl / f / 1e6:6.0f} TF/s)  dgrad {d:6.1f} us  wgrad {g:6.1f} us")

run(64, 8, 1, 1, "floor: 1 tile")
run(512, 8, 1, 1, "floor: 1 tile, K=4608")
run(64, 32, 2, 128, "C2 conv1_2")
run(128, 16, 2, 128, "C2 conv2_2")
run(256, 8, 2, 128, "C2 conv3_2")
run(512, 4, 1, 128, "C2 conv4_2")
run(512, 2, 1, 128, "C2 conv5_2")
