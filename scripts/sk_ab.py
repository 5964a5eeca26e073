"""A/B of the FP32 plans per layer (and batch shard): planner's choice vs forced stream-K vs no
workspace, each timed as a CUDA graph of 20 launches with L2 flushed before the graph (median of 5).
Usage: sk_ab.py [P]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_yanwc20_b200 as wino  # noqa: E402
from paper_conf_ppopp_yanwc20_b200.dist import shard_range  # noqa: E402
from synth_inputs import CONFIGS, make_inputs  # noqa: E402

P = int(sys.argv[1]) if len(sys.argv) > 1 else 1
flush = torch.empty(1 << 27, device="cuda")
for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x"):
    cfg = CONFIGS[name]
    x, w = make_inputs(cfg)
    lo, hi = shard_range(cfg.N, 0, P)
    x = x[..., lo:hi].contiguous().cuda()
    u = wino.filter_transform(w.cuda())
    ws = torch.zeros(wino.conv_workspace_bytes(hi - lo, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8, device="cuda")
    y = torch.empty((cfg.K, cfg.H, cfg.W, hi - lo), device="cuda")
    res = {}
    for mode in ("auto", "on", "off", "nows"):
        fn = (lambda: wino.conv2d(x, u, out=y)) if mode == "nows" else (lambda: wino.conv2d(x, u, out=y, ws=ws, stream_k=mode))
        for _ in range(3):
            fn()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            fn()
        ts = []
        for _ in range(7):
            flush.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            g.replay()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b) * 1e3)
        res[mode] = sorted(ts)[3]
    p = wino.plan(hi - lo, cfg.C, cfg.H, cfg.W, cfg.K, variant=4)
    print(f"P={P} {name} N={hi - lo} planner sk={p.stream_k} split={p.split_c}: " +
          " ".join(f"{k} {v:7.1f}us" for k, v in res.items()), flush=True)
