"""Per-layer device time of the 16-bit tcgen05 kernel (A/B helper: WINO_LIB_PATH selects the build).
L2 flushed before every launch; CUDA events; median of 20."""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import sys

import torch

import paper_conf_ppopp_yanwc20_b200 as wino
from synth_inputs import CONFIGS, make_inputs

dt = torch.float16 if (len(sys.argv) < 2 or sys.argv[1] == "fp16") else torch.bfloat16
mode = sys.argv[2] if len(sys.argv) > 2 else "none"  # stream-K workspace mode: none / auto / on / off
P = int(sys.argv[3]) if len(sys.argv) > 3 else 1     # batch shard of a P-rank job
flush = torch.empty(512 << 18, dtype=torch.float32, device="cuda")
res = {}
for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x"):
    cfg = CONFIGS[name].with_batch(CONFIGS[name].N // P)
    x, w = make_inputs(cfg)
    xh, wh = x.to(dt).cuda(), w.to(dt).cuda()
    uh = wino.filter_transform_half(wh)
    ws = None if mode == "none" else torch.empty(wino.half_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K),
                                                 dtype=torch.uint8, device="cuda")
    kw = {} if mode == "none" else {"ws": ws, "stream_k": mode}
    y = wino.conv2d_half(xh, uh, **kw)
    ts = []
    for _ in range(23):
        flush.fill_(1.0)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        wino.conv2d_half(xh, uh, out=y, **kw)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    t = sorted(ts[3:])[len(ts[3:]) // 2]
    res[name] = {"us": round(t * 1e3, 1), "eff_tflops": round(cfg.eff_flops / (t * 1e-3) / 1e12, 1)}
print(json.dumps(res))
