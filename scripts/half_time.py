"""Per-layer device time of the 16-bit tcgen05 kernel (A/B helper: WINO_LIB_PATH selects the build).
L2 flushed before every launch; CUDA events; median of 20."""
import json
import sys

import torch

import paper_conf_ppopp_yanwc20_b200 as wino
from synth_inputs import CONFIGS, make_inputs

dt = torch.float16 if (len(sys.argv) < 2 or sys.argv[1] == "fp16") else torch.bfloat16
flush = torch.empty(512 << 18, dtype=torch.float32, device="cuda")
res = {}
for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x"):
    cfg = CONFIGS[name]
    x, w = make_inputs(cfg)
    xh, wh = x.to(dt).cuda(), w.to(dt).cuda()
    uh = wino.filter_transform_half(wh)
    y = wino.conv2d_half(xh, uh)
    ts = []
    for _ in range(23):
        flush.fill_(1.0)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        wino.conv2d_half(xh, uh, out=y)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    t = sorted(ts[3:])[len(ts[3:]) // 2]
    res[name] = {"us": round(t * 1e3, 1), "eff_tflops": round(cfg.eff_flops / (t * 1e-3) / 1e12, 1)}
print(json.dumps(res))
