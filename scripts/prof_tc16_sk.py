"""conv5_x fp16 with the regular persistent schedule and with forced stream-K (for an ncu A/B)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_yanwc20_b200 as wino
from synth_inputs import CONFIGS, make_inputs
cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "conv5_x"]
x, w = make_inputs(cfg)
xh, wh = x.half().cuda(), w.half().cuda()
uh = wino.filter_transform_half(wh)
ws = torch.empty(wino.half_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8, device="cuda")
for _ in range(2):
    y = wino.conv2d_half(xh, uh)
    y = wino.conv2d_half(xh, uh, ws=ws, stream_k="on")
torch.cuda.synchronize()
