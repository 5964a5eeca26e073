"""Small launches of every kernel variant for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_yanwc20_b200 as wino
from synth_inputs import Conv3x3Config, make_inputs

shapes = [Conv3x3Config("a", 32, 16, 64, 6, 6),    # FP32 WS (TMA) + tc MM=64
          Conv3x3Config("b", 5, 9, 70, 7, 5),      # FP32 generic cp.async 4 B
          Conv3x3Config("c", 8, 12, 132, 5, 4),    # FP32 generic cp.async 16 B, tc MM=128 XM=1
          Conv3x3Config("d", 64, 8, 256, 3, 3)]    # tc MM=128 TMA
for cfg in shapes:
    x, w = make_inputs(cfg)
    x, w = x.cuda(), w.cuda()
    y = wino.conv2d(x, wino.filter_transform(w))
    for v in ("tf32", "3xtf32"):
        y = wino.conv2d_tc(x, wino.filter_transform_tc(w, v))
torch.cuda.synchronize()
print("ok")
