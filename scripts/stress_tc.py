"""Repeat tensor-core runs (regular and stream-K, both tile heights) on small-integer inputs and
count results that differ from Eq. 4 (exact in TF32 / rounded exactly in 16 bit): a stress test
for rare pipeline hazards."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ppopp_yanwc20_b200 as wino, oracle
from synth_inputs import Conv3x3Config, make_inputs
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 20
bad_total = 0
for shape in [(32, 64, 64, 30, 30), (32, 72, 200, 9, 7), (8, 256, 256, 14, 14), (4, 512, 512, 7, 7)]:
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("s", N, C, K, H, W), kind="smallint")
    ref = oracle.direct_conv(x, w)
    xd, wd = x.cuda(), w.cuda()
    ref16 = torch.from_numpy(ref).float().half().double().numpy()
    cases = {}
    u = wino.filter_transform_tc(wd, "tf32")
    wst = torch.empty(wino.tc_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device="cuda")
    cases["tf32"] = (lambda: wino.conv2d_tc(xd, u), ref)
    if K > 64:
        cases["tf32-sk"] = (lambda: wino.conv2d_tc(xd, u, ws=wst, stream_k="on"), ref)
    uh = wino.filter_transform_half(wd.half())
    wsh = torch.empty(wino.half_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device="cuda")
    xh = xd.half()
    cases["fp16"] = (lambda: wino.conv2d_half(xh, uh), ref16)
    cases["fp16-sk"] = (lambda: wino.conv2d_half(xh, uh, ws=wsh, stream_k="on"), ref16)
    for name, (fn, r) in cases.items():
        bad = 0
        for _ in range(reps):
            y = fn().cpu().double().numpy()
            bad += int((y != r).any())
        bad_total += bad
        print(shape, name, "failing runs", bad, "of", reps, flush=True)
print("TOTAL failing runs", bad_total)
