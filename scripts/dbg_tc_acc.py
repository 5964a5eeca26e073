"""Debug: repeated tcgen05 runs on small integers (exact in TF32) -- count wrong outputs and show
which output positions q (row/column of the 2x2 tile) and tile positions they fall in.
Usage: WINO_LIB_PATH=... python scripts/dbg_tc_acc.py [reps]"""
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ppopp_yanwc20_b200 as wino  # noqa: E402
from synth_inputs import CONFIGS, Conv3x3Config, make_inputs  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 8
cases = [("3xtf32", CONFIGS["conv2_x"], "auto"), ("3xtf32", CONFIGS["conv2_x"], "off"),
         ("tf32", CONFIGS["conv2_x"], "off"), ("tf32", Conv3x3Config("s", 32, 64, 64, 30, 30), "on")]
for variant, cfg, sk in cases:
    x, w = make_inputs(cfg, kind="smallint")
    ref = oracle.direct_conv(x, w)
    xd = x.cuda()
    u = wino.filter_transform_tc(w.cuda(), variant)
    ws = torch.empty(wino.tc_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8, device="cuda")
    fails = 0
    for r in range(reps):
        try:
            y = wino.conv2d_tc(xd, u, ws=ws, stream_k=sk).cpu().double().numpy()
        except wino.WinoError as e:
            print(variant, cfg.name, sk, "error", e)
            break
        bad = np.argwhere(y != ref)
        if len(bad):
            fails += 1
            qs = np.bincount((bad[:, 1] % 2) * 2 + bad[:, 2] % 2, minlength=4)
            print(f"{variant} {cfg.name} sk={sk} rep {r}: {len(bad)} bad, by q {qs.tolist()}, "
                  f"k range {bad[:, 0].min()}..{bad[:, 0].max()}", flush=True)
    print(f"== {variant} {cfg.name} sk={sk}: {fails} of {reps} runs wrong", flush=True)
