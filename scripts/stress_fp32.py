"""Repeat FP32 runs (persistent, cluster split-C, stream-K; batch shards of every BASELINE layer)
on small-integer inputs and count results that differ from Eq. 4 (exact in FP32): a stress
test for rare pipeline hazards in the headline kernel."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ppopp_yanwc20_b200 as wino, oracle
from synth_inputs import CONFIGS, make_inputs, sample_points
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
total = 0
for P in (1, 2, 4, 8):
    for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x"):
        cfg = CONFIGS[name].with_batch(CONFIGS[name].N // P)
        x, w = make_inputs(cfg, kind="smallint")
        idx = sample_points(cfg.K, cfg.H, cfg.W, cfg.N, 3000)
        ref = oracle.direct_sample(x, w, idx)
        ii = idx.cuda()
        xd, u = x.cuda(), wino.filter_transform(w.cuda())
        ws = torch.zeros(wino.conv_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8, device="cuda")
        modes = {"plain": lambda: wino.conv2d(xd, u), "sk-on": lambda: wino.conv2d(xd, u, ws=ws, stream_k="on"),
                 "split2": lambda: wino.conv2d(xd, u, split_c=2)}
        for m, fn in modes.items():
            bad = 0
            for _ in range(reps):
                y = fn()
                got = y[ii[:, 0], ii[:, 1], ii[:, 2], ii[:, 3]].double().cpu().numpy()
                bad += int(not np.array_equal(got, ref))
            total += bad
            if bad:
                print("FAIL", P, name, m, bad, "of", reps, flush=True)
    print("P", P, "done", flush=True)
print("TOTAL failing runs", total)
