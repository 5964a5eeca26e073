"""A/B of the multi-layer FP32 launch (csrc/fused_fp32_ml.cuh) against per-layer launches:
each layer alone through conv2d (planned) and through conv2d_multi with one job, then all four
layers in one conv2d_multi.  CUDA events, L2 flushed before each rep, median of 20.
Usage: ml_ab.py [P ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_yanwc20_b200 as wino  # noqa: E402
from paper_conf_ppopp_yanwc20_b200.dist import shard_range  # noqa: E402
from synth_inputs import CONFIGS, make_inputs  # noqa: E402

flush = torch.empty(1 << 28, device="cuda")


def timeit(fn, reps=20):
    ts = []
    for i in range(reps + 3):
        flush.fill_(i)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        if i >= 3:
            ts.append(a.elapsed_time(b) * 1000)
    ts.sort()
    return ts[len(ts) // 2]


for P in [int(a) for a in sys.argv[1:]] or [1, 8]:
    layers, cfgs = [], []
    for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x"):
        cfg = CONFIGS[name]
        lo, hi = shard_range(cfg.N, 0, P)
        cfg = cfg.with_batch(hi - lo)
        x, w = make_inputs(cfg)
        layers.append((x.cuda(), wino.filter_transform(w.cuda()), torch.empty((cfg.K, cfg.H, cfg.W, cfg.N), device="cuda")))
        cfgs.append(cfg)
    shapes = [(c.N, c.C, c.H, c.W, c.K) for c in cfgs]
    ws = torch.zeros(max(wino.conv_multi_workspace_bytes(shapes), max(wino.conv_workspace_bytes(*s) for s in shapes)),
                     dtype=torch.uint8, device="cuda")
    tot_s = tot_m = 0.0
    for (x, u, y), c in zip(layers, cfgs):
        ts = timeit(lambda: wino.conv2d(x, u, out=y, ws=ws))
        tk = timeit(lambda: wino.conv2d(x, u, out=y, ws=ws, stream_k="on"))
        tn = timeit(lambda: wino.conv2d(x, u, out=y, ws=ws, stream_k="off"))
        tm = timeit(lambda: wino.conv2d_multi([(x, u, y)], ws))
        tot_s += ts
        tot_m += tm
        print(f"P={P} {c.name} N={c.N}: single {ts:7.1f} us (sk on {tk:7.1f}, off {tn:7.1f})  ml(1 job) {tm:7.1f} us")
    ta = timeit(lambda: wino.conv2d_multi(layers, ws))
    print(f"P={P} sum single {tot_s:.1f}  sum ml(1 job) {tot_m:.1f}  ml(4 jobs) {ta:.1f} us")

    def split(k):  # the first k layers in one multi-layer launch, the rest one launch each
        wino.conv2d_multi(layers[:k], ws)
        for x, u, y in layers[k:]:
            wino.conv2d(x, u, out=y, ws=ws)
    for k in (2, 3):
        print(f"P={P} ml(first {k}) + single rest {timeit(lambda: split(k)):.1f} us")
