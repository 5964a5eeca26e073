"""Per-CTA timeline of one multi-layer FP32 launch (build -DWINO_WS_CTATRACE into
build_ab/libwino_ctatrace.so): entry and exit time, unit range -> work balance across layers.
Usage: ml_trace.py [P]"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["WINO_LIB_PATH"] = os.path.abspath(os.environ.get("TRACE_LIB", "build_ab/libwino_ctatrace.so"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_yanwc20_b200 as wino  # noqa: E402
from paper_conf_ppopp_yanwc20_b200.dist import shard_range  # noqa: E402
from synth_inputs import CONFIGS, make_inputs  # noqa: E402

P = int(sys.argv[1]) if len(sys.argv) > 1 else 8
layers, cfgs = [], []
for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x"):
    cfg = CONFIGS[name]
    lo, hi = shard_range(cfg.N, 0, P)
    cfg = cfg.with_batch(hi - lo)
    x, w = make_inputs(cfg)
    layers.append((x[..., :].contiguous().cuda(), wino.filter_transform(w.cuda()),
                   torch.empty((cfg.K, cfg.H, cfg.W, cfg.N), device="cuda")))
    cfgs.append(cfg)
ws = torch.zeros(wino.conv_multi_workspace_bytes([(c.N, c.C, c.H, c.W, c.K) for c in cfgs]), dtype=torch.uint8,
                 device="cuda")
flush = torch.empty(1 << 27, device="cuda")
for rep in range(3):
    flush.fill_(rep)
    torch.cuda.synchronize()
    wino.conv2d_multi(layers, ws)
    torch.cuda.synchronize()
L = wino.lib()
L.wino_debug_cta_trace.argtypes = [ctypes.c_void_p, ctypes.c_int]
buf = (ctypes.c_ulonglong * (256 * 4))()
L.wino_debug_cta_trace(ctypes.cast(buf, ctypes.c_void_p), 256 * 4)
a = np.array(list(buf), dtype=np.int64).reshape(256, 4)
a = a[a[:, 0] > 0]
t0 = a[:, 0].min()
dur = (a[:, 3] - t0) / 1000.0
units = a[:, 2] - a[:, 1]
bounds = np.cumsum([0] + [((c.N * ((c.H + 1) // 2) * ((c.W + 1) // 2) + 31) // 32) * ((c.K + 63) // 64) *
                          ((c.C + 7) // 8) for c in cfgs])
layer = np.searchsorted(bounds, a[:, 1], side="right") - 1
print(f"P={P} CTAs {len(a)} exit median {np.median(dur):.1f} max {dur.max():.1f} us")
for l, c in enumerate(cfgs):
    m = layer == l
    if m.any():
        print(f"  start in {c.name:8s} N={c.N:3d}: CTAs {m.sum():3d} units/CTA {units[m].mean():6.1f} "
              f"exit median {np.median(dur[m]):6.1f} max {dur[m].max():6.1f} us -> us/unit {np.median(dur[m] / units[m]):.3f}")

# per-piece timeline of CTAs 0, 40, 80, 120: main-loop time per channel block and epilogue time per tile
L.wino_debug_ml_piece_trace.argtypes = [ctypes.c_void_p, ctypes.c_int]
pb = (ctypes.c_ulonglong * (4 * 96 * 4))()
L.wino_debug_ml_piece_trace(ctypes.cast(pb, ctypes.c_void_p), 4 * 96 * 4)
pt = np.array(list(pb), dtype=np.int64).reshape(4, 96, 4)
for ci in range(4):
    rows = [r for r in pt[ci] if r[0] > 0]
    if not rows:
        continue
    rows = np.array(rows)
    loop = (rows[:, 1] - rows[:, 0]) / 1000.0
    epi = (rows[:, 2] - rows[:, 1]) / 1000.0
    gap = (rows[1:, 0] - rows[:-1, 2]) / 1000.0
    nst = rows[:, 3]
    whole = nst == nst.max()
    print(f"  CTA {40 * ci:3d}: pieces {len(rows)}, main loop {np.median(loop[whole] / nst[whole]):.3f} us/block "
          f"(nst {int(nst.max())}), epilogue median {np.median(epi):.2f} us, gap to next piece {np.median(gap) if len(gap) else 0:.2f} us")
