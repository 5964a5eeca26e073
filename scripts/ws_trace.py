"""Run the split-C FP32 kernel once with a trace build (-DWINO_WS_TRACE) and print
CTA 0's per-tile clock64 events: main loop start / end, ydone wait end, partials
published (compute warps); yready wait start / end, reduction done (reducer warp)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["WINO_LIB_PATH"] = os.path.abspath(os.environ.get("TRACE_LIB", "build_ab/libwino_wstrace.so"))
import torch
import paper_conf_ppopp_yanwc20_b200 as wino
from paper_conf_ppopp_yanwc20_b200.dist import shard_range
from synth_inputs import CONFIGS, make_inputs
name = sys.argv[1] if len(sys.argv) > 1 else "conv2_x"
P = int(sys.argv[2]) if len(sys.argv) > 2 else 1
split = int(sys.argv[3]) if len(sys.argv) > 3 else 2
cfg = CONFIGS[name]
x, w = make_inputs(cfg)
lo, hi = shard_range(cfg.N, 0, P)
x = x[..., lo:hi].contiguous().cuda()
u = wino.filter_transform(w.cuda())
for _ in range(3):
    y = wino.conv2d(x, u, split_c=split)
torch.cuda.synchronize()
L = wino.lib()
buf = (ctypes.c_ulonglong * (8 * 64))()
L.wino_debug_ws_trace.argtypes = [ctypes.c_void_p, ctypes.c_int]
L.wino_debug_ws_trace(ctypes.cast(buf, ctypes.c_void_p), 8 * 64)
ev = [[buf[e * 64 + t] for t in range(64)] for e in range(8)]
t0 = ev[0][0]
names = ["loop0", "loop1", "yfree_ok", "published", "-", "yready_ok", "reduced"]
print(name, "P", P, "split", split, "cluster slots", [L.wino_debug_cluster_slots(s) for s in (1, 2, 4, 8)])
print("  T " + " ".join(f"{n:>10s}" for n in names))
for t in range(64):
    if not ev[0][t]:
        break
    print(f"{t:3d} " + " ".join(f"{(ev[e][t] - t0) if ev[e][t] else -1:10d}" for e in range(7)))
