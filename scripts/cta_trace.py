"""Per-CTA timeline of one FP32 WS launch (build -DWINO_WS_CTATRACE into build_ab/libwino_ctatrace.so):
%globaltimer at kernel entry, first stage landed, last main loop done, exit -- to see where the fixed
per-launch cost of small batch shards goes.  Usage: cta_trace.py [layer] [P] [stream_k on|off|auto]"""
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

name = sys.argv[1] if len(sys.argv) > 1 else "conv5_x"
P = int(sys.argv[2]) if len(sys.argv) > 2 else 8
sk = sys.argv[3] if len(sys.argv) > 3 else "auto"
cfg = CONFIGS[name]
x, w = make_inputs(cfg)
lo, hi = shard_range(cfg.N, 0, P)
x = x[..., lo:hi].contiguous().cuda()
u = wino.filter_transform(w.cuda())
ws = torch.zeros(wino.conv_workspace_bytes(hi - lo, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8, device="cuda")
flush = torch.empty(1 << 27, device="cuda")
L = wino.lib()
L.wino_debug_cta_trace.argtypes = [ctypes.c_void_p, ctypes.c_int]
for rep in range(4):
    flush.fill_(rep)  # cold L2 as in the bench
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record()
    y = wino.conv2d(x, u, ws=ws, stream_k=sk)
    ev1.record()
    torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * (256 * 4))()
L.wino_debug_cta_trace(ctypes.cast(buf, ctypes.c_void_p), 256 * 4)
a = np.array(list(buf), dtype=np.int64).reshape(256, 4)
a = a[a[:, 0] > 0]
t0 = a[:, 0].min()
r = (a - t0) / 1000.0  # us
p = wino.plan(hi - lo, cfg.C, cfg.H, cfg.W, cfg.K, variant=4)
print(f"{name} P={P} N={hi - lo} plan={p} event time {ev0.elapsed_time(ev1) * 1e3:.1f} us, CTAs {len(a)}")
for i, n in enumerate(["entry", "first stage", "last loop done", "exit"]):
    print(f"  {n:15s} min {r[:, i].min():7.2f}  median {np.median(r[:, i]):7.2f}  max {r[:, i].max():7.2f} us")
