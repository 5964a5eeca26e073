"""Run the 16-bit tcgen05 kernel with a trace build (build_ab/libwino_trace16.so, -DWINO_TC16_TRACE) and
print per-channel-block event times of CTA 0 (clock64, relative)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["WINO_LIB_PATH"] = os.path.abspath("build_ab/libwino_trace16.so")
import torch
import paper_conf_ppopp_yanwc20_b200 as wino
from synth_inputs import CONFIGS, make_inputs
name = sys.argv[1] if len(sys.argv) > 1 else "conv3_x"
cfg = CONFIGS[name]
x, w = make_inputs(cfg)
xh, wh = x.half().cuda(), w.half().cuda()
u = wino.filter_transform_half(wh)
for _ in range(3):
    y = wino.conv2d_half(xh, u)
torch.cuda.synchronize()
L = wino.lib()
NE, NC = 8, 256
buf = (ctypes.c_ulonglong * (NE * NC))()
L.wino_debug_tc16_trace.argtypes = [ctypes.c_void_p, ctypes.c_int]
L.wino_debug_tc16_trace(ctypes.cast(buf, ctypes.c_void_p), NE * NC)
ev = [[buf[e * NC + c] for c in range(NC)] for e in range(NE)]
t0 = min(v for v in ev[0] if v)
names = ["x_issue", "u_issue", "vfull_w0", "vfull_w1", "mma_vfull", "mma_issue", "vfull_w2", "vfull_w3"]
print("gcb " + " ".join(f"{n:>10s}" for n in names))
for c in range(min(NC, 64)):
    if not any(ev[e][c] for e in range(NE)):
        break
    print(f"{c:3d} " + " ".join(f"{(ev[e][c] - t0) if ev[e][c] else -1:10d}" for e in range(NE)))
