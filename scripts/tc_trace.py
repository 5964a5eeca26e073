"""Run the tcgen05 kernel once on a config with a trace build and print per-cb event times (CTA 0)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["WINO_LIB_PATH"] = os.path.abspath("build_ab/libwino_trace.so")
import torch
import paper_conf_ppopp_yanwc20_b200 as wino
from synth_inputs import CONFIGS, make_inputs
name = sys.argv[1] if len(sys.argv) > 1 else "conv5_x"
variant = sys.argv[2] if len(sys.argv) > 2 else "tf32"
cfg = CONFIGS[name]
x, w = make_inputs(cfg)
x, w = x.cuda(), w.cuda()
u = wino.filter_transform_tc(w, variant)
for _ in range(3):
    y = wino.conv2d_tc(x, u)
torch.cuda.synchronize()
L = wino.lib()
buf = (ctypes.c_ulonglong * (8 * 128))()
L.wino_debug_tc_trace.argtypes = [ctypes.c_void_p, ctypes.c_int]
L.wino_debug_tc_trace(ctypes.cast(buf, ctypes.c_void_p), 8 * 128)
ev = [[buf[e * 128 + c] for c in range(128)] for e in range(8)]
t0 = min(v for v in ev[0] if v) if any(ev[0]) else 0
ncb = -(-cfg.C // 8)
names = ["x_issue", "u_issue", "itf_xfull", "itf_done", "mma_vfull", "mma_issued"]
print("cb " + " ".join(f"{n:>10s}" for n in names))
for c in range(min(ncb, 128)):
    print(f"{c:3d} " + " ".join(f"{(ev[e][c] - t0) if ev[e][c] else -1:10d}" for e in range(6)))
print("epilogue start", ev[6][0] - t0, "end", ev[7][0] - t0)
