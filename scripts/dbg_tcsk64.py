"""Debug: forced stream-K of the TF32 kernel with 64-filter tiles (build -DWINO_TC_SK_MM64)."""
import os, sys
sys.path.insert(0, os.getcwd())
os.environ["WINO_LIB_PATH"] = os.path.abspath("build_ab/libwino_tcsk64.so")
import numpy as np, torch
import paper_conf_ppopp_yanwc20_b200 as wino, oracle
from synth_inputs import Conv3x3Config, make_inputs
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 5
for shape in [(32, 64, 64, 30, 30), (32, 64, 64, 16, 16)]:
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("s", N, C, K, H, W), kind="smallint")
    u = wino.filter_transform_tc(w.cuda(), "tf32")
    ws = torch.empty(wino.tc_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device="cuda")
    ref = oracle.direct_conv(x, w)
    for r in range(reps):
        y = wino.conv2d_tc(x.cuda(), u, ws=ws, stream_k="on").cpu().double().numpy()
        print(shape, r, "bad", int((y != ref).sum()))
