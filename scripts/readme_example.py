import sys, os
sys.path.insert(0, os.getcwd())

import torch, paper_conf_ppopp_yanwc20_b200 as wino
x = torch.randn(128, 28, 28, 64, device="cuda")          # (C, H, W, N), the paper's CHWN
w = torch.randn(128, 3, 3, 128, device="cuda")           # (C, 3, 3, K), CRSK
u = wino.filter_transform(w)                              # (C, 4, 4, K) = G w G^T
y = wino.conv2d(x, u)                                     # (K, H, W, N), pad 1, stride 1, FP32
ws = torch.zeros(wino.conv_workspace_bytes(64, 128, 28, 28, 128), dtype=torch.uint8, device="cuda")
y = wino.conv2d(x, u, ws=ws)                              # + stream-K plans where they pay
y16 = wino.conv2d_half(x.half(), wino.filter_transform_half(w.half()))   # FP16 on tcgen05
ytc = wino.conv2d_tc(x, wino.filter_transform_tc(w, "tf32"))             # TF32 on tcgen05

torch.cuda.synchronize()
print('readme ok', y.shape, y16.dtype, ytc.shape)
