"""Small launches of every kernel variant for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_yanwc20_b200 as wino
from synth_inputs import Conv3x3Config, make_inputs

shapes = [Conv3x3Config("a", 32, 16, 64, 6, 6),    # FP32 WS (TMA) + tc MM=64 + half MM=64 TMA
          Conv3x3Config("b", 5, 9, 70, 7, 5),      # FP32 generic cp.async 4 B, half gather
          Conv3x3Config("c", 8, 12, 132, 5, 4),    # FP32 generic cp.async 16 B, tc MM=128 XM=1, half boxes N=8
          Conv3x3Config("d", 64, 8, 256, 3, 3),    # tc MM=128 TMA, half MM=128 TMA
          Conv3x3Config("e", 16, 24, 40, 7, 9)]    # small-N WS boxes, half MM=64 boxes N=16
only = sys.argv[1] if len(sys.argv) > 1 else "all"
for cfg in shapes:
    x, w = make_inputs(cfg)
    x, w = x.cuda(), w.cuda()
    if only in ("all", "fp32", "sk"):
        u = wino.filter_transform(w)
        y = wino.conv2d(x, u)
        if cfg.N % 32 == 0 or cfg.N in (4, 8, 16):  # stream-K (forced) + fixup
            ws = torch.zeros(wino.conv_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8,
                             device="cuda")
            y = wino.conv2d(x, u, ws=ws, stream_k="on")
            if cfg.K > 64:
                y = wino.conv2d_tc(x, wino.filter_transform_tc(w, "tf32"), ws=ws.new_empty(
                    wino.tc_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K)), stream_k="on")
            wsh = torch.empty(wino.half_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8,
                              device="cuda")
            y = wino.conv2d_half(x.half(), wino.filter_transform_half(w.half()), ws=wsh, stream_k="on")
            if cfg.N % 16 == 0:
                y = wino.conv2d_f4(x, wino.filter_transform_f4(w), stream_k="on", ws=torch.empty(
                    wino.f4_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8, device="cuda"))
        wsn = torch.zeros(wino.nchw_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8,
                          device="cuda")
        y = wino.conv2d_nchw(x.permute(3, 0, 1, 2).contiguous(),
                             wino.filter_transform_kcrs(w.permute(3, 0, 1, 2).contiguous()), ws=wsn)
        if cfg.N % 4 == 0:
            y = wino.conv2d(x, u, split_c=2)  # cluster split-C
        y = wino.conv2d_nchw(x.permute(3, 0, 1, 2).contiguous(), wino.filter_transform_kcrs(w.permute(3, 0, 1, 2).contiguous()))
        ws = torch.empty(wino.nonfused_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8, device="cuda")
        y = wino.conv2d_nonfused(x, u, ws)
        if cfg.N % 16 == 0 and cfg.K % 4 == 0:
            y = wino.conv2d_f4(x, wino.filter_transform_f4(w))
    if only in ("all", "tc"):
        for v in ("tf32", "3xtf32"):
            y = wino.conv2d_tc(x, wino.filter_transform_tc(w, v))
    if only in ("all", "half"):
        for dt in (torch.float16, torch.bfloat16):
            y = wino.conv2d_half(x.to(dt), wino.filter_transform_half(w.to(dt)))
if only in ("all", "fp32", "ml"):
    # multi-layer persistent launch (fused_fp32_ml.cuh): N % 32 == 0, N = 16 boxes and vmode N = 4 / 8 in one launch
    cfgs = [Conv3x3Config("m1", 32, 16, 64, 6, 6), Conv3x3Config("m2", 16, 24, 40, 7, 9),
            Conv3x3Config("m3", 4, 40, 72, 7, 7), Conv3x3Config("m4", 8, 8, 16, 5, 5)]
    lay = []
    for c in cfgs:
        x, w = make_inputs(c)
        x, w = x.cuda(), w.cuda()
        lay.append((x, wino.filter_transform(w), torch.empty((c.K, c.H, c.W, c.N), device="cuda")))
    ws = torch.zeros(wino.conv_multi_workspace_bytes([(c.N, c.C, c.H, c.W, c.K) for c in cfgs]), dtype=torch.uint8,
                     device="cuda")
    wino.conv2d_multi(lay, ws)
torch.cuda.synchronize()
print("ok")
