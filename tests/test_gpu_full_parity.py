"""Full-tensor GPU parity at the BASELINE configs: EVERY output element of every plan bench.py
times, against the fp64 oracle's direct convolution (Eq. 4; odd-size discard L1155).

For each (config, input kind) the oracle output is computed ONCE (the whole tensor) and every
variant / plan is compared with it element by element:

* FP32 fused kernel: the planner's plan without workspace, the stream-K workspace plan bench.py
  times (planner's choice), forced stream-K, forced split-C 1;
* batch shards of every rank at P = 2, 4, 8 (what `bench.py --gpus P` runs per rank) against the
  matching slice of the full oracle output, for the FP32, TF32 and FP16 bench plans;
* TF32 / 3xTF32 tcgen05 kernel with and without the stream-K workspace;
* F(4x4) (NEXT row N1), the NCHW front end (N2, both forms), the non-fused ablation (N3);
* FP16 / BF16 (N4) in a separate test against the oracle on the 16-bit input values (R18).

Bars: max|y - y_ref| / max|y_ref| <= 1e-4 (FP32, 3xTF32,
F(4x4)), <= 5e-3 (TF32), <= 5e-3 / 3e-2 (FP16 / BF16 vs the oracle on the 16-bit inputs); on
small-integer inputs every F(2x2) plan is bit-exact (16-bit: y = RNE(exact)).
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ppopp_yanwc20_b200.dist import shard_range
from synth_inputs import CONFIGS, make_inputs

pytestmark = pytest.mark.gpu

DEV = "cuda:0"
TOL = {"fp32": 1e-4, "tf32": 5e-3, "3xtf32": 1e-4, "f4": 1e-4, "nonfused_tf32": 5e-3}
HALF_TOL = {torch.float16: 5e-3, torch.bfloat16: 3e-2}
NAMES = ["tiny", "conv5_x", "conv4_x", "conv3_x", "conv2_x"]


@pytest.fixture(scope="module")
def wino():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanwc20_b200 as w
    w.lib()
    return w


def _err(y: torch.Tensor, ref: np.ndarray) -> float:
    yd = y.detach().double().cpu().numpy()
    assert np.isfinite(yd).all()
    den = float(np.max(np.abs(ref)))
    num = float(np.max(np.abs(yd - ref)))
    return num / den if den > 0 else (0.0 if num == 0 else float("inf"))


def _check(y, ref, exact, tol, what, failures):
    if exact:
        yd = y.detach().double().cpu().numpy()
        if not np.array_equal(yd, ref):
            failures.append(f"{what}: {int((yd != ref).sum())} of {ref.size} elements differ (bit-exact bar)")
    else:
        e = _err(y, ref)
        if not e <= tol:
            failures.append(f"{what}: max rel err {e:.3e} > {tol:g}")


def _ws(nbytes):
    return torch.zeros(max(int(nbytes), 16), dtype=torch.uint8, device=DEV)  # stream-K flags: zero


@pytest.mark.parametrize("kind", ["smallint", "uniform", "resnet"])
@pytest.mark.parametrize("name", NAMES)
def test_full_config_every_plan(wino, name, kind):
    cfg = CONFIGS[name]
    x, w = make_inputs(cfg, kind=kind)
    ref = oracle.direct_conv(x, w)  # the whole output tensor, once
    exact = kind == "smallint"
    N, C, K, H, W = cfg.N, cfg.C, cfg.K, cfg.H, cfg.W
    xd, wd = x.to(DEV), w.to(DEV)
    fails = []

    # ---- FP32 fused kernel: every plan ----
    u = wino.filter_transform(wd)
    ws = _ws(wino.conv_workspace_bytes(N, C, H, W, K))
    plans = {"planner (no workspace)": lambda: wino.conv2d(xd, u),
             "bench plan (stream-K workspace, planner)": lambda: wino.conv2d(xd, u, ws=ws),
             "forced stream-K": lambda: wino.conv2d(xd, u, ws=ws, stream_k="on"),
             "forced split-C 1": lambda: wino.conv2d(xd, u, split_c=1)}
    if N % 4 == 0 and (C + 7) // 8 >= 4:
        plans["forced split-C 2"] = lambda: wino.conv2d(xd, u, split_c=2)
    for what, fn in plans.items():
        y = fn()
        torch.cuda.synchronize()
        _check(y, ref, exact, TOL["fp32"], f"fp32 {what}", fails)

    # ---- per-rank batch shards (bench.py --gpus P) vs slices of the full oracle output ----
    u_tf32 = wino.filter_transform_tc(wd, "tf32")
    for P in (2, 4, 8):
        if N < P:
            continue
        for r in range(P):
            lo, hi = shard_range(N, r, P)
            xs = xd[..., lo:hi].contiguous()
            rs = np.ascontiguousarray(ref[..., lo:hi])
            y = wino.conv2d(xs, u, ws=_ws(wino.conv_workspace_bytes(hi - lo, C, H, W, K)))
            torch.cuda.synchronize()
            _check(y, rs, exact, TOL["fp32"], f"fp32 shard {r}/{P}", fails)
            y = wino.conv2d_tc(xs, u_tf32, ws=_ws(wino.tc_workspace_bytes(hi - lo, C, H, W, K)))
            torch.cuda.synchronize()
            _check(y, rs, exact, TOL["tf32"], f"tf32 shard {r}/{P}", fails)

    # ---- tcgen05 TF32 / 3xTF32 (a5') ----
    for v in ("tf32", "3xtf32"):
        ut = u_tf32 if v == "tf32" else wino.filter_transform_tc(wd, v)
        wst = _ws(wino.tc_workspace_bytes(N, C, H, W, K))
        for what, fn in {"no workspace": lambda: wino.conv2d_tc(xd, ut),
                         "bench plan (workspace)": lambda: wino.conv2d_tc(xd, ut, ws=wst)}.items():
            y = fn()
            torch.cuda.synchronize()
            _check(y, ref, exact, TOL[v], f"{v} {what}", fails)

    # ---- NEXT rows ----
    # F(4x4) (N1), any shape: no exact input class (G4 has 1/6, 1/12, 1/24)
    u4 = wino.filter_transform_f4(wd)
    y = wino.conv2d_f4(xd, u4, ws=_ws(wino.f4_workspace_bytes(N, C, H, W, K)))
    torch.cuda.synchronize()
    _check(y, ref, False, TOL["f4"], "f4 bench plan", fails)
    xn = xd.permute(3, 0, 1, 2).contiguous()
    un = wino.filter_transform_kcrs(wd.permute(3, 0, 1, 2).contiguous())
    refn = np.ascontiguousarray(ref.transpose(3, 0, 1, 2))
    y = wino.conv2d_nchw(xn, un, ws=_ws(wino.nchw_workspace_bytes(N, C, H, W, K)))
    torch.cuda.synchronize()
    _check(y, refn, exact, TOL["fp32"], "nchw (transpose + CHWN kernel)", fails)
    y = wino.conv2d_nchw(xn, un)
    torch.cuda.synchronize()
    _check(y, refn, exact, TOL["fp32"], "nchw (strided kernel)", fails)
    wsn = _ws(wino.nonfused_workspace_bytes(N, C, H, W, K))
    for tf32 in (False, True):
        y = wino.conv2d_nonfused(xd, u, wsn, tf32=tf32)
        torch.cuda.synchronize()
        _check(y, ref, exact, TOL["nonfused_tf32" if tf32 else "fp32"], f"nonfused tf32={tf32}", fails)
    assert not fails, "\n".join(fails)


@pytest.mark.parametrize("dt", [torch.float16, torch.bfloat16], ids=["fp16", "bf16"])
@pytest.mark.parametrize("kind", ["smallint", "uniform", "resnet"])
@pytest.mark.parametrize("name", NAMES)
def test_full_config_half(wino, name, kind, dt):
    """N4 at full size, whole tensors: the bench plan (workspace) and no workspace, plus every rank's
    shard at P = 2, 4, 8; the oracle runs on the 16-bit input values (reading R18)."""
    cfg = CONFIGS[name]
    x, w = make_inputs(cfg, kind=kind)
    xh, wh = x.to(dt), w.to(dt)
    ref = oracle.direct_conv(xh.float(), wh.float())
    exact = kind == "smallint"
    if exact:  # y = RNE(exact integer result)
        ref = torch.from_numpy(ref).to(torch.float32).to(dt).double().numpy()
    N, C, K, H, W = cfg.N, cfg.C, cfg.K, cfg.H, cfg.W
    xd = xh.to(DEV)
    uh = wino.filter_transform_half(wh.to(DEV))
    fails = []
    for what, fn in {"no workspace": lambda: wino.conv2d_half(xd, uh),
                     "bench plan (workspace)": lambda: wino.conv2d_half(
                         xd, uh, ws=_ws(wino.half_workspace_bytes(N, C, H, W, K)))}.items():
        y = fn()
        torch.cuda.synchronize()
        _check(y, ref, exact, HALF_TOL[dt], f"{dt} {what}", fails)
    for P in (2, 4, 8):
        if N < P:
            continue
        for r in range(P):
            lo, hi = shard_range(N, r, P)
            y = wino.conv2d_half(xd[..., lo:hi].contiguous(), uh,
                                 ws=_ws(wino.half_workspace_bytes(hi - lo, C, H, W, K)))
            torch.cuda.synchronize()
            _check(y, np.ascontiguousarray(ref[..., lo:hi]), exact, HALF_TOL[dt], f"{dt} shard {r}/{P}", fails)
    assert not fails, "\n".join(fails)
