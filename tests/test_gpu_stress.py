"""Repeated-run stress of the tcgen05 and FFMA kernels on small-integer inputs, where every plan is
exact: a rare pipeline hazard shows up as a run that differs from Eq. 4.

These shapes reproduced the round-1 intermittent wrong partial outputs of the 64-filter TF32
stream-K plan and, after the round-2 ITF / epilogue rework, of 3xTF32 conv2_x on every run: both
were the missing fence.proxy.async between generic-proxy reads of a TMA-filled shared-memory slot
and its next TMA (async-proxy) refill.  Each case runs REPS times and must be
bit-exact every time."""
import numpy as np
import pytest
import torch

import oracle
from synth_inputs import CONFIGS, Conv3x3Config, make_inputs

pytestmark = pytest.mark.gpu
DEV = "cuda:0"
REPS = 12


@pytest.fixture(scope="module")
def wino():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanwc20_b200 as w
    w.lib()
    return w


CASES = [  # (variant, shape (N, C, K, H, W), stream_k)
    ("tf32", (32, 64, 64, 30, 30), "on"), ("tf32", (32, 64, 48, 14, 14), "on"),
    ("3xtf32", (256, 64, 64, 56, 56), "off"), ("tf32", (256, 64, 64, 56, 56), "off"),
    ("3xtf32", (32, 72, 200, 9, 7), "on"), ("tf32", (4, 512, 512, 7, 7), "on"),
    ("fp16", (32, 64, 64, 30, 30), "on"), ("fp16", (256, 64, 64, 56, 56), "off"),
    ("bf16", (8, 256, 256, 14, 14), "on"),
    ("fp32", (32, 64, 64, 30, 30), "on"), ("fp32", (128, 128, 128, 28, 28), "off"),
    ("f4", (32, 64, 64, 30, 30), "on"),
]


@pytest.mark.parametrize("variant,shape,sk", CASES, ids=[f"{v}-{s}-sk{k}" for v, s, k in CASES])
def test_repeated_runs_exact(wino, variant, shape, sk):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("stress", N, C, K, H, W)
    x, w = make_inputs(cfg, kind="smallint")
    ref = oracle.direct_conv(x, w)
    xd, wd = x.to(DEV), w.to(DEV)
    if variant in ("tf32", "3xtf32"):
        u = wino.filter_transform_tc(wd, variant)
        ws = torch.empty(wino.tc_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
        run = lambda: wino.conv2d_tc(xd, u, ws=ws, stream_k=sk)  # noqa: E731
    elif variant in ("fp16", "bf16"):
        dt = torch.float16 if variant == "fp16" else torch.bfloat16
        ref = torch.from_numpy(ref).float().to(dt).double().numpy()  # y = RNE(exact)
        xd, u = xd.to(dt), wino.filter_transform_half(wd.to(dt))
        ws = torch.empty(wino.half_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
        run = lambda: wino.conv2d_half(xd, u, ws=ws, stream_k=sk)  # noqa: E731
    elif variant == "f4":  # no exact input class for F(4x4): compare runs with each other
        u = wino.filter_transform_f4(wd)
        ws = torch.empty(wino.f4_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
        run = lambda: wino.conv2d_f4(xd, u, ws=ws, stream_k=sk)  # noqa: E731
        ref = run().double().cpu().numpy()
        assert oracle.max_rel_err(ref, oracle.direct_conv(x, w)) <= 1e-4
    else:
        u = wino.filter_transform(wd)
        ws = torch.zeros(wino.conv_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
        run = lambda: wino.conv2d(xd, u, ws=ws, stream_k=sk)  # noqa: E731
    bad_runs = []
    for r in range(REPS):
        y = run()
        torch.cuda.synchronize()
        nbad = int((y.double().cpu().numpy() != ref).sum())
        if nbad:
            bad_runs.append((r, nbad))
    assert not bad_runs, f"runs with wrong outputs (run, count): {bad_runs}"
