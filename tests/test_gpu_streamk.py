"""GPU parity of the stream-K plan of the FP32 warp-specialised kernel (wino_conv2d_f2x3_fwd_ws).

Stream-K cuts the (tile, channel block) iteration space of Alg. 1 (L351-355) into one equal
range per SM; a tile cut at a range boundary is accumulated in pieces whose partial outputs
(Eq. 8 is linear) are added by a fixup kernel in CTA order.  Only the summation order over C
changes (reading R7), so: small-integer inputs stay bit-exact against Eq. 4 (every partial sum
is exact), random inputs stay within the FP32 bar, and repeated runs
are bit-identical.
"""
import ctypes

import numpy as np
import pytest
import torch

import oracle
from synth_inputs import CONFIGS, Conv3x3Config, make_inputs

pytestmark = pytest.mark.gpu

DEV = "cuda:0"
FP32_TOL = 1e-4


@pytest.fixture(scope="module")
def wino():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanwc20_b200 as w
    w.lib()
    return w


def _ws(wino, cfg):
    return torch.zeros(wino.conv_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8, device=DEV)


def _run(wino, x, w, cfg, mode):
    u = wino.filter_transform(w.to(DEV))
    y = wino.conv2d(x.to(DEV), u, ws=_ws(wino, cfg), stream_k=mode)
    torch.cuda.synchronize()
    return y.cpu()


# (N, C, K, H, W) on the warp-specialised kernel (N % 32 == 0 or N in {4, 8, 16}; K % 4 == 0):
# ranges much shorter than a tile (C = 512, few tiles), ranges spanning many tiles, channel
# and filter tails, odd planes, the batch shards of the BASELINE layers at P = 8.
SK_SHAPES = [
    (32, 8, 64, 2, 2), (32, 512, 64, 3, 3), (4, 512, 512, 7, 7), (8, 256, 256, 14, 14),
    (16, 128, 128, 12, 10), (32, 64, 64, 30, 30), (64, 13, 132, 5, 9), (96, 7, 68, 9, 2),
    (32, 1, 4, 1, 1), (4, 24, 40, 3, 5),
]


@pytest.mark.parametrize("shape", SK_SHAPES, ids=[str(s) for s in SK_SHAPES])
def test_streamk_small_int_bit_exact(wino, shape):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("sk", N, C, K, H, W)
    x, w = make_inputs(cfg, kind="smallint")
    y = _run(wino, x, w, cfg, "on")
    assert np.array_equal(y.double().numpy(), oracle.direct_conv(x, w))


@pytest.mark.parametrize("shape", SK_SHAPES, ids=[str(s) for s in SK_SHAPES])
def test_streamk_random(wino, shape):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("sk", N, C, K, H, W)
    x, w = make_inputs(cfg, kind="uniform", seed_x=31, seed_w=32)
    y = _run(wino, x, w, cfg, "on")
    assert np.isfinite(y.numpy()).all()
    assert oracle.max_rel_err(y.double().numpy(), oracle.direct_conv(x, w)) <= FP32_TOL


@pytest.mark.parametrize("P", [2, 4, 8])
def test_streamk_batch_shards(wino, P):
    """The per-rank batch shards of every BASELINE layer at P ranks (planner's choice + workspace)."""
    for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x"):
        cfg = CONFIGS[name].with_batch(CONFIGS[name].N // P)
        x, w = make_inputs(cfg, kind="smallint")
        y = _run(wino, x, w, cfg, "auto")
        assert np.array_equal(y.double().numpy(), oracle.direct_conv(x, w)), (name, cfg.N)


def test_streamk_deterministic_and_matches_regular(wino):
    cfg = CONFIGS["conv4_x"].with_batch(32)
    x, w = make_inputs(cfg)
    xd, u = x.to(DEV), wino.filter_transform(w.to(DEV))
    ws = _ws(wino, cfg)
    y1 = wino.conv2d(xd, u, ws=ws, stream_k="on")
    for _ in range(3):
        y2 = torch.full_like(y1, float("nan"))
        wino.conv2d(xd, u, out=y2, ws=ws, stream_k="on")
        torch.cuda.synchronize()
        assert torch.equal(y1, y2)
    y0 = wino.conv2d(xd, u, ws=ws, stream_k="off")
    torch.cuda.synchronize()
    err = (y1.double() - y0.double()).abs().max() / y0.double().abs().max()
    assert float(err) <= FP32_TOL


def test_streamk_argument_errors(wino):
    cfg = Conv3x3Config("sk", 32, 16, 64, 4, 4)
    x = torch.zeros((cfg.C, cfg.H, cfg.W, cfg.N), device=DEV)
    u = torch.zeros((cfg.C, 4, 4, cfg.K), device=DEV)
    y = torch.empty((cfg.K, cfg.H, cfg.W, cfg.N), device=DEV)
    L = wino.lib()
    p = ctypes.c_void_p
    small = torch.empty(1024, dtype=torch.uint8, device=DEV)
    st = L.wino_conv2d_f2x3_fwd_ws(p(x.data_ptr()), p(u.data_ptr()), p(y.data_ptr()), cfg.N, cfg.C, cfg.H, cfg.W,
                                   cfg.K, 1, 1, 2, p(small.data_ptr()), 1024, None)
    assert st == 1  # forced stream-K with a short workspace
    nbytes = wino.conv_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K)
    st = L.wino_conv2d_f2x3_fwd_ws(p(x.data_ptr()), p(u.data_ptr()), p(y.data_ptr()), cfg.N, cfg.C, cfg.H, cfg.W,
                                   cfg.K, 1, 1, 0, p(y.data_ptr()), nbytes, None)
    assert st == 1  # workspace overlapping y
    st = L.wino_conv2d_f2x3_fwd_ws(p(x.data_ptr()), p(u.data_ptr()), p(y.data_ptr()), cfg.N, cfg.C, cfg.H, cfg.W,
                                   cfg.K, 1, 1, 3, None, 0, None)
    assert st == 1  # unknown mode
    st = L.wino_conv2d_f2x3_fwd_ws(p(x.data_ptr()), p(u.data_ptr()), p(y.data_ptr()), cfg.N, cfg.C, cfg.H, cfg.W,
                                   cfg.K, 1, 1, 1, None, 0, None)
    assert st == 0  # stream-K off needs no workspace


# TF32 / 3xTF32 tcgen05 kernel, forced stream-K (TMA x paths: N % 32 == 0 or N in {4, 8, 16})
TC_SK = [(4, 512, 512, 7, 7), (8, 256, 256, 14, 14), (16, 128, 128, 12, 10), (32, 64, 64, 30, 30),
         (32, 72, 200, 5, 9)]


@pytest.mark.parametrize("variant,tol", [("tf32", 5e-3), ("3xtf32", 1e-4)])
@pytest.mark.parametrize("shape", TC_SK, ids=[str(s) for s in TC_SK])
def test_tc_streamk(wino, shape, variant, tol):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("sk", N, C, K, H, W)
    for kind in ("smallint", "uniform"):
        x, w = make_inputs(cfg, kind=kind)
        u = wino.filter_transform_tc(w.to(DEV), variant)
        ws = torch.empty(wino.tc_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
        y = wino.conv2d_tc(x.to(DEV), u, ws=ws, stream_k="on").cpu()
        torch.cuda.synchronize()
        ref = oracle.direct_conv(x, w)
        if kind == "smallint":  # exact in TF32
            assert np.array_equal(y.double().numpy(), ref)
        else:
            assert oracle.max_rel_err(y.double().numpy(), ref) <= tol


def test_streamk_leaves_flags_zero(wino):
    """The in-kernel reduction of cut tiles clears every flag word it consumed (include/wino.h:
    one zero-fill of the workspace serves any number of calls)."""
    cfg = CONFIGS["conv5_x"].with_batch(8)
    x, w = make_inputs(cfg, kind="smallint")
    ws = _ws(wino, cfg)
    u = wino.filter_transform(w.to(DEV))
    ref = oracle.direct_conv(x, w)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    slot = 64 * 4 * 32 * 4
    for _ in range(3):
        y = wino.conv2d(x.to(DEV), u, ws=ws, stream_k="on")
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().double().numpy(), ref)
        counters = ws[2 * sms * slot: 2 * sms * slot + 4 * sms]  # after the 2 slots per CTA
        assert int(counters.count_nonzero()) == 0
