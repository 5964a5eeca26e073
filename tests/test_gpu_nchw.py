"""GPU parity of NEXT row N2 -- the NCHW front end (Sec. 8.4):
wino_filter_transform_kcrs + wino_conv2d_f2x3_fwd_nchw against the fp64 oracle
(Eq. 4; the oracle works in the paper's CHWN / CRSK layouts, so inputs are
permuted on the host -- a layout change, no arithmetic).

Bars as tests/test_gpu_parity.py: bit-exact on small integers, <= 1e-4 of
max|y| on random inputs; u from the KCRS weight equals u from CRSK bit for bit.
"""
import numpy as np
import pytest
import torch

import oracle
from synth_inputs import CONFIGS, Conv3x3Config, make_inputs

pytestmark = pytest.mark.gpu

FP32_TOL = 1e-4
DEV = "cuda:0"


@pytest.fixture(scope="module")
def wino():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanwc20_b200 as w
    w.lib()
    return w


def _nchw(x_chwn):
    return x_chwn.permute(3, 0, 1, 2).contiguous()


def _kcrs(w_crsk):
    return w_crsk.permute(3, 0, 1, 2).contiguous()


def _run(wino, x, w):
    u = wino.filter_transform_kcrs(_kcrs(w).to(DEV))
    y = wino.conv2d_nchw(_nchw(x).to(DEV), u)
    torch.cuda.synchronize()
    return u.cpu(), y.cpu().permute(1, 2, 3, 0).contiguous()  # (N,K,H,W) -> (K,H,W,N)


SHAPES = [
    (1, 1, 1, 1, 1), (1, 8, 8, 8, 8), (3, 7, 5, 5, 5), (2, 9, 65, 7, 7), (4, 20, 70, 13, 9),
    (5, 17, 130, 6, 10), (32, 16, 64, 9, 9), (2, 64, 64, 16, 16), (7, 40, 72, 11, 12), (1, 3, 3, 1, 17),
]


@pytest.mark.parametrize("shape", SHAPES, ids=[str(s) for s in SHAPES])
def test_nchw_small_int_bit_exact(wino, shape):
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("nchw", N, C, K, H, W), kind="smallint")
    u, y = _run(wino, x, w)
    assert np.array_equal(u.double().numpy(), oracle.filter_transform(w))
    assert np.array_equal(y.double().numpy(), oracle.direct_conv(x, w))


@pytest.mark.parametrize("shape", SHAPES, ids=[str(s) for s in SHAPES])
def test_nchw_random(wino, shape):
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("nchw", N, C, K, H, W), kind="uniform", seed_x=31, seed_w=32)
    u, y = _run(wino, x, w)
    assert np.array_equal(u.numpy(), wino.filter_transform(w.to(DEV)).cpu().numpy())
    assert oracle.max_rel_err(y.double().numpy(), oracle.direct_conv(x, w)) <= FP32_TOL


def test_nchw_matches_chwn_kernel(wino):
    """Same convolution through both layouts: the NCHW path and the CHWN path agree
    within the FP32 bound (their per-output summation orders are the same kernel's)."""
    cfg = Conv3x3Config("both", 16, 64, 128, 14, 14)
    x, w = make_inputs(cfg)
    u = wino.filter_transform(w.to(DEV))
    y_chwn = wino.conv2d(x.to(DEV), u, split_c=1)
    y_nchw = wino.conv2d_nchw(_nchw(x).to(DEV), u).permute(1, 2, 3, 0)
    torch.cuda.synchronize()
    d = (y_chwn.double() - y_nchw.double()).abs().max() / y_chwn.double().abs().max()
    assert float(d) <= FP32_TOL


def _run_ws(wino, x, w):
    u = wino.filter_transform_kcrs(_kcrs(w).to(DEV))
    N, C, H, W = x.shape[3], x.shape[0], x.shape[1], x.shape[2]
    ws = torch.zeros(wino.nchw_workspace_bytes(N, C, H, W, w.shape[3]), dtype=torch.uint8, device=DEV)
    y = wino.conv2d_nchw(_nchw(x).to(DEV), u, ws=ws)
    torch.cuda.synchronize()
    return y.cpu().permute(1, 2, 3, 0).contiguous()


WS_SHAPES = SHAPES + [(64, 24, 40, 10, 9), (4, 40, 72, 7, 7), (16, 13, 68, 12, 5)]


@pytest.mark.parametrize("shape", WS_SHAPES, ids=[str(s) for s in WS_SHAPES])
def test_nchw_ws_small_int_bit_exact(wino, shape):
    """Transpose -> CHWN fused kernel -> transpose (wino_conv2d_f2x3_fwd_nchw_ws)."""
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("nchw", N, C, K, H, W), kind="smallint")
    assert np.array_equal(_run_ws(wino, x, w).double().numpy(), oracle.direct_conv(x, w))


@pytest.mark.parametrize("shape", WS_SHAPES, ids=[str(s) for s in WS_SHAPES])
def test_nchw_ws_random(wino, shape):
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("nchw", N, C, K, H, W), kind="uniform", seed_x=41, seed_w=42)
    y = _run_ws(wino, x, w)
    assert oracle.max_rel_err(y.double().numpy(), oracle.direct_conv(x, w)) <= FP32_TOL


def test_nchw_ws_short_workspace_rejected(wino):
    x = torch.zeros((32, 8, 4, 4), device=DEV)
    u = torch.zeros((8, 4, 4, 16), device=DEV)
    with pytest.raises(wino.WinoError, match="INVALID_ARG"):
        wino.conv2d_nchw(x, u, ws=torch.empty(1024, dtype=torch.uint8, device=DEV))


@pytest.mark.parametrize("shape", [(2, 4, 64, 192, 192), (1, 3, 130, 131, 129)], ids=["KHW=2.36M", "KHW=2.20M"])
def test_nchw_ws_large_plane_transposes(wino, shape):
    """K*H*W (and C*H*W rows) beyond 65535 transpose tiles in one grid dimension: the 2-D
    transposes use a 1-D tile grid (the round-1 grid.y = K*H*W/32 broke above 2,097,120)."""
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("nchw-big", N, C, K, H, W), kind="smallint")
    y = _run_ws(wino, x, w)
    assert np.array_equal(y.double().numpy(), oracle.direct_conv(x, w))
