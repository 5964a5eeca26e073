"""GPU parity for NEXT row N1: fused F(4x4,3x3) FP32 kernel vs the fp64 oracle.

The F(4x4) transforms carry the constants 1/4, 1/6, 1/12, 1/24 (G4) and 4, 5,
2, 8 (B4, A4), so unlike F(2x2) no input class is exact in FP32: every case is
compared with a relative tolerance (F4_TOL), against
both the direct definition (Eq. 4) and the oracle's step-by-step F(4x4)
Winograd (oracle.winograd_f4_conv).  The transformed filter u4 is compared
with oracle.filter_transform_f4 element by element.
"""
import numpy as np
import pytest
import torch

import oracle
from synth_inputs import CONFIGS, Conv3x3Config, make_inputs

pytestmark = pytest.mark.gpu

F4_TOL = 1e-4   # FP32 bar of north_star, kept for F(4x4)
FTF4_TOL = 1e-6
DEV = "cuda:0"


@pytest.fixture(scope="module")
def wino():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanwc20_b200 as w
    w.lib()
    return w


def _run(wino, x, w):
    u4 = wino.filter_transform_f4(w.to(DEV))
    y = wino.conv2d_f4(x.to(DEV), u4)
    torch.cuda.synchronize()
    return u4.cpu(), y.cpu()


# (N, C, K, H, W): N % 16 == 0, K % 4 == 0.  Channel tails (C % 4), filter tails
# (K % 64), plane tails (H, W % 4), 1x1 planes, more tiles than SMs.
F4_EDGE = [
    (16, 1, 4, 1, 1), (16, 3, 8, 5, 5), (16, 7, 68, 9, 7), (32, 13, 132, 6, 10),
    (16, 64, 64, 14, 14), (48, 5, 36, 4, 4), (16, 2, 4, 3, 17), (32, 16, 64, 40, 40),
    (64, 9, 200, 7, 7),
]


@pytest.mark.parametrize("kind", ["uniform", "smallint"])
@pytest.mark.parametrize("shape", F4_EDGE, ids=[str(s) for s in F4_EDGE])
def test_f4_edge_shapes(wino, shape, kind):
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("f4edge", N, C, K, H, W), kind=kind)
    u4, y = _run(wino, x, w)
    assert oracle.max_rel_err(u4.double().numpy(), oracle.filter_transform_f4(w)) <= FTF4_TOL
    yd = y.double().numpy()
    assert np.isfinite(yd).all()
    assert oracle.max_rel_err(yd, oracle.direct_conv(x, w)) <= F4_TOL


def test_f4_matches_oracle_f4_winograd(wino):
    """Same result as the oracle's naive F(4x4) steps (not only the definition)."""
    x, w = make_inputs(Conv3x3Config("f4", 32, 24, 72, 13, 11), kind="uniform")
    _, y = _run(wino, x, w)
    assert oracle.max_rel_err(y.double().numpy(), oracle.winograd_f4_conv(x, w)) <= F4_TOL


@pytest.mark.parametrize("kind", ["uniform", "resnet"])
@pytest.mark.parametrize("name", ["conv2_x", "conv3_x", "conv4_x", "conv5_x"])
def test_f4_full_configs(wino, name, kind):
    """BASELINE configs at full size (no workspace), every output element vs Eq. 4."""
    cfg = CONFIGS[name]
    x, w = make_inputs(cfg, kind=kind)
    u4, y = _run(wino, x, w)
    assert oracle.max_rel_err(u4.double().numpy(), oracle.filter_transform_f4(w)) <= FTF4_TOL
    assert np.isfinite(y.numpy()).all()
    assert oracle.max_rel_err(y.double().numpy(), oracle.direct_conv(x, w)) <= F4_TOL


def test_f4_deterministic_and_overwrites(wino):
    x, w = make_inputs(Conv3x3Config("f4", 32, 20, 68, 9, 9), kind="uniform")
    xd, wd = x.to(DEV), w.to(DEV)
    u4 = wino.filter_transform_f4(wd)
    y1 = wino.conv2d_f4(xd, u4)
    y2 = torch.full_like(y1, float("nan"))
    wino.conv2d_f4(xd, u4, out=y2)
    torch.cuda.synchronize()
    assert torch.equal(y1, y2)


# Generic path (cp.async gathers): N % 16 != 0 and / or K % 4 != 0 -- any N, K, C (L1281)
F4_GEN = [
    (1, 8, 8, 8, 8), (1, 1, 1, 1, 1), (3, 7, 8, 5, 5), (33, 9, 65, 7, 7), (3, 1, 65, 9, 6),
    (8, 4, 8, 5, 5), (16, 4, 6, 5, 5), (24, 3, 8, 4, 4), (5, 17, 130, 6, 10), (33, 64, 64, 14, 14),
    (2, 9, 3, 17, 3), (20, 12, 72, 12, 12),
]


@pytest.mark.parametrize("kind", ["uniform", "smallint"])
@pytest.mark.parametrize("shape", F4_GEN, ids=[str(s) for s in F4_GEN])
def test_f4_generic_shapes(wino, shape, kind):
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("f4gen", N, C, K, H, W), kind=kind)
    u4, y = _run(wino, x, w)
    assert oracle.max_rel_err(u4.double().numpy(), oracle.filter_transform_f4(w)) <= FTF4_TOL
    yd = y.double().numpy()
    assert np.isfinite(yd).all()
    assert oracle.max_rel_err(yd, oracle.direct_conv(x, w)) <= F4_TOL


@pytest.mark.parametrize("shape", [(3, 13, 65, 9, 9), (1, 512, 512, 7, 7), (33, 9, 65, 7, 7)])
def test_f4_generic_stream_k(wino, shape):
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("f4gsk", N, C, K, H, W), kind="uniform", seed_x=63, seed_w=64)
    u4 = wino.filter_transform_f4(w.to(DEV))
    ws = torch.empty(wino.f4_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
    y = wino.conv2d_f4(x.to(DEV), u4, ws=ws, stream_k="on")
    torch.cuda.synchronize()
    assert oracle.max_rel_err(y.cpu().double().numpy(), oracle.direct_conv(x, w)) <= F4_TOL


def test_f4_generic_matches_tma_path(wino):
    """The same convolution through the TMA path (N = 32) and the generic path (a batch shard of
    N = 31 plus the last image as N = 1): within the FP32 bar of each other image by image."""
    cfg = Conv3x3Config("f4ab", 32, 24, 68, 10, 10)
    x, w = make_inputs(cfg, kind="uniform", seed_x=65, seed_w=66)
    _, y = _run(wino, x, w)
    _, ya = _run(wino, x[..., :31].contiguous(), w)
    _, yb = _run(wino, x[..., 31:].contiguous(), w)
    yg = torch.cat([ya, yb], dim=-1).double()
    assert float((yg - y.double()).abs().max() / y.double().abs().max()) <= F4_TOL


# stream-K plan (workspace): ranges shorter than a tile, spanning tiles, tails; forced and auto
F4_SK = [(16, 512, 512, 7, 7), (32, 256, 256, 14, 14), (16, 64, 64, 28, 28), (32, 13, 132, 6, 10),
         (16, 3, 8, 5, 5)]


@pytest.mark.parametrize("mode", ["on", "auto"])
@pytest.mark.parametrize("shape", F4_SK, ids=[str(s) for s in F4_SK])
def test_f4_stream_k(wino, shape, mode):
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("f4sk", N, C, K, H, W), kind="uniform", seed_x=61, seed_w=62)
    u4 = wino.filter_transform_f4(w.to(DEV))
    ws = torch.empty(wino.f4_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
    y = wino.conv2d_f4(x.to(DEV), u4, ws=ws, stream_k=mode)
    torch.cuda.synchronize()
    yd = y.cpu().double().numpy()
    assert np.isfinite(yd).all()
    assert oracle.max_rel_err(yd, oracle.direct_conv(x, w)) <= F4_TOL
    y2 = wino.conv2d_f4(x.to(DEV), u4, ws=ws, stream_k=mode)
    torch.cuda.synchronize()
    assert torch.equal(y.cpu(), y2.cpu())  # deterministic
