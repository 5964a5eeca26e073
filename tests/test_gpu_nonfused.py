"""GPU parity of NEXT row N3 -- the NON-fused Winograd path (Sec. 9; Sec. 7.3
obs. 4-6): u arrangement + ITF kernel -> V workspace, 16 batched GEMMs on the library's
own tcgen05 kernel (3xTF32: FP32-level accuracy; the _tf32 entry: plain TF32), OTF kernel,
through wino_conv2d_f2x3_fwd_nonfused, against the fp64 oracle.

Bars as tests/test_gpu_parity.py: bit-exact vs Eq. 4 on small integers (every
intermediate is an exact dyadic rational below 2^24), <= 1e-4 of max|y| on random
inputs.  Also checked against the oracle's naive Winograd (Eq. 5-8), whose steps the
non-fused path mirrors one launch each.
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


def _run(wino, x, w):
    C, H, W, N = x.shape
    K = w.shape[3]
    u = wino.filter_transform(w.to(DEV))
    ws = torch.empty(wino.nonfused_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
    y = wino.conv2d_nonfused(x.to(DEV), u, ws)
    torch.cuda.synchronize()
    return y.cpu()


SHAPES = [
    (1, 1, 1, 1, 1), (1, 8, 8, 8, 8), (3, 7, 5, 5, 5), (2, 9, 65, 7, 7), (33, 8, 64, 3, 3),
    (4, 20, 70, 13, 9), (5, 17, 130, 6, 10), (32, 24, 96, 4, 6), (7, 40, 72, 11, 12),
    # GEMM tiling: several 128-nu tiles + tail, several 32-channel stages + C % 4 tail, UMMA N = 16
    # (K <= 16), N = 256 tiles with a K tail (K > 256), C = 1
    (16, 67, 12, 17, 15), (8, 33, 300, 9, 9), (64, 1, 520, 4, 4), (2, 130, 16, 12, 12),
]


@pytest.mark.parametrize("shape", SHAPES, ids=[str(s) for s in SHAPES])
def test_nonfused_tf32_small_int_bit_exact(wino, shape):
    """Small integers are exact in TF32 (|V| <= 12, 4|U| <= 27): the TF32 GEMMs give Eq. 4 bit for bit."""
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("nf", N, C, K, H, W), kind="smallint")
    u = wino.filter_transform(w.to(DEV))
    ws = torch.empty(wino.nonfused_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
    y = wino.conv2d_nonfused(x.to(DEV), u, ws, tf32=True)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().double().numpy(), oracle.direct_conv(x, w))


@pytest.mark.parametrize("shape", SHAPES, ids=[str(s) for s in SHAPES])
def test_nonfused_small_int_bit_exact(wino, shape):
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("nf", N, C, K, H, W), kind="smallint")
    y = _run(wino, x, w)
    assert np.array_equal(y.double().numpy(), oracle.direct_conv(x, w))


@pytest.mark.parametrize("shape", SHAPES, ids=[str(s) for s in SHAPES])
def test_nonfused_random(wino, shape):
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("nf", N, C, K, H, W), kind="uniform", seed_x=51, seed_w=52)
    y = _run(wino, x, w).double().numpy()
    assert oracle.max_rel_err(y, oracle.direct_conv(x, w)) <= FP32_TOL
    assert oracle.max_rel_err(y, oracle.winograd_conv(x, w)) <= FP32_TOL


def test_nonfused_workspace_checks(wino):
    cfg = Conv3x3Config("nf", 4, 8, 8, 6, 6)
    x, w = make_inputs(cfg)
    u = wino.filter_transform(w.to(DEV))
    need = wino.nonfused_workspace_bytes(4, 8, 6, 6, 8)
    small = torch.empty(need - 256, dtype=torch.uint8, device=DEV)
    with pytest.raises(wino.WinoError) as e:
        wino.conv2d_nonfused(x.to(DEV), u, small)
    assert e.value.status == 1


@pytest.mark.parametrize("shape", [(32, 64, 64, 14, 14), (5, 17, 130, 6, 10), (32, 512, 512, 7, 7)],
                         ids=["conv2like", "ragged", "conv5"])
def test_nonfused_tf32_tensor_core_gemms(wino, shape):
    """N3 with plain TF32 tcgen05 GEMMs: within the TF32 bar of Eq. 4."""
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("nf", N, C, K, H, W), kind="uniform", seed_x=71, seed_w=72)
    u = wino.filter_transform(w.to(DEV))
    ws = torch.empty(wino.nonfused_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
    y = wino.conv2d_nonfused(x.to(DEV), u, ws, tf32=True)
    torch.cuda.synchronize()
    assert oracle.max_rel_err(y.cpu().double().numpy(), oracle.direct_conv(x, w)) <= 5e-3
