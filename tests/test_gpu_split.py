"""GPU parity of the small-batch paths of the FP32 kernel: multi-box TMA input
loads for N in {4, 8, 16} and split-C over thread-block clusters with the
partial outputs reduced through distributed shared memory (wino.h
wino_conv2d_f2x3_fwd_split).  These are the launch
configurations a rank runs under batch sharding.

Bars as tests/test_gpu_parity.py: bit-exact vs Eq. 4 on small integers (every
FP32 partial and their sum are exact dyadic rationals, so the split order
cannot change a bit), <= 1e-4 of max|y| on random inputs.
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ppopp_yanwc20_b200.dist import shard_range
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


# (N, C, K, H, W): N | 32 boxes, C tails (C % 8), K tails (K % 64), odd and tiny
# planes, tile runs that wrap image rows and run past the last tile
SMALL_N = [
    (4, 16, 64, 7, 7), (8, 24, 68, 5, 9), (16, 40, 128, 3, 3), (4, 64, 4, 1, 1),
    (16, 17, 132, 14, 14), (8, 72, 64, 2, 11), (4, 8, 8, 8, 8), (32, 48, 64, 6, 5),
]


@pytest.mark.parametrize("split", [0, 1, 2, 4, 8])
@pytest.mark.parametrize("shape", SMALL_N, ids=[str(s) for s in SMALL_N])
def test_small_n_split_small_int_bit_exact(wino, shape, split):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("split", N, C, K, H, W)
    x, w = make_inputs(cfg, kind="smallint")
    u = wino.filter_transform(w.to(DEV))
    y = wino.conv2d(x.to(DEV), u, split_c=split)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().double().numpy(), oracle.direct_conv(x, w))


@pytest.mark.parametrize("split", [1, 2, 8])
@pytest.mark.parametrize("shape", SMALL_N, ids=[str(s) for s in SMALL_N])
def test_small_n_split_random(wino, shape, split):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("split", N, C, K, H, W)
    x, w = make_inputs(cfg, kind="uniform", seed_x=21, seed_w=22)
    u = wino.filter_transform(w.to(DEV))
    y = wino.conv2d(x.to(DEV), u, split_c=split)
    torch.cuda.synchronize()
    assert oracle.max_rel_err(y.cpu().double().numpy(), oracle.direct_conv(x, w)) <= FP32_TOL


def test_split_deterministic_and_consistent(wino):
    """Repeated split runs are bit-identical; on small integers every split factor
    gives the same bits."""
    cfg = Conv3x3Config("det", 8, 128, 128, 14, 14)
    x, w = make_inputs(cfg, kind="uniform")
    u = wino.filter_transform(w.to(DEV))
    xd = x.to(DEV)
    for s in (2, 4, 8):
        a = wino.conv2d(xd, u, split_c=s)
        b = wino.conv2d(xd, u, split_c=s)
        torch.cuda.synchronize()
        assert torch.equal(a, b), s
    xi, wi = make_inputs(cfg, kind="smallint")
    ui = wino.filter_transform(wi.to(DEV))
    ys = [wino.conv2d(xi.to(DEV), ui, split_c=s) for s in (1, 2, 4, 8)]
    torch.cuda.synchronize()
    for y in ys[1:]:
        assert torch.equal(y, ys[0])


@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("name", ["conv5_x", "conv4_x", "conv3_x", "conv2_x"])
@pytest.mark.parametrize("kind", ["smallint", "uniform"])
def test_rank_shards(wino, name, P, kind):
    """The first and last rank's batch shard of every BASELINE layer at P = 2, 4, 8,
    in the launch configuration the planner picks (what bench.py --gpus P runs per
    rank), against Eq. 4, every output element."""
    cfg = CONFIGS[name]
    x, w = make_inputs(cfg, kind=kind)
    u = wino.filter_transform(w.to(DEV))
    for r in (0, P - 1):
        lo, hi = shard_range(cfg.N, r, P)
        xs = x[..., lo:hi].contiguous()
        y = wino.conv2d(xs.to(DEV), u)
        torch.cuda.synchronize()
        ref = oracle.direct_conv(xs, w)  # the whole shard output
        got = y.cpu().double().numpy()
        if kind == "smallint":
            assert np.array_equal(got, ref), (name, P, r)
        else:
            assert np.isfinite(got).all()
            assert oracle.max_rel_err(got, ref) <= FP32_TOL, (name, P, r)


# ---------------------------------------------------------------------------
# tcgen05 variant (a5') on the same small-batch shapes: N in {4, 8, 16} load 32/N
# TMA boxes per nu-half (XM = 3).  TF32 <= 5e-3, 3xTF32 <= 1e-4; small integers
# are exact in TF32 (tests/test_gpu_parity.py).
# ---------------------------------------------------------------------------
TC_TOL = {"tf32": 5e-3, "3xtf32": 1e-4}


@pytest.mark.parametrize("variant", ["tf32", "3xtf32"])
@pytest.mark.parametrize("shape", SMALL_N, ids=[str(s) for s in SMALL_N])
def test_tc_small_n(wino, shape, variant):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("tcsplit", N, C, K, H, W)
    for kind in ("smallint", "uniform"):
        x, w = make_inputs(cfg, kind=kind, seed_x=41, seed_w=42)
        u = wino.filter_transform_tc(w.to(DEV), variant)
        y = wino.conv2d_tc(x.to(DEV), u)
        torch.cuda.synchronize()
        ref = oracle.direct_conv(x, w)
        if kind == "smallint":
            assert np.array_equal(y.cpu().double().numpy(), ref)
        else:
            assert oracle.max_rel_err(y.cpu().double().numpy(), ref) <= TC_TOL[variant]


@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("name", ["conv5_x", "conv4_x", "conv3_x", "conv2_x"])
def test_tc_rank_shards(wino, name, P):
    cfg = CONFIGS[name]
    x, w = make_inputs(cfg, kind="uniform")
    for variant in ("tf32", "3xtf32"):
        u = wino.filter_transform_tc(w.to(DEV), variant)
        lo, hi = shard_range(cfg.N, P - 1, P)
        xs = x[..., lo:hi].contiguous()
        y = wino.conv2d_tc(xs.to(DEV), u)
        torch.cuda.synchronize()
        got = y.cpu().double().numpy()
        assert oracle.max_rel_err(got, oracle.direct_conv(xs, w)) <= TC_TOL[variant], (name, P, variant)
