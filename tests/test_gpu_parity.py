"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle.

Bars (BASELINE.json north_star / SURVEY 8(c)):
* small-integer inputs: bit-exact vs the direct definition (Eq. 4) -- every FP32
  intermediate is a small dyadic rational;
* random inputs: max|y - y_ref| / max|y_ref| <= 1e-4 (FP32 kernel);
* transformed filter u vs oracle U: bit-exact on small integers, <= 1e-6 random.
The BASELINE configs at full size are compared element by element, in every plan
bench.py times, in tests/test_gpu_full_parity.py.
"""
import numpy as np
import pytest
import torch

import oracle
from synth_inputs import CONFIGS, Conv3x3Config, make_inputs

pytestmark = pytest.mark.gpu

FP32_TOL = 1e-4
FTF_TOL = 1e-6


@pytest.fixture(scope="module")
def wino():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanwc20_b200 as w
    w.lib()
    return w


DEV = "cuda:0"


def _run(wino, x, w, variant="fp32"):
    u = wino.filter_transform(w.to(DEV))
    y = wino.conv2d(x.to(DEV), u, variant=variant)
    torch.cuda.synchronize()
    return u.cpu(), y.cpu()


# Shapes spanning several k-blocks / nu-blocks / channel steps with ragged tails,
# odd and tiny planes, N%4 != 0 and K%4 != 0 (generic load paths), C%8 != 0.
EDGE = [
    (1, 1, 1, 1, 1), (1, 8, 8, 8, 8), (3, 7, 5, 5, 5), (2, 9, 65, 7, 7), (33, 8, 64, 3, 3),
    (4, 20, 70, 13, 9), (5, 17, 130, 6, 10), (64, 16, 128, 2, 2), (1, 3, 3, 1, 17),
    (6, 12, 3, 14, 1), (32, 24, 96, 4, 6), (2, 64, 64, 16, 16), (7, 40, 72, 11, 12),
    # persistent warp-specialised FP32 path (N % 32 == 0, K % 4 == 0): C tails, K tails,
    # odd planes, more tiles than SMs
    (32, 7, 68, 5, 9), (64, 13, 132, 3, 7), (96, 1, 4, 9, 2), (32, 16, 64, 40, 40),
]


@pytest.mark.parametrize("shape", EDGE, ids=[str(s) for s in EDGE])
def test_edge_shapes_small_int_bit_exact(wino, shape):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("edge", N, C, K, H, W)
    x, w = make_inputs(cfg, kind="smallint")
    u, y = _run(wino, x, w)
    assert np.array_equal(u.double().numpy(), oracle.filter_transform(w))
    assert np.array_equal(y.double().numpy(), oracle.direct_conv(x, w))


@pytest.mark.parametrize("shape", EDGE, ids=[str(s) for s in EDGE])
def test_edge_shapes_random(wino, shape):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("edge", N, C, K, H, W)
    x, w = make_inputs(cfg, kind="uniform", seed_x=11, seed_w=12)
    u, y = _run(wino, x, w)
    assert oracle.max_rel_err(u.double().numpy(), oracle.filter_transform(w)) <= FTF_TOL
    assert oracle.max_rel_err(y.double().numpy(), oracle.direct_conv(x, w)) <= FP32_TOL


def test_tiny_full_oracle_both_forms(wino):
    """Tiny config (the one the oracle runs in full): y vs direct AND vs naive Winograd."""
    cfg = CONFIGS["tiny"]
    x, w = make_inputs(cfg)
    _, y = _run(wino, x, w)
    yd = y.double().numpy()
    assert oracle.max_rel_err(yd, oracle.direct_conv(x, w)) <= FP32_TOL
    assert oracle.max_rel_err(yd, oracle.winograd_conv(x, w)) <= FP32_TOL


def test_deterministic_and_batch_shard_consistent(wino):
    """Same output on repeated runs, and conv of a contiguous batch shard equals the
    shard of the full output bit for bit when neither splits C (per-output arithmetic
    does not depend on which CTA, kernel variant or batch size computes it) -- the
    property batch-sharded dispatch relies on.  With the planner's split-C choice
    (which depends on the shard size) only the summation order over C changes:
    within the FP32 bound."""
    cfg = CONFIGS["conv3_x"].with_batch(16)
    x, w = make_inputs(cfg)
    u = wino.filter_transform(w.to(DEV))
    xd = x.to(DEV)
    y1 = wino.conv2d(xd, u, split_c=1)
    y2 = wino.conv2d(xd, u, split_c=1)
    torch.cuda.synchronize()
    assert torch.equal(y1, y2)
    for lo, hi in [(0, 8), (8, 16), (3, 10), (15, 16), (4, 8)]:
        xs = xd[..., lo:hi].contiguous()
        ys = wino.conv2d(xs, u, split_c=1)
        ya = wino.conv2d(xs, u)  # planner's choice (may split C)
        torch.cuda.synchronize()
        assert torch.equal(ys, y1[..., lo:hi])
        ref = y1[..., lo:hi].double()
        assert float((ya.double() - ref).abs().max() / ref.abs().max()) <= FP32_TOL


def test_host_entry_point_matches_device_path(wino):
    cfg = Conv3x3Config("host", 8, 24, 40, 10, 9)
    x, w = make_inputs(cfg)
    u, y = _run(wino, x, w)
    xh, wh = x.pin_memory(), w.pin_memory()
    yh = torch.empty((cfg.K, cfg.H, cfg.W, cfg.N), dtype=torch.float32).pin_memory()
    ws = torch.empty(wino.host_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8,
                     device=DEV)
    wino.conv2d_host(xh, wh, yh, ws)
    torch.cuda.synchronize()
    assert torch.equal(yh, y)


def test_host_multi_matches_device_path(wino):
    """The pipelined multi-layer host call (K slices, batch slices with 2-D copies) is
    bit-identical to the device path layer by layer."""
    cfgs = [Conv3x3Config("a", 4, 16, 256, 7, 7), Conv3x3Config("b", 256, 8, 64, 6, 5),
            Conv3x3Config("c", 3, 5, 130, 9, 4), Conv3x3Config("d", 2, 3, 7, 3, 3)]
    layers, refs = [], []
    for i, cfg in enumerate(cfgs):
        x, w = make_inputs(cfg, seed_x=40 + i, seed_w=50 + i)
        refs.append(_run(wino, x, w)[1])
        layers.append((x.pin_memory(), w.pin_memory(),
                       torch.full((cfg.K, cfg.H, cfg.W, cfg.N), float("nan")).pin_memory()))
    ws = torch.empty(wino.host_multi_workspace_bytes(layers), dtype=torch.uint8, device=DEV)
    wino.conv2d_host_multi(layers, ws)
    torch.cuda.synchronize()
    for (xh, wh, yh), ref in zip(layers, refs):
        assert torch.equal(yh, ref)


def test_k_slices_equal_full(wino):
    """Slicing K (the library's host pipeline does) cannot change any output bit."""
    cfg = Conv3x3Config("ks", 32, 24, 256, 10, 10)
    x, w = make_inputs(cfg)
    _, y = _run(wino, x, w)
    for k0, k1 in [(0, 64), (64, 256), (128, 192)]:
        _, ys = _run(wino, x, w[..., k0:k1].contiguous())
        assert torch.equal(ys, y[k0:k1])


def test_output_fully_overwritten(wino):
    cfg = Conv3x3Config("ow", 3, 5, 6, 7, 5)
    x, w = make_inputs(cfg)
    u = wino.filter_transform(w.to(DEV))
    out = torch.full((cfg.K, cfg.H, cfg.W, cfg.N), float("nan"), device=DEV)
    wino.conv2d(x.to(DEV), u, out=out)
    torch.cuda.synchronize()
    assert torch.isfinite(out).all()
    assert oracle.max_rel_err(out.cpu().double().numpy(), oracle.direct_conv(x, w)) <= FP32_TOL


def test_device_side_errors(wino):
    base = torch.zeros(3 * 4 * 4 * 4 + 1, device=DEV)
    x_mis = base[1:].view(3, 4, 4, 4)  # contiguous but 4-byte aligned only
    u = torch.zeros(3, 4, 4, 5, device=DEV)
    with pytest.raises(wino.WinoError) as e:
        wino.conv2d(x_mis, u)
    assert e.value.status == 3  # WINO_ERR_MISALIGNED
    big = torch.zeros(16 * 3 * 5 + 5 * 4 * 4 * 4, device=DEV)
    u2 = big[:240].view(3, 4, 4, 5)
    y_alias = big[:320].view(5, 4, 4, 4)  # overlaps u2
    with pytest.raises(wino.WinoError) as e:
        wino.conv2d(torch.zeros(3, 4, 4, 4, device=DEV), u2, out=y_alias)
    assert e.value.status == 1  # WINO_ERR_INVALID_ARG (aliasing)


# ---------------------------------------------------------------------------
# tcgen05 variant (a5'): TF32 <= 5e-3, 3xTF32 <= 1e-4 (BASELINE / SURVEY 8(c))
# ---------------------------------------------------------------------------
TC_TOL = {"tf32": 5e-3, "3xtf32": 1e-4}


def _run_tc(wino, x, w, variant):
    u = wino.filter_transform_tc(w.to(DEV), variant)
    y = wino.conv2d_tc(x.to(DEV), u)
    torch.cuda.synchronize()
    return y.cpu()


@pytest.mark.parametrize("variant", ["tf32", "3xtf32"])
@pytest.mark.parametrize("shape", EDGE, ids=[str(s) for s in EDGE])
def test_tc_edge_shapes_random(wino, shape, variant):
    N, C, K, H, W = shape
    cfg = Conv3x3Config("edge", N, C, K, H, W)
    x, w = make_inputs(cfg, kind="uniform", seed_x=11, seed_w=12)
    y = _run_tc(wino, x, w, variant)
    assert oracle.max_rel_err(y.double().numpy(), oracle.direct_conv(x, w)) <= TC_TOL[variant]


@pytest.mark.parametrize("variant", ["tf32", "3xtf32"])
@pytest.mark.parametrize("shape", EDGE[:8], ids=[str(s) for s in EDGE[:8]])
def test_tc_edge_shapes_small_int(wino, shape, variant):
    """Small integers are exact in TF32 (|V| <= 12, 4|U| <= 27), so the tensor-core
    path must reproduce the definition exactly if it accumulates in >= FP32."""
    N, C, K, H, W = shape
    cfg = Conv3x3Config("edge", N, C, K, H, W)
    x, w = make_inputs(cfg, kind="smallint")
    y = _run_tc(wino, x, w, variant)
    assert np.array_equal(y.double().numpy(), oracle.direct_conv(x, w))


def test_filter_transform_multi_matches_single(wino):
    """One launch for several layers' FTFs (wino_filter_transform_multi) = the per-layer FTF, bit for bit."""
    pairs, singles = [], []
    for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x", "tiny"):
        _, w = make_inputs(CONFIGS[name])
        wd = w.to(DEV)
        pairs.append((wd, torch.empty((w.shape[0], 4, 4, w.shape[3]), device=DEV)))
        singles.append(wino.filter_transform(wd))
    wino.filter_transform_multi(pairs)
    torch.cuda.synchronize()
    for (_, u), u1 in zip(pairs, singles):
        assert torch.equal(u, u1)
    bad_u = pairs[0][0].reshape(-1)[: pairs[1][1].numel()].view(pairs[1][1].shape)  # aliases job 0's w
    with pytest.raises(wino.WinoError, match="INVALID_ARG"):  # an output overlapping another job's input
        wino.filter_transform_multi([pairs[0], (pairs[1][0], bad_u)])
