"""Several independent layers through wino_conv2d_f2x3_fwd_multi (shared persistent stream-K launch,
csrc/fused_fp32_ml.cuh; layers with >= 64 tiles per SM run alone through the planner) against the
fp64 oracle, every output element of every layer.

Bars as tests/test_gpu_parity.py: bit-exact vs Eq. 4 on small integers, <= 1e-4 of max|y| on
random inputs (per layer).  Covered: the four BASELINE ResNet layers at their global batch and
every rank's shard at P = 2 / 4 / 8 (mixed x-box modes: N % 32 == 0 and N in {4, 8, 16} in one
launch), ragged shapes (C, K, H, W tails, one tile, tiny layers next to big ones), more than 4
layers (two launches), a group falling back to per-layer launches (N = 3), determinism, the
arrival counters left zero, argument errors."""
import ctypes

import numpy as np
import pytest
import torch

import oracle
from paper_conf_ppopp_yanwc20_b200.dist import shard_range
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


def _run_multi(wino, cfgs, kind, seed0=0, reps=1):
    data, layers = [], []
    for i, cfg in enumerate(cfgs):
        x, w = make_inputs(cfg, kind=kind, seed_x=1234 + seed0 + i, seed_w=1235 + seed0 + i)
        xd, wd = x.to(DEV), w.to(DEV)
        u = wino.filter_transform(wd)
        y = torch.full((cfg.K, cfg.H, cfg.W, cfg.N), float("nan"), device=DEV)
        data.append((x, w))
        layers.append((xd, u, y))
    ws = torch.zeros(wino.conv_multi_workspace_bytes([(c.N, c.C, c.H, c.W, c.K) for c in cfgs]),
                     dtype=torch.uint8, device=DEV)
    outs = []
    for _ in range(reps):
        wino.conv2d_multi(layers, ws)
        torch.cuda.synchronize()
        outs.append([y.cpu().double().numpy() for _, _, y in layers])
    return data, outs, ws


def _check(data, ys, kind):
    for (x, w), y in zip(data, ys):
        ref = oracle.direct_conv(x, w)
        if kind == "smallint":
            assert np.array_equal(y, ref), int((y != ref).sum())
        else:
            assert np.isfinite(y).all()
            assert oracle.max_rel_err(y, ref) <= FP32_TOL


RESNET = [CONFIGS[n] for n in ("conv5_x", "conv4_x", "conv3_x", "conv2_x")]


@pytest.mark.parametrize("kind", ["smallint", "uniform"])
@pytest.mark.parametrize("P", [1, 2, 4, 8])
def test_resnet_step_and_shards(wino, P, kind):
    for r in sorted({0, P - 1}):
        cfgs = [c.with_batch(shard_range(c.N, r, P)[1] - shard_range(c.N, r, P)[0]) for c in RESNET]
        data, outs, ws = _run_multi(wino, cfgs, kind, seed0=10 * r)
        _check(data, outs[0], kind)


RAGGED = [
    [Conv3x3Config("a", 32, 7, 68, 5, 9), Conv3x3Config("b", 8, 13, 132, 3, 7), Conv3x3Config("c", 4, 1, 4, 9, 2)],
    [Conv3x3Config("t", 32, 8, 8, 2, 2), Conv3x3Config("big", 64, 64, 64, 40, 40)],
    [Conv3x3Config("s", 16, 24, 40, 7, 9), Conv3x3Config("m", 32, 512, 512, 7, 7), Conv3x3Config("n", 4, 40, 72, 7, 7),
     Conv3x3Config("o", 96, 16, 64, 6, 5)],
]


@pytest.mark.parametrize("kind", ["smallint", "uniform"])
@pytest.mark.parametrize("group", range(len(RAGGED)), ids=["tails", "tiny+big", "four-mixed"])
def test_ragged_groups(wino, group, kind):
    data, outs, _ = _run_multi(wino, RAGGED[group], kind, seed0=100 + group)
    _check(data, outs[0], kind)


def test_more_than_four_layers_and_fallback(wino):
    """6 layers = a launch of 4 + a group of 2; the second group holds N = 3 (not warp-specialised
    eligible), so it runs layer by layer through the planner."""
    cfgs = RAGGED[2] + [Conv3x3Config("f1", 3, 9, 20, 6, 6), Conv3x3Config("f2", 32, 16, 36, 5, 5)]
    data, outs, _ = _run_multi(wino, cfgs, "smallint", seed0=200)
    _check(data, outs[0], "smallint")


def test_deterministic_and_counters_zero(wino):
    cfgs = [c.with_batch(c.N // 8) for c in RESNET]
    data, outs, ws = _run_multi(wino, cfgs, "uniform", seed0=300, reps=3)
    for a, b in zip(outs[0], outs[2]):
        assert np.array_equal(a, b)
    _check(data, outs[0], "uniform")
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    slot = 64 * 4 * 32 * 4
    assert int(ws[2 * sms * slot: 2 * sms * slot + 4 * sms].count_nonzero()) == 0
    # the dynamic tail's grab / done counters (2 words after the arrival counters) are reset too
    assert int(ws[2 * sms * slot + 4 * sms: 2 * sms * slot + 4 * sms + 8].count_nonzero()) == 0


def test_matches_single_layer_calls(wino):
    """The same layers through wino_conv2d_f2x3_fwd_ws one by one: equal within the FP32 bar
    (only the summation order of cut tiles can differ)."""
    cfgs = [c.with_batch(c.N // 4) for c in RESNET]
    data, outs, _ = _run_multi(wino, cfgs, "uniform", seed0=400)
    for (x, w), ym, cfg in zip(data, outs[0], cfgs):
        u = wino.filter_transform(w.to(DEV))
        ws = torch.zeros(wino.conv_workspace_bytes(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K), dtype=torch.uint8, device=DEV)
        ys = wino.conv2d(x.to(DEV), u, ws=ws).cpu().double().numpy()
        assert float(np.max(np.abs(ys - ym)) / np.max(np.abs(ys))) <= FP32_TOL


def test_argument_errors(wino):
    cfg = Conv3x3Config("e", 32, 8, 16, 4, 4)
    x = torch.zeros((cfg.C, cfg.H, cfg.W, cfg.N), device=DEV)
    u = torch.zeros((cfg.C, 4, 4, cfg.K), device=DEV)
    y = torch.empty((cfg.K, cfg.H, cfg.W, cfg.N), device=DEV)
    y2 = torch.empty((cfg.K, cfg.H, cfg.W, cfg.N), device=DEV)
    ws = torch.zeros(wino.conv_multi_workspace_bytes([(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K)]), dtype=torch.uint8,
                     device=DEV)
    with pytest.raises(wino.WinoError, match="INVALID_ARG"):  # two jobs writing the same y
        wino.conv2d_multi([(x, u, y), (x, u, y)], ws)
    with pytest.raises(wino.WinoError, match="INVALID_ARG"):  # short workspace
        wino.conv2d_multi([(x, u, y)], ws[:1024])
    with pytest.raises(wino.WinoError, match="INVALID_ARG"):  # y of one job is another job's x
        wino.conv2d_multi([(x, u, y), (y[:cfg.C], u, y2)], ws)
    L = wino.lib()
    assert L.wino_conv2d_f2x3_fwd_multi(None, 1, ctypes.c_void_p(ws.data_ptr()), ws.numel(), None, None) == 1
    wino.conv2d_multi([(x, u, y), (x, u, y2)], ws)  # shared inputs are fine
    torch.cuda.synchronize()


def test_u_ready_event_orders_the_convolutions(wino):
    """FTF on a side stream, convolutions on the main stream ordered only by the u_ready event
    (the N = 4 / 8 input transforms are queued before the wait): every element as the oracle."""
    cfgs = [c.with_batch(c.N // 8) for c in RESNET]  # N = 4, 8, 16, 32: two vmode layers
    main, side = torch.cuda.current_stream(), torch.cuda.Stream()
    data, layers, ws_list = [], [], []
    for i, cfg in enumerate(cfgs):
        x, w = make_inputs(cfg, kind="smallint", seed_x=500 + i, seed_w=600 + i)
        data.append((x, w))
        layers.append((x.to(DEV), torch.full((cfg.C, 4, 4, cfg.K), float("nan"), device=DEV),
                       torch.full((cfg.K, cfg.H, cfg.W, cfg.N), float("nan"), device=DEV), w.to(DEV)))
    ws = torch.zeros(wino.conv_multi_workspace_bytes([(c.N, c.C, c.H, c.W, c.K) for c in cfgs]),
                     dtype=torch.uint8, device=DEV)
    torch.cuda.synchronize()
    side.wait_stream(main)
    wino.filter_transform_multi([(wd, u) for _, u, _, wd in layers], stream=side)
    ev = torch.cuda.Event()
    ev.record(side)
    wino.conv2d_multi([(x, u, y) for x, u, y, _ in layers], ws, u_ready=ev)
    torch.cuda.synchronize()
    _check(data, [y.cpu().double().numpy() for _, _, y, _ in layers], "smallint")


def test_big_layer_runs_alone_next_to_shared_ones(wino):
    """A layer with >= 64 tiles per SM (10240 tiles of 64 x 32 here) is launched alone through the
    planner in the same call as a shared group: both bit-exact on small integers."""
    big = Conv3x3Config("big", 32, 1, 640, 64, 64)
    cfgs = [Conv3x3Config("s1", 8, 40, 72, 7, 7), big, Conv3x3Config("s2", 32, 16, 36, 5, 5)]
    shapes = [(c.N, c.C, c.H, c.W, c.K) for c in cfgs]
    # the shared launch (+ its input transform for N = 8) and the planner's launch for the big layer
    assert wino.conv_multi_launches(shapes) == 2 + wino.plan(*shapes[1][:4], shapes[1][4], variant=4).launches
    data, outs, _ = _run_multi(wino, cfgs, "smallint", seed0=700)
    _check(data, outs[0], "smallint")
