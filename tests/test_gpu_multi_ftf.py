"""Filter transform + convolutions of several layers in one call (wino_conv2d_f2x3_fwd_multi_ftf):
when every layer joins one shared persistent launch, the FTFs (Eq. 5) and the vmode input transforms
(Eq. 6) run as a prologue of that launch, gated by a grid-wide count (cooperative launch).

Checked: u equals wino_filter_transform's output bit for bit (same ftf_4x4 arithmetic); y equals the
two-call form (filter_transform_multi + conv2d_multi) bit for bit -- the same kernel, plan and
summation order -- and the fp64 oracle element by element (bit-exact on small integers, <= 1e-4 of
max|y| on random inputs); the ResNet step at P = 1 and every P = 2 / 4 / 8 shard (x-box and vmode
layers), ragged groups, the non-fused fallback (a layer that runs alone, more than 4 layers), repeated
calls (the barrier words are reset by the kernel), argument errors."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ppopp_yanwc20_b200.dist import shard_range
from synth_inputs import CONFIGS, Conv3x3Config, make_inputs

pytestmark = pytest.mark.gpu
DEV = "cuda:0"
FP32_TOL = 1e-4
RESNET = [CONFIGS[n] for n in ("conv5_x", "conv4_x", "conv3_x", "conv2_x")]


@pytest.fixture(scope="module")
def wino():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanwc20_b200 as w
    w.lib()
    return w


def _run(wino, cfgs, kind, seed0=0, reps=1):
    data, fused, plain = [], [], []
    for i, cfg in enumerate(cfgs):
        x, w = make_inputs(cfg, kind=kind, seed_x=1234 + seed0 + i, seed_w=1235 + seed0 + i)
        xd, wd = x.to(DEV), w.to(DEV)
        nan = float("nan")
        fused.append((xd, wd, torch.full((cfg.C, 4, 4, cfg.K), nan, device=DEV),
                      torch.full((cfg.K, cfg.H, cfg.W, cfg.N), nan, device=DEV)))
        plain.append((xd, wino.filter_transform(wd), torch.full((cfg.K, cfg.H, cfg.W, cfg.N), nan, device=DEV)))
        data.append((x, w))
    shapes = [(c.N, c.C, c.H, c.W, c.K) for c in cfgs]
    ws = torch.zeros(wino.conv_multi_workspace_bytes(shapes), dtype=torch.uint8, device=DEV)
    ws2 = torch.zeros_like(ws)
    ys = []
    for _ in range(reps):
        wino.conv2d_multi_ftf(fused, ws)
        torch.cuda.synchronize()
        ys.append([y.cpu().double().numpy() for (_, _, _, y) in fused])
    wino.conv2d_multi(plain, ws2)
    torch.cuda.synchronize()
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    slot = 64 * 4 * 32 * 4
    counters = ws[2 * sms * slot: 2 * sms * slot + 4 * sms + 8]
    assert int(counters.count_nonzero()) == 0, "arrival counters / barrier words not left zero"
    for (_, _, u, y), (_, u2, y2) in zip(fused, plain):
        assert torch.equal(u, u2), "u differs from wino_filter_transform"
        assert torch.equal(y, y2), "y differs from the two-call form"
    return data, ys


def _check(data, ys, kind):
    for (x, w), y in zip(data, ys):
        ref = oracle.direct_conv(x, w)
        if kind == "smallint":
            assert np.array_equal(y, ref), int((y != ref).sum())
        else:
            assert np.isfinite(y).all()
            assert oracle.max_rel_err(y, ref) <= FP32_TOL


@pytest.mark.parametrize("kind", ["smallint", "uniform"])
@pytest.mark.parametrize("P", [1, 2, 4, 8])
def test_resnet_step_and_shards(wino, P, kind):
    cfgs = [c.with_batch(shard_range(c.N, P - 1, P)[1] - shard_range(c.N, P - 1, P)[0]) for c in RESNET]
    assert wino.conv_multi_ftf_launches([(c.N, c.C, c.H, c.W, c.K) for c in cfgs]) == 1
    data, ys = _run(wino, cfgs, kind, seed0=10 * P)
    _check(data, ys[0], kind)


GROUPS = [
    [Conv3x3Config("a", 32, 7, 68, 5, 9), Conv3x3Config("b", 8, 13, 132, 3, 7), Conv3x3Config("c", 4, 1, 4, 9, 2)],
    [Conv3x3Config("s", 16, 24, 40, 7, 9), Conv3x3Config("m", 32, 512, 512, 7, 7), Conv3x3Config("n", 4, 40, 72, 7, 7),
     Conv3x3Config("o", 96, 16, 64, 6, 5)],
    # not fusable: a layer with >= 64 tiles per SM runs alone; N = 3 is not warp-specialised eligible
    [Conv3x3Config("t", 32, 8, 8, 2, 2), Conv3x3Config("big", 512, 8, 8, 56, 56)],
    [Conv3x3Config("f1", 3, 9, 20, 6, 6), Conv3x3Config("f2", 32, 16, 36, 5, 5)],
    # more than 4 layers: two launches + one FTF launch
    [Conv3x3Config(f"l{i}", 8, 16, 24, 5, 7) for i in range(5)],
]


@pytest.mark.parametrize("kind", ["smallint", "uniform"])
@pytest.mark.parametrize("g", range(len(GROUPS)), ids=["tails", "four-mixed", "alone", "n3", "five"])
def test_groups(wino, g, kind):
    data, ys = _run(wino, GROUPS[g], kind, seed0=100 + g)
    _check(data, ys[0], kind)
    fused = wino.conv_multi_ftf_launches([(c.N, c.C, c.H, c.W, c.K) for c in GROUPS[g]]) == 1
    assert fused == (g < 2)


def test_repeated_calls_deterministic(wino):
    cfgs = [c.with_batch(c.N // 8) for c in RESNET]
    data, ys = _run(wino, cfgs, "uniform", seed0=300, reps=4)
    for a, b in zip(ys[0], ys[3]):
        assert np.array_equal(a, b)
    _check(data, ys[0], "uniform")


def test_argument_errors(wino):
    cfg = Conv3x3Config("e", 32, 8, 16, 4, 4)
    x = torch.zeros((cfg.C, cfg.H, cfg.W, cfg.N), device=DEV)
    w = torch.zeros((cfg.C, 3, 3, cfg.K), device=DEV)
    u = torch.zeros((cfg.C, 4, 4, cfg.K), device=DEV)
    y = torch.zeros((cfg.K, cfg.H, cfg.W, cfg.N), device=DEV)
    ws = torch.zeros(wino.conv_multi_workspace_bytes([(cfg.N, cfg.C, cfg.H, cfg.W, cfg.K)]), dtype=torch.uint8,
                     device=DEV)
    buf = torch.zeros(25 * cfg.C * cfg.K, device=DEV)  # w and an overlapping u in one allocation
    with pytest.raises(wino.WinoError):  # u (an output) aliasing w
        wino.conv2d_multi_ftf([(x, buf[: w.numel()].view(w.shape), buf[4 * cfg.C * cfg.K: 20 * cfg.C * cfg.K].view(u.shape),
                                y)], ws)
    with pytest.raises(wino.WinoError):  # u aliasing x
        wino.conv2d_multi_ftf([(x, w, x.view(-1)[: u.numel()].view(u.shape), y)], ws)
    with pytest.raises(wino.WinoError):  # workspace too small
        wino.conv2d_multi_ftf([(x, w, u, y)], ws[:64])
    with pytest.raises((wino.WinoError, ValueError)):  # misaligned w
        wb = torch.zeros(w.numel() + 1, device=DEV)[1:].view(w.shape)
        wino.conv2d_multi_ftf([(x, wb, u, y)], ws)
    wino.conv2d_multi_ftf([(x, w, u, y)], ws)
    torch.cuda.synchronize()
