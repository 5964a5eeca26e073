"""Pins for the oracle (CPU only).  Each test ties the oracle to something other
than itself: the paper's printed text and numbers, a mathematical identity, a
library routine (torch.conv2d fp64), brute force, or an invariant.

PAPER.md citations: Eq. 1-3, Eq. 4, Eq. 5-8,
op counts L115, workspace L993, odd sizes L1155, implicit padding L335.
"""
import json
import os
import random
from fractions import Fraction as Fr

import numpy as np
import pytest
import torch

import oracle
from oracle import exact
from synth_inputs import CONFIGS, make_inputs, sample_points

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _golden():
    with open(os.path.join(GOLDEN, "paper_constants.json")) as f:
        return json.load(f)


# --------------------------------------------------------------------------
# Eq. 2-3: the matrices, pinned to the paper's own (garbled) text
# --------------------------------------------------------------------------
def _render(m):
    def cell(v):
        if v == Fr(1, 2):
            return "12"
        if v == Fr(-1, 2):
            return "−12"
        if v < 0:
            return "−" + str(-v)
        return str(v)
    return "".join("".join(cell(v) for v in row) for row in m)


def test_matrices_render_to_paper_scrape():
    text = open(os.path.join(GOLDEN, "eq2_eq3_scrape.txt"), encoding="utf-8").read()
    squashed = "".join(text.split())
    at_part = squashed[squashed.index("AT=[") + 4: squashed.index("],(2)")]
    g_part = squashed[squashed.index("G=") + 2: squashed.index(",BT=")]
    bt_part = squashed[squashed.index(",BT=") + 4: squashed.index(".(3)")]
    assert _render(exact.AT) == at_part
    assert _render(exact.G) == g_part
    assert _render(exact.BT) == bt_part


def test_op_counts_match_paper():
    g = _golden()
    assert exact.count_itf_adds() == g["itf_float_additions"]["value"]
    assert exact.count_otf_adds() == g["otf_float_additions"]["value"]
    assert exact.count_ftf_instructions() == g["ftf_float_instructions"]["value"]
    # L83: 36 multiplications direct vs 16 element-wise for one 2x2 output tile
    assert 2 * 2 * 3 * 3 == g["direct_multiplications_per_tile"]["value"]
    assert len(exact.BT) * len(exact.BT) == g["winograd_multiplications_per_tile"]["value"]


# --------------------------------------------------------------------------
# Eq. 1: exact identity on rational tiles (correlation, no flip)
# --------------------------------------------------------------------------
def _rand_frac(rng):
    return Fr(rng.randint(-50, 50), rng.randint(1, 9))


def test_eq1_identity_exact_rational():
    rng = random.Random(2020)
    flipped_differs = 0
    for _ in range(400):
        d = [[_rand_frac(rng) for _ in range(4)] for _ in range(4)]
        g = [[_rand_frac(rng) for _ in range(3)] for _ in range(3)]
        assert exact.winograd_tile(d, g) == exact.correlate_tile(d, g)
        flipped_differs += exact.winograd_tile(d, g) != exact.convolve_tile_flipped(d, g)
    assert flipped_differs > 390  # Eq. 1 computes correlation, not flipped convolution


def test_c_tile_transforms_equal_exact():
    """The C oracle's Eq. 5/6/8 transforms equal the exact-rational ones (dyadic inputs
    are exact in fp64), so the C matrices are the pinned matrices."""
    rng = random.Random(5)
    for _ in range(200):
        g = [[Fr(rng.randint(-64, 64), 4) for _ in range(3)] for _ in range(3)]
        d = [[Fr(rng.randint(-64, 64), 2) for _ in range(4)] for _ in range(4)]
        m = [[Fr(rng.randint(-64, 64), 8) for _ in range(4)] for _ in range(4)]
        as_np = lambda a: np.array([[float(v) for v in r] for r in a])
        assert np.array_equal(oracle.ftf_tile(as_np(g)), as_np(exact.ftf(g)))
        assert np.array_equal(oracle.itf_tile(as_np(d)), as_np(exact.itf(d)))
        assert np.array_equal(oracle.otf_tile(as_np(m)), as_np(exact.otf(m)))


# --------------------------------------------------------------------------
# Eq. 4: the direct oracle vs a library routine and vs brute force
# --------------------------------------------------------------------------
def _torch_ref(x_chwn, w_crsk):
    x = torch.as_tensor(np.asarray(x_chwn, dtype=np.float64)).permute(3, 0, 1, 2)  # NCHW
    w = torch.as_tensor(np.asarray(w_crsk, dtype=np.float64)).permute(3, 0, 1, 2)  # KCRS
    y = torch.nn.functional.conv2d(x, w, padding=1)  # correlation, no flip
    return y.permute(1, 2, 3, 0).numpy()  # KHWN


@pytest.mark.parametrize("shape", [(1, 1, 1, 1, 1), (2, 3, 4, 5, 7), (3, 8, 5, 9, 9),
                                   (4, 16, 12, 14, 14), (1, 7, 3, 2, 13)])
def test_direct_vs_torch_conv2d_fp64(shape):
    N, C, K, H, W = shape
    rng = np.random.default_rng(sum(shape))
    x = rng.uniform(-1, 1, (C, H, W, N))
    w = rng.uniform(-1, 1, (C, 3, 3, K))
    y = oracle.direct_conv(x, w)
    ref = _torch_ref(x, w)
    assert np.max(np.abs(y - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))


def _brute(x, w):
    C, H, W, N = x.shape
    K = w.shape[3]
    y = np.zeros((K, H, W, N))
    for k in range(K):
        for i in range(H):
            for j in range(W):
                for n in range(N):
                    acc = 0.0
                    for c in range(C):
                        for r in range(3):
                            for s in range(3):
                                h, ww = i + r - 1, j + s - 1
                                if 0 <= h < H and 0 <= ww < W:
                                    acc += x[c, h, ww, n] * w[c, r, s, k]
                    y[k, i, j, n] = acc
    return y


@pytest.mark.parametrize("seed", range(6))
def test_direct_vs_bruteforce_tiny(seed):
    rng = np.random.default_rng(100 + seed)
    N, C, K = (int(v) for v in rng.integers(1, 4, 3))
    H, W = (int(v) for v in rng.integers(1, 7, 2))
    x = rng.integers(-5, 6, (C, H, W, N)).astype(np.float64)
    w = rng.integers(-5, 6, (C, 3, 3, K)).astype(np.float64)
    assert np.array_equal(oracle.direct_conv(x, w), _brute(x, w))


def test_direct_sample_bit_identical_to_full():
    cfg = CONFIGS["tiny"].with_batch(3)
    x, w = make_inputs(cfg)
    y = oracle.direct_conv(x, w)
    idx = sample_points(cfg.K, cfg.H, cfg.W, cfg.N, 200)
    s = oracle.direct_sample(x, w, idx)
    idx = idx.numpy()
    assert np.array_equal(s, y[idx[:, 0], idx[:, 1], idx[:, 2], idx[:, 3]])


# --------------------------------------------------------------------------
# Eq. 5-8: naive Winograd vs the definition
# --------------------------------------------------------------------------
SMALL_SHAPES = [(1, 8, 8, 8, 8), (2, 3, 5, 7, 7), (3, 5, 4, 1, 1), (2, 4, 3, 1, 6),
                (1, 9, 2, 5, 3), (4, 2, 6, 2, 2), (2, 16, 16, 13, 11)]


@pytest.mark.parametrize("shape", SMALL_SHAPES)
def test_winograd_equals_direct_small_int_exact(shape):
    """Closed-form exactness: on integers every intermediate is a
    small dyadic rational, so Winograd == direct bit for bit in fp64."""
    N, C, K, H, W = shape
    rng = np.random.default_rng(N * 1000 + C * 100 + K * 10 + H + W)
    x = rng.integers(-3, 4, (C, H, W, N)).astype(np.float64)
    w = rng.integers(-3, 4, (C, 3, 3, K)).astype(np.float64)
    assert np.array_equal(oracle.winograd_conv(x, w), oracle.direct_conv(x, w))


@pytest.mark.parametrize("name", ["conv5_x", "conv4_x", "conv3_x", "conv2_x"])
def test_winograd_equals_direct_small_int_resnet_shapes(name):
    """The four ResNet layers at reduced batch / channel count (C up to 512 for conv5)."""
    cfg = CONFIGS[name]
    n = 1 if name != "conv5_x" else 2
    c = cfg.C if name == "conv5_x" else min(cfg.C, 64)
    k = 4
    sub = type(cfg)(name, n, c, k, cfg.H, cfg.W)
    x, w = make_inputs(sub, kind="smallint")
    assert np.array_equal(oracle.winograd_conv(x, w), oracle.direct_conv(x, w))


@pytest.mark.parametrize("shape", SMALL_SHAPES)
def test_winograd_vs_direct_random_fp64(shape):
    N, C, K, H, W = shape
    rng = np.random.default_rng(7 + C)
    x = rng.uniform(-1, 1, (C, H, W, N))
    w = rng.uniform(-1, 1, (C, 3, 3, K))
    assert oracle.max_rel_err(oracle.winograd_conv(x, w), oracle.direct_conv(x, w)) <= 1e-12


def test_filter_transform_layout_matches_exact():
    """U (C,4,4,K) with element (r',s') of G g G^T at [c, r', s', k] (reading R6)."""
    rng = np.random.default_rng(3)
    C, K = 3, 5
    w = rng.integers(-3, 4, (C, 3, 3, K)).astype(np.float64)
    u = oracle.filter_transform(w)
    y, u2 = oracle.winograd_conv(rng.uniform(size=(C, 4, 4, 1)), w, return_u=True)
    assert np.array_equal(u, u2)
    for c in range(C):
        for k in range(K):
            g = [[Fr(int(w[c, r, s, k])) for s in range(3)] for r in range(3)]
            ref = exact.ftf(g)
            assert np.array_equal(u[c, :, :, k], np.array([[float(v) for v in row] for row in ref]))


def test_workspace_size_matches_paper():
    """L993: the transformed filter is 16KC floats = 0.25/1/4/16 MB for Conv2..Conv5."""
    g = _golden()["workspace_MB"]["value"]
    for name, mb in g.items():
        cfg = CONFIGS[name]
        u = oracle.filter_transform(np.zeros((cfg.C, 3, 3, cfg.K)))
        assert u.size * 4 == int(mb * 2 ** 20)


# --------------------------------------------------------------------------
# Invariants (padding, orientation, linearity, batch equivariance)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("fn", ["direct_conv", "winograd_conv"])
def test_center_tap_identity(fn):
    rng = np.random.default_rng(11)
    C, H, W, N = 4, 7, 6, 3
    # dyadic values: every Winograd intermediate is exact, so equality is exact
    x = rng.integers(-512, 513, (C, H, W, N)) / 64.0
    w = np.zeros((C, 3, 3, C))
    for c in range(C):
        w[c, 1, 1, c] = 1.0
    assert np.array_equal(getattr(oracle, fn)(x, w), x)


@pytest.mark.parametrize("fn", ["direct_conv", "winograd_conv"])
@pytest.mark.parametrize("tap", [(0, 0), (0, 2), (2, 0), (2, 2), (0, 1), (1, 0), (2, 1), (1, 2)])
def test_single_tap_shift_zero_fill(fn, tap):
    """A single tap at (r,s) gives y[i,j] = x[i+r-1, j+s-1] with zeros past every border (L335)."""
    r, s = tap
    rng = np.random.default_rng(r * 3 + s)
    C, H, W, N = 2, 5, 7, 2
    x = rng.integers(-9, 10, (C, H, W, N)).astype(np.float64)
    w = np.zeros((C, 3, 3, C))
    for c in range(C):
        w[c, r, s, c] = 1.0
    xp = np.zeros((C, H + 2, W + 2, N))
    xp[:, 1:-1, 1:-1, :] = x
    expect = xp[:, r:r + H, s:s + W, :]
    assert np.array_equal(getattr(oracle, fn)(x, w), expect)


def test_linearity_and_batch_permutation():
    rng = np.random.default_rng(21)
    C, K, H, W, N = 3, 4, 6, 5, 5
    x1, x2 = rng.uniform(-1, 1, (2, C, H, W, N))
    w = rng.uniform(-1, 1, (C, 3, 3, K))
    y1, y2 = oracle.winograd_conv(x1, w), oracle.winograd_conv(x2, w)
    y12 = oracle.winograd_conv(2.0 * x1 - 3.0 * x2, w)
    assert np.max(np.abs(y12 - (2 * y1 - 3 * y2))) < 1e-12
    perm = rng.permutation(N)
    assert np.array_equal(oracle.winograd_conv(x1[..., perm], w), y1[..., perm])


def test_odd_size_extra_outputs_discarded():
    """L1155: on odd H/W the last tile computes an extra row/column that is discarded;
    outputs must still equal the definition at every valid position."""
    rng = np.random.default_rng(31)
    for H, W in [(1, 1), (1, 2), (3, 3), (5, 4), (7, 7)]:
        x = rng.integers(-3, 4, (2, H, W, 2)).astype(np.float64)
        w = rng.integers(-3, 4, (2, 3, 3, 3)).astype(np.float64)
        y = oracle.winograd_conv(x, w)
        assert y.shape == (3, H, W, 2)
        assert np.array_equal(y, _brute(x, w))


def test_max_rel_err_metric():
    ref = np.array([1.0, -4.0, 2.0])
    assert oracle.max_rel_err(ref + np.array([0, 0.004, 0]), ref) == pytest.approx(1e-3)
    assert oracle.max_rel_err(np.zeros(3), np.zeros(3)) == 0.0
    assert oracle.max_rel_err(np.ones(3), np.zeros(3)) == float("inf")


# --------------------------------------------------------------------------
# NEXT row N1: F(4x4,3x3) oracle pins
# --------------------------------------------------------------------------
def test_f4_identity_exact_rational():
    rng = random.Random(44)
    for _ in range(60):
        d = [[_rand_frac(rng) for _ in range(6)] for _ in range(6)]
        g = [[_rand_frac(rng) for _ in range(3)] for _ in range(3)]
        assert exact.winograd_f4_tile(d, g) == exact.correlate_tile_f4(d, g)


def test_f4_c_tiles_match_exact():
    rng = random.Random(45)
    as_np = lambda a: np.array([[float(v) for v in r] for r in a])
    for _ in range(50):
        g = [[Fr(rng.randint(-9, 9)) for _ in range(3)] for _ in range(3)]
        d = [[Fr(rng.randint(-9, 9)) for _ in range(6)] for _ in range(6)]
        m = [[Fr(rng.randint(-9, 9)) for _ in range(6)] for _ in range(6)]
        u = exact.matmul(exact.matmul(exact.G4, g), exact.transpose(exact.G4))
        v = exact.matmul(exact.matmul(exact.BT4, d), exact.transpose(exact.BT4))
        o = exact.matmul(exact.matmul(exact.AT4, m), exact.transpose(exact.AT4))
        assert np.allclose(oracle.ftf4_tile(as_np(g)), as_np(u), rtol=0, atol=1e-13)
        assert np.array_equal(oracle.itf4_tile(as_np(d)), as_np(v))
        assert np.array_equal(oracle.otf4_tile(as_np(m)), as_np(o))


@pytest.mark.parametrize("shape", [(2, 3, 4, 7, 7), (1, 8, 5, 8, 8), (3, 5, 2, 1, 9), (2, 16, 8, 14, 13)])
def test_f4_winograd_vs_direct(shape):
    N, C, K, H, W = shape
    rng = np.random.default_rng(9 + C)
    x = rng.uniform(-1, 1, (C, H, W, N))
    w = rng.uniform(-1, 1, (C, 3, 3, K))
    assert oracle.max_rel_err(oracle.winograd_f4_conv(x, w), oracle.direct_conv(x, w)) <= 1e-12
