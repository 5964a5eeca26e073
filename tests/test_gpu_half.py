"""GPU parity for NEXT row N4: FP16 / BF16 operands on tcgen05 kind::f16 vs the fp64 oracle.

The path stores x, w, y in a 16-bit type; transforms and accumulation run in FP32;
U, V and y are rounded to the 16-bit type (reading R18).  The oracle is the
definition (Eq. 4) evaluated in fp64 on the 16-bit input values.

Bars:
* small-integer inputs: every U, V, product and partial sum is exact (|V| <= 12, 4|U|
  <= 27 fit any 16-bit significand; FP32 sums stay < 2^24), so y equals the
  round-to-nearest-even of the exact integer result bit for bit, and u equals the
  oracle's U (exact in the 16-bit type);
* random inputs: max|y - y_ref| / max|y_ref| <= 5e-3 (fp16) / 3e-2 (bf16) -- about
  7x the error the rounding model of scripts/half_error_model.py predicts
  (7e-4 / 4.4e-3, dominated by the final rounding of y);
* u vs oracle U rounded to the 16-bit type: within one unit in the last place.
"""
import numpy as np
import pytest
import torch

import oracle
from synth_inputs import CONFIGS, Conv3x3Config, make_inputs

pytestmark = pytest.mark.gpu

DEV = "cuda:0"
TOL = {torch.float16: 5e-3, torch.bfloat16: 3e-2}
DTYPES = [torch.float16, torch.bfloat16]
IDS = ["fp16", "bf16"]


@pytest.fixture(scope="module")
def wino():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanwc20_b200 as w
    w.lib()
    return w


def _inputs(cfg, kind, dt, **kw):
    x, w = make_inputs(cfg, kind=kind, **kw)
    return x.to(dt), w.to(dt)  # the 16-bit inputs; the oracle sees exactly these values


def _run(wino, xh, wh):
    uh = wino.filter_transform_half(wh.to(DEV))
    y = wino.conv2d_half(xh.to(DEV), uh)
    torch.cuda.synchronize()
    return uh, y.cpu()


def _unpack_u(uh):
    """(C,4,4,K) from the documented operand layout [cb][kb][xi][m/8][c/8][m%8][c%8], MM = 64 rows
    per kb when K <= 64, else 128 (include/wino.h)."""
    C, K = uh.C, uh.K
    mm = 64 if K <= 64 else 128
    ncb, nkb = (C + 15) // 16, (K + mm - 1) // mm
    a = uh.data.cpu().float().reshape(ncb, nkb, 16, mm // 8, 2, 8, 8)
    # -> [cb][c/8][c%8][xi][kb][m/8][m%8]
    a = a.permute(0, 4, 6, 2, 1, 3, 5).reshape(ncb * 16, 16, nkb * mm)
    return a[:C, :, :K].reshape(C, 4, 4, K)


def _round(ref64, dt):
    """Round-to-nearest-even of exact fp64 values to dt (via fp32, exact for |v| < 2^24 integers)."""
    return torch.from_numpy(ref64).to(torch.float32).to(dt).float().numpy()


# (N, C, K, H, W): TMA path (N % 32 == 0), boxes per image tile (N in {8, 16}),
# generic gather (other N); C tails (C % 16), K tails (K % 128), odd / tiny planes,
# more tiles than SMs.
EDGE = [
    (1, 1, 1, 1, 1), (1, 8, 8, 8, 8), (3, 7, 5, 5, 5), (2, 17, 130, 6, 10), (4, 20, 70, 13, 9),
    (40, 16, 16, 6, 6), (32, 16, 128, 4, 4), (32, 7, 68, 5, 9), (64, 33, 132, 3, 7), (96, 1, 4, 9, 2),
    (32, 16, 64, 40, 40), (8, 24, 136, 7, 7), (16, 40, 72, 11, 12), (16, 3, 8, 1, 17),
    # 64-filter tiles (K <= 64) on every load path: TMA, per-tile boxes (N = 8), gather
    (64, 20, 64, 10, 10), (8, 5, 40, 9, 6), (4, 16, 64, 6, 6), (96, 33, 17, 3, 5),
    # N = 4 (batch shards): generic gather, odd and even W
    (4, 24, 136, 7, 10), (4, 9, 40, 5, 2),
]


@pytest.mark.parametrize("dt", DTYPES, ids=IDS)
@pytest.mark.parametrize("shape", EDGE, ids=[str(s) for s in EDGE])
def test_half_edge_small_int_bit_exact(wino, shape, dt):
    N, C, K, H, W = shape
    xh, wh = _inputs(Conv3x3Config("h", N, C, K, H, W), "smallint", dt)
    uh, y = _run(wino, xh, wh)
    assert np.array_equal(_unpack_u(uh).double().numpy(), oracle.filter_transform(wh.float()))
    ref = oracle.direct_conv(xh.float(), wh.float())
    assert np.array_equal(y.float().numpy(), _round(ref, dt))


@pytest.mark.parametrize("dt", DTYPES, ids=IDS)
@pytest.mark.parametrize("shape", EDGE, ids=[str(s) for s in EDGE])
def test_half_edge_random(wino, shape, dt):
    N, C, K, H, W = shape
    xh, wh = _inputs(Conv3x3Config("h", N, C, K, H, W), "uniform", dt, seed_x=21, seed_w=22)
    uh, y = _run(wino, xh, wh)
    u_ref = oracle.filter_transform(wh.float())
    u_got = _unpack_u(uh).double().numpy()
    fi = torch.finfo(dt)  # rounding to dt: |error| <= half an ulp <= eps/2 * |u| (+ subnormal spacing)
    assert np.all(np.abs(u_got - u_ref) <= np.abs(u_ref) * fi.eps + fi.tiny * fi.eps)
    yd = y.double().numpy()
    assert np.isfinite(yd).all()
    assert oracle.max_rel_err(yd, oracle.direct_conv(xh.float(), wh.float())) <= TOL[dt]


@pytest.mark.parametrize("dt", DTYPES, ids=IDS)
def test_half_matches_oracle_winograd(wino, dt):
    """Also within the bar of the oracle's step-by-step Winograd (Eq. 5-8), not only of Eq. 4."""
    xh, wh = _inputs(Conv3x3Config("h", 32, 24, 72, 13, 11), "uniform", dt)
    _, y = _run(wino, xh, wh)
    assert oracle.max_rel_err(y.double().numpy(), oracle.winograd_conv(xh.float(), wh.float())) <= TOL[dt]


@pytest.mark.parametrize("dt", DTYPES, ids=IDS)
def test_half_deterministic_and_batch_shard_consistent(wino, dt):
    """Repeated runs are identical, outputs are overwritten, and a contiguous batch shard
    (the unit of batch-sharded dispatch) gives the shard of the full output bit for bit:
    per-output arithmetic does not depend on N or on the load path (TMA / per-tile boxes /
    gather)."""
    xh, wh = _inputs(CONFIGS["conv3_x"].with_batch(64), "uniform", dt)
    xd = xh.to(DEV)
    uh = wino.filter_transform_half(wh.to(DEV))
    y1 = wino.conv2d_half(xd, uh)
    for _ in range(4):
        y2 = torch.full_like(y1, float("nan"))
        wino.conv2d_half(xd, uh, out=y2)
        torch.cuda.synchronize()
        assert torch.equal(y1, y2)
    for lo, hi in [(0, 32), (32, 64), (16, 32), (8, 16), (5, 9)]:
        ys = wino.conv2d_half(xd[..., lo:hi].contiguous(), uh)
        torch.cuda.synchronize()
        assert torch.equal(ys, y1[..., lo:hi])


def test_half_argument_errors(wino):
    x = torch.zeros((16, 4, 4, 32), dtype=torch.float16, device=DEV)
    wh = torch.zeros((16, 3, 3, 64), dtype=torch.float16, device=DEV)
    uh = wino.filter_transform_half(wh)
    with pytest.raises(TypeError):
        wino.conv2d_half(x.float(), uh)
    with pytest.raises(ValueError):
        wino.conv2d_half(x.to(torch.bfloat16), uh)  # filter built for fp16
    L = wino.lib()
    import ctypes
    p = ctypes.c_void_p
    st = L.wino_conv2d_f2x3_fwd_half(p(x.data_ptr()), p(uh.data.data_ptr()), p(x.data_ptr()), 32, 16, 4, 4, 64,
                                     1, 1, 0, None)
    assert st == 1  # y aliases x -> INVALID_ARG
    y = torch.empty((64, 4, 4, 32), dtype=torch.float16, device=DEV)
    st = L.wino_conv2d_f2x3_fwd_half(p(x.data_ptr()), p(uh.data.data_ptr()), p(y.data_ptr()), 32, 16, 4, 4, 64,
                                     1, 1, 7, None)
    assert st == 1  # unknown type
    st = L.wino_conv2d_f2x3_fwd_half(p(x.data_ptr()), p(uh.data.data_ptr()), p(y.data_ptr()), 32, 16, 4, 4, 64,
                                     0, 1, 0, None)
    assert st == 2  # pad != 1 -> UNSUPPORTED


def _run_ws(wino, xh, wh, mode):
    C, H, W, N = xh.shape
    K = wh.shape[3]
    uh = wino.filter_transform_half(wh.to(DEV))
    ws = torch.empty(wino.half_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
    y = wino.conv2d_half(xh.to(DEV), uh, ws=ws, stream_k=mode)
    torch.cuda.synchronize()
    return y.cpu()


# stream-K: ranges shorter than a tile (large C, few tiles), spanning several tiles, every load path
SK_EDGE = [(32, 512, 256, 5, 5), (4, 512, 512, 7, 7), (8, 256, 256, 14, 14), (16, 128, 128, 12, 10),
           (32, 64, 64, 30, 30), (64, 33, 132, 9, 7), (96, 40, 17, 11, 3)]


@pytest.mark.parametrize("dt", DTYPES, ids=IDS)
@pytest.mark.parametrize("shape", SK_EDGE, ids=[str(s) for s in SK_EDGE])
def test_half_stream_k_small_int_bit_exact(wino, shape, dt):
    N, C, K, H, W = shape
    xh, wh = _inputs(Conv3x3Config("h", N, C, K, H, W), "smallint", dt)
    y = _run_ws(wino, xh, wh, "on")
    assert np.array_equal(y.float().numpy(), _round(oracle.direct_conv(xh.float(), wh.float()), dt))


@pytest.mark.parametrize("dt", DTYPES, ids=IDS)
@pytest.mark.parametrize("shape", SK_EDGE[:4], ids=[str(s) for s in SK_EDGE[:4]])
def test_half_stream_k_random(wino, shape, dt):
    N, C, K, H, W = shape
    xh, wh = _inputs(Conv3x3Config("h", N, C, K, H, W), "uniform", dt, seed_x=51, seed_w=52)
    y = _run_ws(wino, xh, wh, "on")
    assert oracle.max_rel_err(y.double().numpy(), oracle.direct_conv(xh.float(), wh.float())) <= TOL[dt]


@pytest.mark.parametrize("P", [1, 2, 4, 8])
def test_half_stream_k_configs_and_shards(wino, P):
    """BASELINE layers and their P-rank batch shards with the workspace (planner's choice)."""
    for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x"):
        cfg = CONFIGS[name].with_batch(CONFIGS[name].N // P)
        xh, wh = _inputs(cfg, "smallint", torch.float16)
        y = _run_ws(wino, xh, wh, "auto")
        ref = _round(oracle.direct_conv(xh.float(), wh.float()), torch.float16)
        assert np.array_equal(y.float().numpy(), ref), (name, cfg.N)


def test_half_stream_k_deterministic(wino):
    xh, wh = _inputs(CONFIGS["conv4_x"].with_batch(16), "uniform", torch.bfloat16)
    y1 = _run_ws(wino, xh, wh, "on")
    y2 = _run_ws(wino, xh, wh, "on")
    assert torch.equal(y1, y2)
