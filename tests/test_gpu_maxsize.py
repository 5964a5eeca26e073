"""GPU parity at the maximum tensor size the C ABI accepts (just under 2^31 elements per tensor).

Catches 32-bit index overflow anywhere in the load / store / workspace paths: x and y of
C*H*W*N = 2,146,959,360 elements (8.6 GB each in fp32).  The inputs are seeded small
integers generated on the device; each sampled output is checked bit for bit against the
oracle's Eq. 4 evaluated on the 3x3 neighbourhood of that output (the crop of x around it
keeps the zero padding of the true borders, so the value is the full-size one).
"""
import numpy as np
import pytest
import torch

import oracle

pytestmark = pytest.mark.gpu

DEV = "cuda:0"
N, C, K, H, W = 256, 64, 64, 362, 362  # C*H*W*N = 2,146,959,360 < 2^31 - 1


@pytest.fixture(scope="module")
def big():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    free, _ = torch.cuda.mem_get_info()
    if free < 40 << 30:
        pytest.skip("needs ~40 GB of free device memory")
    import paper_conf_ppopp_yanwc20_b200 as wino
    wino.lib()
    g = torch.Generator(device=DEV).manual_seed(77)
    x = torch.randint(-3, 4, (C, H, W, N), generator=g, device=DEV, dtype=torch.int8).to(torch.float32)
    w = torch.randint(-3, 4, (C, 3, 3, K), generator=g, device=DEV, dtype=torch.int8).to(torch.float32)
    gp = torch.Generator().manual_seed(78)
    pts = torch.stack([torch.randint(0, K, (300,), generator=gp), torch.randint(0, H, (300,), generator=gp),
                       torch.randint(0, W, (300,), generator=gp), torch.randint(0, N, (300,), generator=gp)], 1)
    corners = torch.tensor([[K - 1, H - 1, W - 1, N - 1], [0, 0, 0, 0], [K - 1, 0, W - 1, N - 1],
                            [0, H - 1, 0, N - 1]], dtype=torch.int64)
    pts = torch.cat([corners, pts])
    ref = []
    wc = w.cpu()
    for k, i, j, n in pts.tolist():
        r0, r1, c0, c1 = max(i - 1, 0), min(i + 2, H), max(j - 1, 0), min(j + 2, W)
        crop = x[:, r0:r1, c0:c1, n:n + 1].cpu()
        ref.append(oracle.direct_sample(crop, wc, np.array([[k, i - r0, j - c0, 0]]))[0])
    return wino, x, w, pts, np.array(ref)


def _check(y, pts, ref, dt=None):
    ii = pts.to(DEV)
    got = y[ii[:, 0], ii[:, 1], ii[:, 2], ii[:, 3]].float().cpu().double().numpy()
    if dt is not None:  # 16-bit output: RNE of the exact integer result
        ref = torch.from_numpy(ref).to(torch.float32).to(dt).double().numpy()
    assert np.array_equal(got, ref)


def test_maxsize_fp32_regular_and_stream_k(big):
    wino, x, w, pts, ref = big
    u = wino.filter_transform(w)
    y = wino.conv2d(x, u)
    torch.cuda.synchronize()
    _check(y, pts, ref)
    ws = torch.zeros(wino.conv_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device=DEV)
    y.fill_(float("nan"))
    wino.conv2d(x, u, out=y, ws=ws, stream_k="on")
    torch.cuda.synchronize()
    _check(y, pts, ref)


def test_maxsize_tf32(big):
    wino, x, w, pts, ref = big
    y = wino.conv2d_tc(x, wino.filter_transform_tc(w, "tf32"))
    torch.cuda.synchronize()
    _check(y, pts, ref)  # small integers: exact in TF32 too


def test_maxsize_fp16(big):
    wino, x, w, pts, ref = big
    xh = x.half()
    y = wino.conv2d_half(xh, wino.filter_transform_half(w.half()))
    del xh
    torch.cuda.synchronize()
    _check(y, pts, ref, torch.float16)
