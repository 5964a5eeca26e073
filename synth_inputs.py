"""Seeded synthetic inputs shared by tests, bench.py and smoke().

Holds NONE of the method's arithmetic: only shapes (BASELINE.json ``configs``,
which are the ResNet 3x3 layers of Table 1, L127-129 of PAPER.md) and seeded
random tensors in the paper's layouts (Table 4):
x (C,H,W,N) "CHWN", w (C,3,3,K) "CRSK".  The recipe is stated in DESIGN.md
("Input recipe"):

* ``uniform``  x, w ~ U[-1, 1) fp32  (torch CPU generator, seeds 1234 / 1235)
* ``smallint`` x, w integers in [-3, 3] stored as fp32 (exactness checks)
* ``resnet``   x = ReLU(N(0,1)) (about half zeros), w ~ N(0, 2/(9C)) (He init)

Both the oracle side and the CUDA side read the same tensors from here.
"""
from __future__ import annotations

import math
from dataclasses import dataclass

import torch

SEED_X = 1234
SEED_W = 1235


@dataclass(frozen=True)
class Conv3x3Config:
    name: str
    N: int
    C: int
    K: int
    H: int
    W: int

    @property
    def tiles(self) -> int:
        """T = ceil(H/2) * ceil(W/2) output tiles per image (Table 3 note, L167)."""
        return ((self.H + 1) // 2) * ((self.W + 1) // 2)

    @property
    def eff_flops(self) -> int:
        """Direct-conv-equivalent flops 2*N*K*C*H*W*9 (BASELINE.json metric)."""
        return 18 * self.N * self.K * self.C * self.H * self.W

    def with_batch(self, n: int) -> "Conv3x3Config":
        return Conv3x3Config(self.name, n, self.C, self.K, self.H, self.W)


# BASELINE.json "configs" (pad=1, stride=1, fp32)
CONFIGS = {
    "tiny": Conv3x3Config("tiny", 1, 8, 8, 8, 8),
    "conv5_x": Conv3x3Config("conv5_x", 32, 512, 512, 7, 7),
    "conv4_x": Conv3x3Config("conv4_x", 64, 256, 256, 14, 14),
    "conv3_x": Conv3x3Config("conv3_x", 128, 128, 128, 28, 28),
    "conv2_x": Conv3x3Config("conv2_x", 256, 64, 64, 56, 56),
}
RESNET_LAYERS = ("conv2_x", "conv3_x", "conv4_x", "conv5_x")


def make_inputs(cfg: Conv3x3Config, kind: str = "uniform", seed_x: int = SEED_X,
                seed_w: int = SEED_W):
    """Return (x (C,H,W,N), w (C,3,3,K)) as contiguous fp32 CPU tensors."""
    gx = torch.Generator().manual_seed(seed_x)
    gw = torch.Generator().manual_seed(seed_w)
    xs = (cfg.C, cfg.H, cfg.W, cfg.N)
    ws = (cfg.C, 3, 3, cfg.K)
    if kind == "uniform":
        x = torch.rand(xs, generator=gx, dtype=torch.float32) * 2 - 1
        w = torch.rand(ws, generator=gw, dtype=torch.float32) * 2 - 1
    elif kind == "smallint":
        x = torch.randint(-3, 4, xs, generator=gx).to(torch.float32)
        w = torch.randint(-3, 4, ws, generator=gw).to(torch.float32)
    elif kind == "resnet":
        x = torch.relu(torch.randn(xs, generator=gx, dtype=torch.float32))
        w = torch.randn(ws, generator=gw, dtype=torch.float32) * math.sqrt(2.0 / (9 * cfg.C))
    else:
        raise ValueError(f"unknown input kind {kind!r}")
    return x.contiguous(), w.contiguous()


def sample_points(K: int, H: int, W: int, N: int, n_pts: int, seed: int = 7):
    """Seeded output sample (n_pts, 4) of (k, i, j, n) that always includes the
    four corners / borders of the output plane and the first and last k, n."""
    g = torch.Generator().manual_seed(seed)
    pts = torch.stack([torch.randint(0, K, (n_pts,), generator=g),
                       torch.randint(0, H, (n_pts,), generator=g),
                       torch.randint(0, W, (n_pts,), generator=g),
                       torch.randint(0, N, (n_pts,), generator=g)], dim=1)
    fixed = []
    for k in {0, K - 1}:
        for i in {0, H - 1}:
            for j in {0, W - 1}:
                for n in {0, N - 1}:
                    fixed.append((k, i, j, n))
    return torch.cat([torch.tensor(fixed, dtype=torch.int64), pts.to(torch.int64)], dim=0)
