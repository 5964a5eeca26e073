"""Error model for NEXT row N4 (FP16 / BF16 operands on tcgen05 kind::f16) -- design tool.

Simulates, in numpy on the CPU, the rounding the half-precision path performs:
inputs x, w stored in the half type; U = G w G^T and V = B^T d B computed in fp32
and rounded (round-to-nearest-even) to the half type; M = sum_c U*V accumulated
in fp32; Y = A^T M A in fp32; y rounded to the half type.  Reports
max|y - y_ref| / max|y_ref| against the fp64 direct convolution (Eq. 4) of the
half-valued inputs.  Used to set the tolerances in DESIGN.md sec. 4 (not by tests).
"""
import sys

import numpy as np
import torch

Bt = np.array([[1, 0, -1, 0], [0, 1, 1, 0], [0, -1, 1, 0], [0, 1, 0, -1]], np.float32)
G = np.array([[1, 0, 0], [.5, .5, .5], [.5, -.5, .5], [0, 0, 1]], np.float32)
At = np.array([[1, 1, 1, 0], [0, 1, -1, -1]], np.float32)


def rnd(a, dt):
    return torch.from_numpy(np.ascontiguousarray(a, np.float32)).to(dt).to(torch.float32).numpy()


def run(N, C, K, H, W, dt, seed=0):
    g = np.random.default_rng(seed)
    x = rnd(g.uniform(-1, 1, (C, H, W, N)), dt)
    w = rnd(g.uniform(-1, 1, (C, 3, 3, K)), dt)
    # fp64 direct (Eq. 4) on the half-valued inputs
    xp = np.zeros((C, H + 2, W + 2, N)); xp[:, 1:-1, 1:-1] = x
    ref = np.zeros((K, H, W, N))
    for r in range(3):
        for s in range(3):
            ref += np.einsum("chwn,ck->khwn", xp[:, r:r + H, s:s + W], w[:, r, s, :].astype(np.float64))
    U = rnd(np.einsum("ir,crsk,js->cijk", G, w, G), dt)                      # (C,4,4,K)
    TH, TW = (H + 1) // 2, (W + 1) // 2
    xq = np.zeros((C, 2 * TH + 2, 2 * TW + 2, N), np.float32); xq[:, 1:H + 1, 1:W + 1] = x
    d = np.stack([np.stack([xq[:, 2 * a:2 * a + 4, 2 * b:2 * b + 4] for b in range(TW)], 1) for a in range(TH)], 1)
    V = rnd(np.einsum("ir,cabrsn,js->cabijn", Bt, d, Bt), dt)               # (C,TH,TW,4,4,N)
    M = np.einsum("cijk,cabijn->kabijn", U, V, dtype=np.float32)            # fp32 accumulate
    Y = np.einsum("pi,kabijn,qj->kabpqn", At, M, At).astype(np.float32)
    y = Y.transpose(0, 1, 3, 2, 4, 5).reshape(K, 2 * TH, 2 * TW, N)[:, :H, :W]
    y = rnd(y, dt)
    return np.abs(y - ref).max() / np.abs(ref).max(), np.median(np.abs(y - ref)) / np.abs(ref).max()


if __name__ == "__main__":
    shapes = {"conv5": (4, 512, 64, 7, 7), "conv4": (4, 256, 64, 14, 14), "conv3": (4, 128, 64, 28, 28),
              "conv2": (4, 64, 64, 56, 56), "tiny": (1, 8, 8, 8, 8)}
    for name, dt in (("fp16", torch.float16), ("bf16", torch.bfloat16)):
        for k, s in shapes.items():
            mx, med = run(*s, dt)
            print(f"{name} {k:6s} max {mx:.2e} median {med:.2e}")
        sys.stdout.flush()
