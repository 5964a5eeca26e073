"""Debug: forced stream-K of the TF32 kernel with 64-filter tiles (build -DWINO_TC_SK_MM64 into
build_ab/libwino_tcsk64.so).  For every wrong output prints where it sits: tile, nu-half, nu within
the half, filter, output position q, and the stream-K piece structure of that tile."""
import os
import sys

sys.path.insert(0, os.getcwd())
os.environ.setdefault("WINO_LIB_PATH", os.path.abspath("build_ab/libwino_tcsk64.so"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ppopp_yanwc20_b200 as wino  # noqa: E402
from synth_inputs import Conv3x3Config, make_inputs  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
sms = torch.cuda.get_device_properties(0).multi_processor_count
total_bad = 0
for shape in [(32, 64, 64, 30, 30), (32, 64, 64, 16, 16), (32, 64, 48, 14, 14)]:
    N, C, K, H, W = shape
    x, w = make_inputs(Conv3x3Config("s", N, C, K, H, W), kind="smallint")
    xd = x.cuda()
    u = wino.filter_transform_tc(w.cuda(), "tf32")
    ws = torch.empty(wino.tc_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device="cuda")
    ref = oracle.direct_conv(x, w)
    TW, TH = (W + 1) // 2, (H + 1) // 2
    NV = N * TH * TW
    ncb = (C + 7) // 8
    tiles = (NV + 63) // 64
    units = tiles * ncb
    q, r = divmod(units, min(sms, 256))
    starts = [b * q + min(b, r) for b in range(min(sms, 256) + 1)]
    for rep in range(reps):
        ws.fill_(255 if rep % 2 else 0)  # NaN pattern / zeros in the partial-tile slots
        y = wino.conv2d_tc(xd, u, ws=ws, stream_k="on")
        torch.cuda.synchronize()
        yn = y.cpu().double().numpy()
        bad = np.argwhere(yn != ref)
        total_bad += len(bad) > 0
        print(shape, "rep", rep, "bad", len(bad), flush=True)
        seen = set()
        for k, i, j, n in bad[:4000]:
            t = (i // 2) * TW + (j // 2)
            nu = t * N + n
            tile, jj = nu // 64, nu % 64
            key = (tile, jj // 8, k // 16)
            if key in seen:
                continue
            seen.add(key)
            u0, u1 = tile * ncb, tile * ncb + ncb
            cuts = [(b, starts[b]) for b in range(len(starts) - 1) if u0 < starts[b] < u1]
            print(f"   tile {tile} half {jj // 32} nu {jj % 32} k {k} q {(i % 2) * 2 + j % 2} "
                  f"got {yn[k, i, j, n]:.0f} want {ref[k, i, j, n]:.0f} cuts(b,start) {cuts} "
                  f"tile units [{u0},{u1})", flush=True)
            if len(seen) > 24:
                break
print("TOTAL failing runs", total_bad)

# ---- which piece is wrong: compare every workspace slot of the failing shape with the oracle's
# partial output over that piece's channel range (Eq. 8 is linear: a piece's partial outputs are
# the convolution restricted to its channels) ----
N, C, K, H, W = 32, 64, 64, 30, 30
x, w = make_inputs(Conv3x3Config("s", N, C, K, H, W), kind="smallint")
xd = x.cuda()
u = wino.filter_transform_tc(w.cuda(), "tf32")
ws = torch.empty(wino.tc_workspace_bytes(N, C, H, W, K), dtype=torch.uint8, device="cuda")
TW, TH = (W + 1) // 2, (H + 1) // 2
NV, ncb = N * TH * TW, (C + 7) // 8
G = min(sms, 256)
units = ((NV + 63) // 64) * ncb
q, r = divmod(units, G)
starts = [b * q + min(b, r) for b in range(G + 1)]
partial_cache = {}


def partial_ref(c0, c1):
    if (c0, c1) not in partial_cache:
        xm, wm = x.clone(), w.clone()
        xm[:c0] = 0
        xm[c1:] = 0
        wm[:c0] = 0
        wm[c1:] = 0
        partial_cache[(c0, c1)] = oracle.direct_conv(xm, wm)
    return partial_cache[(c0, c1)]


SLOT = 64 * 4 * 64
for rep in range(reps):
    ws.fill_(255)
    wino.conv2d_tc(xd, u, ws=ws, stream_k="on")
    torch.cuda.synchronize()
    wsf = ws.view(torch.float32).cpu().numpy()
    nbad = 0
    for b in range(G):
        a0, a1 = starts[b], starts[b + 1]
        pieces, a, n = [], a0, 0
        while a < a1:
            tile = a // ncb
            lo = a - tile * ncb
            hi = min(ncb, lo + (a1 - a))
            a += hi - lo
            n += 1
            if hi - lo != ncb:
                pieces.append((tile, lo, hi, 2 * b + (1 if n > 1 else 0), n))
        for tile, lo, hi, slot, n in pieces:
            ref = partial_ref(lo * 8, hi * 8)
            got = wsf[slot * SLOT:(slot + 1) * SLOT].reshape(64, 4, 64)  # [kl][q][j]
            for j in range(64):
                nu = tile * 64 + j
                if nu >= NV:
                    continue
                t, nn = divmod(nu, N)
                th, tw = divmod(t, TW)
                for qq in range(4):
                    i, jj = 2 * th + qq // 2, 2 * tw + qq % 2
                    if i >= H or jj >= W:
                        continue
                    bad = np.nonzero(got[:, qq, j] != ref[:, i, jj, nn])[0]
                    if len(bad):
                        nbad += len(bad)
                        shown = globals().setdefault("shown", set())
                        key = (rep, b, n, j // 8, qq)
                        if key not in shown and len(shown) < 60:
                            shown.add(key)
                            print(f"rep {rep} CTA {b} piece#{n} tile {tile} cb [{lo},{hi}) slot {slot} nu {j} q {qq} "
                                  f"k {list(bad[:4])} got {got[bad[0], qq, j]} want {ref[bad[0], i, jj, nn]}",
                                  flush=True)
    print("rep", rep, "bad partial entries", nbad, flush=True)
