"""C-ABI checks that need no GPU: the library loads, exports every symbol that
include/wino.h declares, and its host-only logic (status strings, workspace
sizes, launch plans, argument validation that precedes any device access)
behaves as the header documents."""
import ctypes
import json
import os
import re

import pytest

import paper_conf_ppopp_yanwc20_b200 as wino
from synth_inputs import CONFIGS

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "wino.h")


def _declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(wino_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    L = wino.lib()
    names = _declared_functions()
    assert len(names) >= 10, names
    for n in names:
        assert hasattr(L, n), f"libwino.so does not export {n}"


def test_status_strings_and_version():
    L = wino.lib()
    assert wino.version() >= 100
    for code, name in [(0, b"WINO_OK"), (1, b"WINO_ERR_INVALID_ARG"), (2, b"WINO_ERR_UNSUPPORTED"),
                       (3, b"WINO_ERR_MISALIGNED"), (4, b"WINO_ERR_TOO_LARGE"), (5, b"WINO_ERR_CUDA")]:
        assert L.wino_status_string(code) == name
    assert L.wino_status_string(99) == b"WINO_ERR_UNKNOWN"


def test_filter_workspace_bytes_matches_paper():
    """L993: 16KC floats = 0.25 / 1 / 4 / 16 MB for Conv2..Conv5."""
    with open(os.path.join(ROOT, "tests", "golden", "paper_constants.json")) as f:
        mb = json.load(f)["workspace_MB"]["value"]
    for name, v in mb.items():
        cfg = CONFIGS[name]
        assert wino.filter_workspace_bytes(cfg.C, cfg.K) == int(v * 2 ** 20)
    assert wino.filter_workspace_bytes(0, 5) == 0
    assert wino.filter_workspace_bytes(3, -1) == 0


def test_host_workspace_bytes():
    n = wino.host_workspace_bytes(2, 3, 5, 5, 4)
    need = 3 * 25 * 2 * 4 + 9 * 3 * 4 * 4 + 16 * 3 * 4 * 4 + 4 * 25 * 2 * 4
    assert need <= n <= need + 4 * 256
    assert wino.host_workspace_bytes(0, 3, 5, 5, 4) == 0


@pytest.mark.parametrize("name", list(CONFIGS))
def test_plan_shapes(name):
    c = CONFIGS[name]
    p = wino.plan(c.N, c.C, c.H, c.W, c.K)
    assert p.variant == 0 and (p.bk, p.bn, p.bc) == (64, 32, 8)
    nv = c.N * c.tiles
    assert p.ctas == -(-nv // p.bn) * -(-c.K // p.bk) * p.split_c
    ws = (c.N % 32 == 0 or c.N in (4, 8, 16)) and c.K % 4 == 0  # warp-specialised TMA kernel
    assert p.threads == (384 if ws else 256) and 0 < p.smem_bytes <= 232448
    assert p.load_x == (2 if (ws or c.N % 32 == 0) else (1 if c.N % 4 == 0 else 0))
    assert p.split_c in (1, 2, 4, 8) and (ws or p.split_c == 1)
    assert p.load_u == (2 if c.K % 4 == 0 else 0)
    assert p.launches >= 1


def test_plan_rejects_bad_shapes():
    with pytest.raises(wino.WinoError) as e:
        wino.plan(0, 1, 1, 1, 1)
    assert e.value.status == 1
    with pytest.raises(wino.WinoError) as e:
        wino.plan(1 << 16, 1 << 10, 64, 64, 1)  # x has 2^42 elements
    assert e.value.status == 4


# Validation that happens before any device access (so it runs here without a GPU).
def _fwd(x, u, y, N=2, C=3, H=4, W=4, K=5, pad=1, stride=1):
    L = wino.lib()
    return L.wino_conv2d_f2x3_fwd(ctypes.c_void_p(x), ctypes.c_void_p(u), ctypes.c_void_p(y),
                                  N, C, H, W, K, pad, stride, None)


def test_fwd_argument_validation_host_side():
    X, U, Y = 0x100000, 0x200000, 0x300000  # fake, never dereferenced on these paths
    assert _fwd(0, U, Y) == 1                      # NULL
    assert _fwd(X, U, Y, N=0) == 1                 # dim <= 0
    assert _fwd(X, U, Y, K=-3) == 1
    assert _fwd(X, U, Y, pad=0) == 2               # pad != 1
    assert _fwd(X, U, Y, stride=2) == 2            # stride != 1
    assert _fwd(X + 4, U, Y) == 3                  # misaligned
    assert _fwd(X, U, Y + 8) == 3
    assert _fwd(X, U, X) == 1                      # y aliases x
    assert _fwd(X, U, U + 16) == 1                 # y overlaps u
    assert _fwd(X, U, Y, N=1 << 14, C=1 << 10, H=16, W=16) == 4  # too large
    L = wino.lib()
    assert L.wino_filter_transform(None, ctypes.c_void_p(U), 3, 5, None) == 1
    assert L.wino_filter_transform(ctypes.c_void_p(X + 4), ctypes.c_void_p(U), 3, 5, None) == 3
    assert L.wino_conv2d_f2x3_fwd_tc(ctypes.c_void_p(X), ctypes.c_void_p(U), ctypes.c_void_p(Y),
                                     2, 3, 4, 4, 5, 1, 1, 7, None) == 1  # unknown mode
    assert L.wino_filter_transform_tc(ctypes.c_void_p(X), ctypes.c_void_p(U), 3, 5, 7, None) == 1
    assert L.wino_conv2d_f2x3_fwd_tc(ctypes.c_void_p(X), ctypes.c_void_p(U), ctypes.c_void_p(Y),
                                     2, 3, 4, 4, 5, 2, 1, 0, None) == 2  # pad != 1
    for bad in (-1, 3, 5, 16):  # split-C factor must be 0 (auto), 1, 2, 4 or 8
        assert L.wino_conv2d_f2x3_fwd_split(ctypes.c_void_p(X), ctypes.c_void_p(U), ctypes.c_void_p(Y),
                                            2, 3, 4, 4, 5, 1, 1, bad, None) == 1
    assert L.wino_conv2d_f2x3_fwd_split(ctypes.c_void_p(X), ctypes.c_void_p(U), ctypes.c_void_p(Y),
                                        2, 3, 4, 4, 5, 0, 1, 2, None) == 2  # pad != 1


def test_nonfused_workspace_bytes():
    """NEXT row N3 (include/wino.h): V[16*2][NV][Cp4] + Ug[16*2][K][Cp4] + M[16][K][NV] floats
    (two TF32 planes per operand for the 3xTF32 GEMMs, Cp4 = 4*ceil(C/4)), each part rounded up
    to 256 B; 4 launches per call."""
    rnd = lambda b: -(-b // 256) * 256  # noqa: E731
    for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x", "tiny"):
        c = CONFIGS[name]
        nv = c.N * c.tiles
        c4 = -(-c.C // 4) * 4
        assert wino.nonfused_workspace_bytes(c.N, c.C, c.H, c.W, c.K) == \
            rnd(128 * nv * c4) + rnd(128 * c.K * c4) + rnd(64 * c.K * nv)
    assert wino.nonfused_workspace_bytes(3, 5, 5, 5, 4) == rnd(128 * 27 * 8) + rnd(128 * 4 * 8) + rnd(64 * 4 * 27)
    assert wino.nonfused_workspace_bytes(0, 3, 5, 5, 4) == 0
    assert wino.nonfused_launches() == 4


@pytest.mark.parametrize("P", [2, 4, 8])
def test_plan_splits_small_shards(P):
    """Per-rank batch shards with fewer (k, nu) tiles than SMs get split-C,
    and every shard of the BASELINE layers takes the warp-specialised TMA kernel."""
    from paper_conf_ppopp_yanwc20_b200.dist import shard_range
    for name in ("conv5_x", "conv4_x", "conv3_x", "conv2_x"):
        c = CONFIGS[name]
        lo, hi = shard_range(c.N, 0, P)
        p = wino.plan(hi - lo, c.C, c.H, c.W, c.K)
        assert p.threads == 384 and p.load_x == 2, (name, P)
        tiles = p.ctas // p.split_c
        if tiles < 64:
            assert p.split_c > 1, (name, P, tiles)
        assert p.split_c * 2 * 8 <= c.C or p.split_c == 1  # >= 2 channel blocks per CTA


def test_tc_workspace_and_plan():
    # [ceil(C/8)][ceil(K/128)][16 xi][planes][128 x 8] floats
    for (C, K) in [(1, 1), (8, 128), (9, 129), (512, 512), (64, 64)]:
        for mode, planes in [("tf32", 1), ("3xtf32", 2)]:
            mm = 64 if (planes == 1 and K <= 64) else 128  # tile height rule of the tc kernel
            want = -(-C // 8) * -(-K // mm) * 16 * planes * mm * 8 * 4
            assert wino.filter_workspace_bytes_tc(C, K, mode) == want
    assert wino.lib().wino_filter_workspace_bytes_tc(8, 8, 5) == 0
    c = CONFIGS["conv3_x"]
    p = wino.plan(c.N, c.C, c.H, c.W, c.K, variant=1)
    assert (p.bk, p.bn, p.bc, p.threads) == (128, 32, 8, 512)
    c2 = CONFIGS["conv2_x"]  # K = 64: 64-filter tiles with two nu-halves in TMEM
    p2 = wino.plan(c2.N, c2.C, c2.H, c2.W, c2.K, variant=1)
    assert (p2.bk, p2.bn) == (64, 64)
    assert p.ctas == -(-(c.N * c.tiles) // 32) * -(-c.K // 128)
    assert p.smem_bytes <= 232448 and wino.plan(c.N, c.C, c.H, c.W, c.K, variant=2).smem_bytes <= 232448


def test_python_layer_refuses_cpu_tensors():
    import torch
    x = torch.zeros(3, 4, 4, 2)
    with pytest.raises(ValueError):
        wino.conv2d(x, torch.zeros(3, 4, 4, 5))
    with pytest.raises(ValueError):
        wino.filter_transform(torch.zeros(3, 3, 3, 5))
    with pytest.raises(TypeError):
        wino.conv2d(x.double(), torch.zeros(3, 4, 4, 5))


def test_product_package_never_imports_oracle():
    """The product path must not route through the oracle (no CPU fallback)."""
    pkg = os.path.join(ROOT, "paper_conf_ppopp_yanwc20_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f), errors="ignore").read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", src, re.M), f
                assert "wino_oracle" not in src and "liboracle" not in src, f


def test_stream_k_plan_and_workspace():
    """Host-only planning (no device): the stream-K plan replaces the 2.65-wave conv4_x schedule
    (392 tiles on 148 SMs) and is not taken for conv2_x (42.4 waves: nothing to gain).  One launch:
    the cut tiles are reduced inside the kernel (round 2; round 1 had a fixup launch)."""
    c4, c2 = CONFIGS["conv4_x"], CONFIGS["conv2_x"]
    p = wino.plan(c4.N, c4.C, c4.H, c4.W, c4.K, variant=4)
    assert p.stream_k == 1 and p.launches == 1 and p.ctas == 148 and p.split_c == 1
    assert wino.plan(c4.N, c4.C, c4.H, c4.W, c4.K).stream_k == 0  # no workspace -> regular plan
    assert wino.plan(c2.N, c2.C, c2.H, c2.W, c2.K, variant=4).stream_k == 0
    assert wino.conv_workspace_bytes(c4.N, c4.C, c4.H, c4.W, c4.K) == 148 * 2 * 64 * 4 * 32 * 4 + 768  # + counters
    assert wino.conv_workspace_bytes(0, 1, 1, 1, 1) == 0


def test_multi_layer_launch_grouping():
    """Host-only (148 SMs without a device): wino_conv2d_f2x3_fwd_multi puts the layers with fewer
    than 64 tiles per SM into one shared persistent launch per group of <= 4 and runs the others
    alone through the planner.  ResNet step: all four layers shared (conv2_x at N = 256: 6272 tiles
    = 42 per SM) -> 1 launch, plus one ml_itf_kernel launch when a shard has N = 4 or 8 (P = 4:
    conv5_x; P = 8: conv5_x, conv4_x); a 64-tiles-per-SM layer runs alone."""
    names = ("conv5_x", "conv4_x", "conv3_x", "conv2_x")
    sk = 148 * 2 * 64 * 4 * 32 * 4 + 768
    for P, want in ((1, 1), (2, 1), (4, 2), (8, 2)):
        shapes = [(CONFIGS[n].N // P, CONFIGS[n].C, CONFIGS[n].H, CONFIGS[n].W, CONFIGS[n].K) for n in names]
        assert wino.conv_multi_launches(shapes) == want, P
        # N = 4 / 8 layers (vmode): + one input-transform launch and a V buffer of 16 x C x NV floats
        vbytes = sum(-(-16 * C * N * ((H + 1) // 2) * ((W + 1) // 2) * 4 // 256) * 256
                     for N, C, H, W, K in shapes if N in (4, 8))
        assert wino.conv_multi_workspace_bytes(shapes) == sk + vbytes, P
    big = (512, 64, 56, 56, 64)  # 25088 tiles = 169.5 per SM: alone (the planner's one launch)
    assert wino.conv_multi_launches([big]) == wino.plan(*big[:4], big[4], variant=4).launches == 1
    assert wino.conv_multi_launches([big, (32, 64, 9, 9, 64)]) == 2
    small = (32, 64, 9, 9, 64)
    assert wino.conv_multi_launches([small] * 4) == 1
    assert wino.conv_multi_launches([small] * 5) == 2  # groups of at most 4
    odd = (3, 16, 8, 8, 16)  # N = 3: not warp-specialised -> its own plan (one launch)
    assert wino.conv_multi_launches([small, odd, small]) == 1 + wino.plan(*odd[:4], odd[4], variant=4).launches
    assert wino.conv_multi_launches([(8, 16, 8, 8, 18)]) == 1  # K % 4 != 0: planner, 1 launch
    with pytest.raises(wino.WinoError):
        wino.conv_multi_launches([(0, 1, 1, 1, 1)])


def test_tensor_core_stream_k_plans_and_workspaces():
    """Host-only planning: the 16-bit and TF32 tcgen05 kernels take stream-K only for tile-starved
    shapes (conv5_x: 64 tiles of 128 x 32 for 148 SMs), never for the many-tile layers, with either
    tile height (64-filter TF32 tiles for K <= 64 included); workspace sizes are 2 slots of 64 KiB per
    SM (148 without a device)."""
    c5, c4, c2 = CONFIGS["conv5_x"], CONFIGS["conv4_x"], CONFIGS["conv2_x"]
    for v in (5, 6, 7):
        p = wino.plan(c5.N, c5.C, c5.H, c5.W, c5.K, variant=v)
        assert p.stream_k == 1 and p.launches == 2 and p.ctas == 148, (v, p)
        assert wino.plan(c2.N, c2.C, c2.H, c2.W, c2.K, variant=v).stream_k == 0
    assert wino.plan(c5.N, c5.C, c5.H, c5.W, c5.K, variant=3).stream_k == 0  # no workspace
    assert wino.plan(c5.N // 8, c2.C, c2.H, c2.W, c2.K, variant=6).stream_k == 0  # 49 tiles x 8 blocks: whole tiles
    p64 = wino.plan(32, 512, 7, 7, 64, variant=6)  # TF32, K <= 64: 8 tiles of 64 x 64 for 148 SMs
    assert p64.bk == 64 and p64.stream_k == 1 and p64.launches == 2
    assert wino.half_workspace_bytes(c4.N, c4.C, c4.H, c4.W, c4.K) == 148 * 2 * 64 * 1024
    assert wino.tc_workspace_bytes(c4.N, c4.C, c4.H, c4.W, c4.K) == 148 * 2 * 64 * 1024
    hwn = c4.H * c4.W * c4.N
    assert wino.nchw_workspace_bytes(c4.N, c4.C, c4.H, c4.W, c4.K) == \
        (c4.C * hwn * 4 + 255) // 256 * 256 + (c4.K * hwn * 4 + 255) // 256 * 256 + 148 * 64 * 1024 + 768


def test_header_is_plain_c99(tmp_path):
    """include/wino.h is a C ABI: it compiles as ISO C99 with -pedantic -Werror (no C++ or torch types)."""
    import shutil
    import subprocess
    if shutil.which("gcc") is None:
        pytest.skip("gcc not available")
    src = tmp_path / "use_header.c"
    src.write_text('#include "wino.h"\nint main(void) { wino_plan_t p; wino_ftf_job_t j; wino_host_layer_t l;\n'
                   '  (void)p; (void)j; (void)l; return wino_filter_workspace_bytes(1, 1) == 64 ? 0 : 1; }\n')
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run(["gcc", "-std=c99", "-Wall", "-Wextra", "-pedantic", "-Werror", "-I", os.path.join(root, "include"),
                        "-c", str(src), "-o", str(tmp_path / "use_header.o")], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
