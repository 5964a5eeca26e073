"""Oracle for the fused batched Winograd F(2x2,3x3) convolution -- TEST INFRASTRUCTURE.

A plain fp64 CPU reference written from Yan, Wang & Chu (PPoPP'20),
/root/reference/PAPER.md (cited as L<n>):

* :func:`direct_conv`       Eq. 4 (L177-187), the definition the method must reproduce.
* :func:`winograd_conv`     Eq. 5-8 (L191-207), the naive step-by-step method.
* :func:`filter_transform`  Eq. 5 (L191), U = G g G^T in the (C,4,4,K) layout of Table 4 (L507).
* :func:`direct_sample`     Eq. 4 at selected output points (full-size parity checks).
* :mod:`oracle.exact`       exact-rational single-tile transforms (Eq. 1-3, 5-8).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` arm may import this package.  The product path
(``paper_conf_ppopp_yanwc20_b200``) never does; the two share no code.

Parity status: every function here is pinned by tests/test_oracle.py
(identity on rational tiles, torch.conv2d fp64, brute force, exact small-integer
agreement, invariants, paper-printed constants).  No function is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "wino_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle/wino_oracle.c -> oracle/liboracle.so (gcc, OpenMP, fp64, no contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-shared", "-fPIC",
               _SRC, "-o", _LIB]
        subprocess.check_call(cmd)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        dp = ctypes.POINTER(ctypes.c_double)
        i = ctypes.c_int
        lib.oracle_direct_conv.argtypes = [dp, dp, dp, i, i, i, i, i]
        lib.oracle_direct_conv.restype = None
        lib.oracle_direct_sample.argtypes = [dp, dp, i, i, i, i, i,
                                             ctypes.POINTER(ctypes.c_int64), ctypes.c_long, dp]
        lib.oracle_direct_sample.restype = None
        lib.oracle_filter_transform.argtypes = [dp, dp, i, i]
        lib.oracle_filter_transform.restype = None
        lib.oracle_winograd_conv.argtypes = [dp, dp, dp, dp, i, i, i, i, i]
        lib.oracle_winograd_conv.restype = ctypes.c_int
        for name in ("oracle_ftf_tile", "oracle_itf_tile", "oracle_otf_tile"):
            getattr(lib, name).argtypes = [dp, dp]
            getattr(lib, name).restype = None
        lib.oracle_filter_transform_f4.argtypes = [dp, dp, i, i]
        lib.oracle_filter_transform_f4.restype = None
        lib.oracle_winograd_f4_conv.argtypes = [dp, dp, dp, i, i, i, i, i]
        lib.oracle_winograd_f4_conv.restype = ctypes.c_int
        for name in ("oracle_ftf4_tile", "oracle_itf4_tile", "oracle_otf4_tile"):
            getattr(lib, name).argtypes = [dp, dp]
            getattr(lib, name).restype = None
        lib.oracle_num_threads.argtypes = []
        lib.oracle_num_threads.restype = ctypes.c_int
        lib.oracle_set_num_threads.argtypes = [ctypes.c_int]
        lib.oracle_set_num_threads.restype = None
        _lib = lib
    return _lib


def _f64(a) -> np.ndarray:
    """Promote stored values (fp32 or otherwise) to a contiguous fp64 numpy array (exact)."""
    if hasattr(a, "detach"):  # torch tensor
        a = a.detach().cpu().numpy()
    return np.ascontiguousarray(np.asarray(a, dtype=np.float64))


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def set_num_threads(n: int) -> None:
    """OpenMP threads of the following oracle calls (plumbing; no arithmetic)."""
    _load().oracle_set_num_threads(int(n))


def direct_conv(x_chwn, w_crsk) -> np.ndarray:
    """Eq. 4 (L177-187), pad 1, stride 1: x (C,H,W,N), w (C,3,3,K) -> y (K,H,W,N), fp64."""
    x, w = _f64(x_chwn), _f64(w_crsk)
    C, H, W, N = x.shape
    assert w.shape[:3] == (C, 3, 3), w.shape
    K = w.shape[3]
    y = np.empty((K, H, W, N), dtype=np.float64)
    _load().oracle_direct_conv(_ptr(x), _ptr(w), _ptr(y), N, C, H, W, K)
    return y


def direct_sample(x_chwn, w_crsk, idx) -> np.ndarray:
    """Eq. 4 at points idx (n_pts, 4) = (k, i, j, n); bit-identical to direct_conv's entries."""
    x, w = _f64(x_chwn), _f64(w_crsk)
    C, H, W, N = x.shape
    K = w.shape[3]
    idx = np.ascontiguousarray(np.asarray(idx, dtype=np.int64).reshape(-1, 4))
    assert (idx >= 0).all() and (idx[:, 0] < K).all() and (idx[:, 1] < H).all() \
        and (idx[:, 2] < W).all() and (idx[:, 3] < N).all()
    out = np.empty(idx.shape[0], dtype=np.float64)
    _load().oracle_direct_sample(_ptr(x), _ptr(w), N, C, H, W, K,
                                 idx.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                 idx.shape[0], _ptr(out))
    return out


def filter_transform(w_crsk) -> np.ndarray:
    """Eq. 5 (L191): U (C,4,4,K) = G w G^T per (c,k), element (r',s') at [c,r',s',k]."""
    w = _f64(w_crsk)
    C, K = w.shape[0], w.shape[3]
    u = np.empty((C, 4, 4, K), dtype=np.float64)
    _load().oracle_filter_transform(_ptr(w), _ptr(u), C, K)
    return u


def winograd_conv(x_chwn, w_crsk, return_u: bool = False):
    """Eq. 5-8 (L191-207) step by step in fp64: y (K,H,W,N) [and U (C,4,4,K)]."""
    x, w = _f64(x_chwn), _f64(w_crsk)
    C, H, W, N = x.shape
    K = w.shape[3]
    y = np.empty((K, H, W, N), dtype=np.float64)
    u = np.empty((C, 4, 4, K), dtype=np.float64)
    rc = _load().oracle_winograd_conv(_ptr(x), _ptr(w), _ptr(y), _ptr(u), N, C, H, W, K)
    if rc != 0:
        raise MemoryError("oracle_winograd_conv: allocation failed")
    return (y, u) if return_u else y


def filter_transform_f4(w_crsk) -> np.ndarray:
    """NEXT row N1: F(4x4,3x3) filter transform U4 (C,6,6,K) = G4 w G4^T (Lavin-Gray matrices)."""
    w = _f64(w_crsk)
    C, K = w.shape[0], w.shape[3]
    u = np.empty((C, 6, 6, K), dtype=np.float64)
    _load().oracle_filter_transform_f4(_ptr(w), _ptr(u), C, K)
    return u


def winograd_f4_conv(x_chwn, w_crsk) -> np.ndarray:
    """NEXT row N1: naive F(4x4,3x3) Winograd conv in fp64 (same steps as Eq. 5-8, alpha = 6)."""
    x, w = _f64(x_chwn), _f64(w_crsk)
    C, H, W, N = x.shape
    K = w.shape[3]
    y = np.empty((K, H, W, N), dtype=np.float64)
    if _load().oracle_winograd_f4_conv(_ptr(x), _ptr(w), _ptr(y), N, C, H, W, K) != 0:
        raise MemoryError("oracle_winograd_f4_conv: allocation failed")
    return y


def ftf4_tile(g3x3) -> np.ndarray:
    return _tile("oracle_ftf4_tile", g3x3, 36).reshape(6, 6)


def itf4_tile(d6x6) -> np.ndarray:
    return _tile("oracle_itf4_tile", d6x6, 36).reshape(6, 6)


def otf4_tile(m6x6) -> np.ndarray:
    return _tile("oracle_otf4_tile", m6x6, 16).reshape(4, 4)


def _tile(fn, inp, n_out):
    a = _f64(inp).reshape(-1)
    out = np.empty(n_out, dtype=np.float64)
    getattr(_load(), fn)(_ptr(a), _ptr(out))
    return out


def ftf_tile(g3x3) -> np.ndarray:
    return _tile("oracle_ftf_tile", g3x3, 16).reshape(4, 4)


def itf_tile(d4x4) -> np.ndarray:
    return _tile("oracle_itf_tile", d4x4, 16).reshape(4, 4)


def otf_tile(m4x4) -> np.ndarray:
    return _tile("oracle_otf_tile", m4x4, 4).reshape(2, 2)


def max_rel_err(y_test, y_ref) -> float:
    """SURVEY 8(c) acceptance metric: max|y_test - y_ref| / max|y_ref| (0 if both all-zero)."""
    t = _f64(y_test)
    r = _f64(y_ref)
    den = float(np.max(np.abs(r))) if r.size else 0.0
    num = float(np.max(np.abs(t - r))) if r.size else 0.0
    if den == 0.0:
        return 0.0 if num == 0.0 else float("inf")
    return num / den
