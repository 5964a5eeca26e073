"""Python binding of libwino.so -- fused batched Winograd F(2x2,3x3) on B200.

Yan, Wang & Chu, "Optimizing Batched Winograd Convolution on GPUs" (PPoPP'20),
re-designed for sm_100a.  This module only marshals arguments: it checks
dtype / device / contiguity / shape of torch tensors, passes raw pointers and
the current CUDA stream to the C ABI declared in include/wino.h, and raises on
any non-OK status.  Every step of the computation runs in the CUDA kernels of
libwino.so; if the library is missing the import of any op raises -- there is
no CPU or PyTorch fallback.

Layouts (Table 4): x (C,H,W,N), w (C,3,3,K), u (C,4,4,K), y (K,H,W,N).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import torch

__all__ = [
    "WinoError", "lib", "version", "filter_workspace_bytes", "filter_transform", "conv2d",
    "conv2d_host", "host_workspace_bytes", "plan", "Plan", "TC_TF32", "TC_3XTF32",
    "TcFilter", "filter_workspace_bytes_tc", "filter_transform_tc", "conv2d_tc",
    "host_multi_workspace_bytes", "conv2d_host_multi",
    "filter_workspace_bytes_f4", "filter_transform_f4", "conv2d_f4",
    "filter_transform_kcrs", "conv2d_nchw", "nonfused_workspace_bytes", "conv2d_nonfused", "nonfused_launches",
    "HALF_FP16", "HALF_BF16", "HalfFilter", "filter_workspace_bytes_half", "filter_transform_half",
    "conv2d_half", "conv_workspace_bytes", "conv2d_multi", "conv_multi_workspace_bytes", "nchw_workspace_bytes", "half_workspace_bytes", "tc_workspace_bytes", "f4_workspace_bytes", "filter_transform_multi",
]

_PKG = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.environ.get("WINO_LIB_PATH") or os.path.join(_PKG, "libwino.so")  # override: A/B builds
_lib = None

TC_TF32 = 0
TC_3XTF32 = 1
HALF_FP16 = 0
HALF_BF16 = 1
_HALF_DTYPES = {torch.float16: HALF_FP16, torch.bfloat16: HALF_BF16}
_STATUS = {0: "WINO_OK", 1: "WINO_ERR_INVALID_ARG", 2: "WINO_ERR_UNSUPPORTED",
           3: "WINO_ERR_MISALIGNED", 4: "WINO_ERR_TOO_LARGE", 5: "WINO_ERR_CUDA"}


class WinoError(RuntimeError):
    def __init__(self, status: int, where: str, cuda_error: int = 0):
        self.status = status
        self.cuda_error = cuda_error
        msg = f"{where}: {_STATUS.get(status, status)}"
        if status == 5:
            msg += f" (cudaError {cuda_error})"
        super().__init__(msg)


class _Plan(ctypes.Structure):
    _fields_ = [("variant", ctypes.c_int), ("bk", ctypes.c_int), ("bn", ctypes.c_int),
                ("bc", ctypes.c_int), ("load_x", ctypes.c_int), ("load_u", ctypes.c_int),
                ("split_c", ctypes.c_int), ("ctas", ctypes.c_int64), ("threads", ctypes.c_int),
                ("smem_bytes", ctypes.c_int), ("launches", ctypes.c_int), ("stream_k", ctypes.c_int)]


class _HostLayer(ctypes.Structure):
    _fields_ = [("x_host", ctypes.c_void_p), ("w_host", ctypes.c_void_p), ("y_host", ctypes.c_void_p),
                ("N", ctypes.c_int), ("C", ctypes.c_int), ("H", ctypes.c_int), ("W", ctypes.c_int),
                ("K", ctypes.c_int)]


@dataclass(frozen=True)
class Plan:
    variant: int
    bk: int
    bn: int
    bc: int
    load_x: int  # 0 cp.async 4 B, 1 cp.async 16 B, 2 TMA
    load_u: int
    split_c: int
    ctas: int
    threads: int
    smem_bytes: int
    launches: int
    stream_k: int = 0


class _ConvJob(ctypes.Structure):
    _fields_ = [("x", ctypes.c_void_p), ("u", ctypes.c_void_p), ("y", ctypes.c_void_p),
                ("N", ctypes.c_int), ("C", ctypes.c_int), ("H", ctypes.c_int), ("W", ctypes.c_int),
                ("K", ctypes.c_int)]


def lib() -> ctypes.CDLL:
    """Load libwino.so (built in-tree by __graft_entry__.build()); raise if absent."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise ImportError(f"libwino.so not built at {_LIB_PATH}; run __graft_entry__.build() "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(_LIB_PATH)
    vp, i, st = ctypes.c_void_p, ctypes.c_int, ctypes.c_size_t
    L.wino_version.restype = i
    L.wino_version.argtypes = []
    L.wino_status_string.restype = ctypes.c_char_p
    L.wino_status_string.argtypes = [i]
    L.wino_last_cuda_error.restype = i
    L.wino_last_cuda_error.argtypes = []
    L.wino_filter_workspace_bytes.restype = st
    L.wino_filter_workspace_bytes.argtypes = [i, i]
    L.wino_filter_transform.restype = i
    L.wino_filter_transform.argtypes = [vp, vp, i, i, vp]
    L.wino_conv2d_f2x3_fwd.restype = i
    L.wino_conv2d_f2x3_fwd.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, vp]
    if hasattr(L, "wino_conv2d_f2x3_fwd_split") or not os.environ.get("WINO_LIB_PATH"):  # A/B builds may predate it
        L.wino_conv2d_f2x3_fwd_split.restype = i
        L.wino_conv2d_f2x3_fwd_split.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, i, vp]
    for name in ("wino_filter_transform_kcrs", "wino_conv2d_f2x3_fwd_nchw"):
        if hasattr(L, name) or not os.environ.get("WINO_LIB_PATH"):  # A/B builds may predate them
            getattr(L, name).restype = i
    if hasattr(L, "wino_filter_transform_kcrs") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_filter_transform_kcrs.argtypes = [vp, vp, i, i, vp]
        L.wino_conv2d_f2x3_fwd_nchw.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, vp]
    if hasattr(L, "wino_conv2d_f2x3_fwd_nonfused") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_nonfused_workspace_bytes.restype = st
        L.wino_nonfused_workspace_bytes.argtypes = [i, i, i, i, i]
        L.wino_conv2d_f2x3_fwd_nonfused.restype = i
        L.wino_conv2d_f2x3_fwd_nonfused.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, vp, st, vp]
    if hasattr(L, "wino_conv2d_f2x3_fwd_nonfused_tf32") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_conv2d_f2x3_fwd_nonfused_tf32.restype = i
        L.wino_conv2d_f2x3_fwd_nonfused_tf32.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, vp, st, vp]
    L.wino_conv2d_f2x3_fwd_tc.restype = i
    L.wino_conv2d_f2x3_fwd_tc.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, i, vp]
    L.wino_filter_workspace_bytes_tc.restype = st
    L.wino_filter_workspace_bytes_tc.argtypes = [i, i, i]
    L.wino_filter_transform_tc.restype = i
    L.wino_filter_transform_tc.argtypes = [vp, vp, i, i, i, vp]
    L.wino_host_workspace_bytes.restype = st
    L.wino_host_workspace_bytes.argtypes = [i, i, i, i, i]
    L.wino_conv2d_f2x3_fwd_host.restype = i
    L.wino_conv2d_f2x3_fwd_host.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, vp, st, vp]
    L.wino_host_multi_workspace_bytes.restype = st
    L.wino_host_multi_workspace_bytes.argtypes = [ctypes.POINTER(_HostLayer), i]
    L.wino_conv2d_f2x3_fwd_host_multi.restype = i
    L.wino_conv2d_f2x3_fwd_host_multi.argtypes = [ctypes.POINTER(_HostLayer), i, vp, st, vp]
    L.wino_filter_workspace_bytes_f4.restype = st
    L.wino_filter_workspace_bytes_f4.argtypes = [i, i]
    L.wino_filter_transform_f4.restype = i
    L.wino_filter_transform_f4.argtypes = [vp, vp, i, i, vp]
    L.wino_conv2d_f4x3_fwd.restype = i
    L.wino_conv2d_f4x3_fwd.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, vp]
    if hasattr(L, "wino_conv2d_f4x3_fwd_ws") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_f4_workspace_bytes.restype = st
        L.wino_f4_workspace_bytes.argtypes = [i, i, i, i, i]
        L.wino_conv2d_f4x3_fwd_ws.restype = i
        L.wino_conv2d_f4x3_fwd_ws.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, i, vp, st, vp]
    if hasattr(L, "wino_conv2d_f2x3_fwd_half") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_filter_workspace_bytes_half.restype = st
        L.wino_filter_workspace_bytes_half.argtypes = [i, i]
        L.wino_filter_transform_half.restype = i
        L.wino_filter_transform_half.argtypes = [vp, vp, i, i, i, vp]
        L.wino_conv2d_f2x3_fwd_half.restype = i
        L.wino_conv2d_f2x3_fwd_half.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, i, vp]
    if hasattr(L, "wino_conv2d_f2x3_fwd_tc_ws") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_tc_workspace_bytes.restype = st
        L.wino_tc_workspace_bytes.argtypes = [i, i, i, i, i]
        L.wino_conv2d_f2x3_fwd_tc_ws.restype = i
        L.wino_conv2d_f2x3_fwd_tc_ws.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, i, i, vp, st, vp]
    if hasattr(L, "wino_conv2d_f2x3_fwd_half_ws") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_half_workspace_bytes.restype = st
        L.wino_half_workspace_bytes.argtypes = [i, i, i, i, i]
        L.wino_conv2d_f2x3_fwd_half_ws.restype = i
        L.wino_conv2d_f2x3_fwd_half_ws.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, i, i, vp, st, vp]
    if hasattr(L, "wino_conv2d_f2x3_fwd_ws") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_conv_workspace_bytes.restype = st
        L.wino_conv_workspace_bytes.argtypes = [i, i, i, i, i]
        L.wino_conv2d_f2x3_fwd_ws.restype = i
        L.wino_conv2d_f2x3_fwd_ws.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, i, vp, st, vp]
    if hasattr(L, "wino_conv2d_f2x3_fwd_multi") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_conv_multi_workspace_bytes.restype = st
        L.wino_conv_multi_workspace_bytes.argtypes = [ctypes.POINTER(_ConvJob), i]
        L.wino_conv_multi_launches.restype = i
        L.wino_conv_multi_launches.argtypes = [ctypes.POINTER(_ConvJob), i]
        L.wino_conv2d_f2x3_fwd_multi.restype = i
        L.wino_conv2d_f2x3_fwd_multi.argtypes = [ctypes.POINTER(_ConvJob), i, vp, st, vp, vp]
    if hasattr(L, "wino_conv2d_f2x3_fwd_nchw_ws") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_nchw_workspace_bytes.restype = st
        L.wino_nchw_workspace_bytes.argtypes = [i, i, i, i, i]
        L.wino_conv2d_f2x3_fwd_nchw_ws.restype = i
        L.wino_conv2d_f2x3_fwd_nchw_ws.argtypes = [vp, vp, vp, i, i, i, i, i, i, i, vp, st, vp]
    if hasattr(L, "wino_filter_transform_multi") or not os.environ.get("WINO_LIB_PATH"):
        L.wino_filter_transform_multi.restype = i
        L.wino_filter_transform_multi.argtypes = [ctypes.c_void_p, i, vp]
    L.wino_plan.restype = i
    L.wino_plan.argtypes = [i, i, i, i, i, i, ctypes.POINTER(_Plan)]
    _lib = L
    return L


def _check(status: int, where: str):
    if status != 0:
        raise WinoError(status, where, lib().wino_last_cuda_error() if status == 5 else 0)


def version() -> int:
    return lib().wino_version()


def _stream_ptr(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _need_cuda_f32(t: torch.Tensor, name: str, ndim: int):
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name} must be a torch.Tensor")
    if t.dtype != torch.float32:
        raise TypeError(f"{name} must be float32, got {t.dtype}")
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor (no CPU fallback)")
    if t.dim() != ndim:
        raise ValueError(f"{name} must have {ndim} dims, got shape {tuple(t.shape)}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")

def _same_device(ref: torch.Tensor, **tensors):
    """Every tensor the library touches in one call must live on ref's device (a pointer into
    another GPU's memory would fault inside the kernel and kill the CUDA context)."""
    for name, t in tensors.items():
        if t is None:
            continue
        if not t.is_cuda or t.device != ref.device:
            raise ValueError(f"{name} must be on {ref.device}, got {t.device}")


def _need_ws(ws: torch.Tensor | None, ref: torch.Tensor):
    """A workspace is a contiguous CUDA byte buffer on ref's device."""
    if ws is None:
        return
    if not isinstance(ws, torch.Tensor) or not ws.is_cuda:
        raise ValueError("ws must be a CUDA tensor")
    if not ws.is_contiguous():
        raise ValueError("ws must be contiguous")
    _same_device(ref, ws=ws)


def filter_workspace_bytes(C: int, K: int) -> int:
    """16*C*K*4 bytes (L993)."""
    return int(lib().wino_filter_workspace_bytes(C, K))


def host_workspace_bytes(N: int, C: int, H: int, W: int, K: int) -> int:
    return int(lib().wino_host_workspace_bytes(N, C, H, W, K))


def plan(N: int, C: int, H: int, W: int, K: int, variant: int = 0) -> Plan:
    p = _Plan()
    _check(lib().wino_plan(N, C, H, W, K, variant, ctypes.byref(p)), "wino_plan")
    return Plan(**{f: getattr(p, f) for f, _ in _Plan._fields_})


def filter_transform(w: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """FTF, Eq. 5 (L191): w (C,3,3,K) -> u (C,4,4,K) on the GPU."""
    _need_cuda_f32(w, "w", 4)
    C, r, s, K = w.shape
    if (r, s) != (3, 3):
        raise ValueError(f"w must be (C,3,3,K), got {tuple(w.shape)}")
    if out is None:
        out = torch.empty((C, 4, 4, K), dtype=torch.float32, device=w.device)
    _need_cuda_f32(out, "out", 4)
    if tuple(out.shape) != (C, 4, 4, K):
        raise ValueError("out must be (C,4,4,K)")
    _same_device(w, out=out)
    with torch.cuda.device(w.device):
        _check(lib().wino_filter_transform(ctypes.c_void_p(w.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                           C, K, _stream_ptr(stream)), "wino_filter_transform")
    return out


class _FtfJob(ctypes.Structure):
    _fields_ = [("w", ctypes.c_void_p), ("u", ctypes.c_void_p), ("C", ctypes.c_int), ("K", ctypes.c_int)]


def filter_transform_multi(pairs, stream=None) -> None:
    """Several FTFs (Eq. 5) in one launch (wino_filter_transform_multi): pairs = [(w (C,3,3,K), u (C,4,4,K))]."""
    jobs = (_FtfJob * len(pairs))()
    for j, (w, u) in enumerate(pairs):
        _need_cuda_f32(w, "w", 4)
        _need_cuda_f32(u, "u", 4)
        C, r, s_, K = w.shape
        if (r, s_) != (3, 3) or tuple(u.shape) != (C, 4, 4, K):
            raise ValueError(f"job {j}: w must be (C,3,3,K) and u (C,4,4,K)")
        _same_device(pairs[0][0], w=w, u=u)
        jobs[j] = _FtfJob(w.data_ptr(), u.data_ptr(), C, K)
    with torch.cuda.device(pairs[0][0].device):
        _check(lib().wino_filter_transform_multi(jobs, len(pairs), _stream_ptr(stream)), "wino_filter_transform_multi")


@dataclass
class TcFilter:
    """Transformed filter in the tensor-core operand layout (wino_filter_transform_tc)."""
    data: torch.Tensor  # flat float32 CUDA tensor, wino_filter_workspace_bytes_tc bytes
    C: int
    K: int
    mode: int  # TC_TF32 or TC_3XTF32


def _tc_mode(variant) -> int:
    if variant in ("tf32", TC_TF32):
        return TC_TF32
    if variant in ("3xtf32", TC_3XTF32):
        return TC_3XTF32
    raise ValueError(f"unknown tensor-core variant {variant!r}")


def filter_workspace_bytes_tc(C: int, K: int, variant="tf32") -> int:
    return int(lib().wino_filter_workspace_bytes_tc(C, K, _tc_mode(variant)))


def filter_transform_tc(w: torch.Tensor, variant="tf32", out: TcFilter | None = None, stream=None) -> TcFilter:
    """FTF (Eq. 5) into the tcgen05 operand layout, TF32-rounded (3xTF32: + residual plane)."""
    _need_cuda_f32(w, "w", 4)
    C, r, s_, K = w.shape
    if (r, s_) != (3, 3):
        raise ValueError(f"w must be (C,3,3,K), got {tuple(w.shape)}")
    mode = _tc_mode(variant)
    nbytes = filter_workspace_bytes_tc(C, K, mode)
    if out is None:
        out = TcFilter(torch.empty(nbytes // 4, dtype=torch.float32, device=w.device), C, K, mode)
    if (out.C, out.K, out.mode) != (C, K, mode) or out.data.numel() * 4 < nbytes:
        raise ValueError("out TcFilter does not match w / variant")
    _need_cuda_f32(out.data, "out.data", out.data.dim())
    _same_device(w, out=out.data)
    with torch.cuda.device(w.device):
        _check(lib().wino_filter_transform_tc(ctypes.c_void_p(w.data_ptr()), ctypes.c_void_p(out.data.data_ptr()),
                                              C, K, mode, _stream_ptr(stream)), "wino_filter_transform_tc")
    return out


def tc_workspace_bytes(N: int, C: int, H: int, W: int, K: int) -> int:
    """Device workspace that lets ``conv2d_tc`` use the stream-K plan (wino_tc_workspace_bytes)."""
    return int(lib().wino_tc_workspace_bytes(N, C, H, W, K))


def conv2d_tc(x: torch.Tensor, u_tc: TcFilter, out: torch.Tensor | None = None, stream=None,
              ws: torch.Tensor | None = None, stream_k: str = "auto") -> torch.Tensor:
    """Fused Winograd conv with the Winograd-domain GEMM on tcgen05 (TF32 / 3xTF32).  ws (>=
    tc_workspace_bytes) enables the stream-K plan (wino_conv2d_f2x3_fwd_tc_ws)."""
    _need_cuda_f32(x, "x", 4)
    C, H, W, N = x.shape
    if u_tc.C != C:
        raise ValueError(f"u_tc was built for C={u_tc.C}, x has C={C}")
    K = u_tc.K
    if out is None:
        out = torch.empty((K, H, W, N), dtype=torch.float32, device=x.device)
    _need_cuda_f32(out, "out", 4)
    if tuple(out.shape) != (K, H, W, N):
        raise ValueError("out must be (K,H,W,N)")
    _need_cuda_f32(u_tc.data, "u_tc.data", u_tc.data.dim())
    _same_device(x, u_tc=u_tc.data, out=out)
    _need_ws(ws, x)
    args = (ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(u_tc.data.data_ptr()), ctypes.c_void_p(out.data_ptr()),
            N, C, H, W, K, 1, 1, u_tc.mode)
    with torch.cuda.device(x.device):
        if ws is not None or stream_k == "on":
            wp, wb = (ctypes.c_void_p(ws.data_ptr()), ws.numel() * ws.element_size()) if ws is not None else (None, 0)
            _check(lib().wino_conv2d_f2x3_fwd_tc_ws(*args, {"auto": 0, "off": 1, "on": 2}[stream_k], wp, wb,
                                                    _stream_ptr(stream)), "wino_conv2d_f2x3_fwd_tc_ws")
        else:
            _check(lib().wino_conv2d_f2x3_fwd_tc(*args, _stream_ptr(stream)), "wino_conv2d_f2x3_fwd_tc")
    return out


def _need_cuda_half(t: torch.Tensor, name: str, ndim: int):
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name} must be a torch.Tensor")
    if t.dtype not in _HALF_DTYPES:
        raise TypeError(f"{name} must be float16 or bfloat16, got {t.dtype}")
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor (no CPU fallback)")
    if t.dim() != ndim:
        raise ValueError(f"{name} must have {ndim} dims, got shape {tuple(t.shape)}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")


@dataclass
class HalfFilter:
    """Transformed filter in the kind::f16 operand layout (wino_filter_transform_half)."""
    data: torch.Tensor  # flat 16-bit CUDA tensor of the filter's dtype
    C: int
    K: int
    dtype: torch.dtype


def filter_workspace_bytes_half(C: int, K: int) -> int:
    return int(lib().wino_filter_workspace_bytes_half(C, K))


def filter_transform_half(w: torch.Tensor, out: HalfFilter | None = None, stream=None) -> HalfFilter:
    """NEXT row N4: FTF (Eq. 5) of a float16 / bfloat16 w (C,3,3,K) in FP32, rounded to w's type, in the
    tcgen05 kind::f16 operand layout (Sec. 8.3)."""
    _need_cuda_half(w, "w", 4)
    C, r, s_, K = w.shape
    if (r, s_) != (3, 3):
        raise ValueError(f"w must be (C,3,3,K), got {tuple(w.shape)}")
    nbytes = filter_workspace_bytes_half(C, K)
    if out is None:
        out = HalfFilter(torch.empty(nbytes // 2, dtype=w.dtype, device=w.device), C, K, w.dtype)
    if (out.C, out.K, out.dtype) != (C, K, w.dtype) or out.data.numel() * 2 < nbytes:
        raise ValueError("out HalfFilter does not match w")
    _need_cuda_half(out.data, "out.data", out.data.dim())
    _same_device(w, out=out.data)
    with torch.cuda.device(w.device):
        _check(lib().wino_filter_transform_half(ctypes.c_void_p(w.data_ptr()), ctypes.c_void_p(out.data.data_ptr()),
                                                C, K, _HALF_DTYPES[w.dtype], _stream_ptr(stream)),
               "wino_filter_transform_half")
    return out


def half_workspace_bytes(N: int, C: int, H: int, W: int, K: int) -> int:
    """Device workspace that lets ``conv2d_half`` use the stream-K plan (wino_half_workspace_bytes)."""
    return int(lib().wino_half_workspace_bytes(N, C, H, W, K))


def conv2d_half(x: torch.Tensor, u_h: HalfFilter, out: torch.Tensor | None = None, stream=None,
                ws: torch.Tensor | None = None, stream_k: str = "auto") -> torch.Tensor:
    """NEXT row N4: fused Winograd conv on float16 / bfloat16 x (C,H,W,N) -> y (K,H,W,N) of the same type,
    Winograd-domain GEMM on tcgen05 kind::f16 with FP32 accumulation.  ws (>= half_workspace_bytes)
    enables the stream-K plan (wino_conv2d_f2x3_fwd_half_ws): stream_k "auto" / "off" / "on"."""
    _need_cuda_half(x, "x", 4)
    C, H, W, N = x.shape
    if u_h.C != C or u_h.dtype != x.dtype:
        raise ValueError(f"u_h was built for C={u_h.C} {u_h.dtype}, x has C={C} {x.dtype}")
    K = u_h.K
    if out is None:
        out = torch.empty((K, H, W, N), dtype=x.dtype, device=x.device)
    _need_cuda_half(out, "out", 4)
    if tuple(out.shape) != (K, H, W, N) or out.dtype != x.dtype:
        raise ValueError("out must be (K,H,W,N) of x's dtype")
    _need_cuda_half(u_h.data, "u_h.data", u_h.data.dim())
    _same_device(x, u_h=u_h.data, out=out)
    _need_ws(ws, x)
    args = (ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(u_h.data.data_ptr()), ctypes.c_void_p(out.data_ptr()),
            N, C, H, W, K, 1, 1, _HALF_DTYPES[x.dtype])
    with torch.cuda.device(x.device):
        if ws is not None or stream_k == "on":
            wp, wb = (ctypes.c_void_p(ws.data_ptr()), ws.numel() * ws.element_size()) if ws is not None else (None, 0)
            _check(lib().wino_conv2d_f2x3_fwd_half_ws(*args, {"auto": 0, "off": 1, "on": 2}[stream_k], wp, wb,
                                                      _stream_ptr(stream)), "wino_conv2d_f2x3_fwd_half_ws")
        else:
            _check(lib().wino_conv2d_f2x3_fwd_half(*args, _stream_ptr(stream)), "wino_conv2d_f2x3_fwd_half")
    return out


def conv_workspace_bytes(N: int, C: int, H: int, W: int, K: int) -> int:
    """Device workspace that lets ``conv2d`` use the stream-K plan (wino_conv_workspace_bytes)."""
    return int(lib().wino_conv_workspace_bytes(N, C, H, W, K))


def conv2d(x: torch.Tensor, u: torch.Tensor, out: torch.Tensor | None = None, variant: str = "fp32",
           stream=None, split_c: int = 0, ws: torch.Tensor | None = None, stream_k: str = "auto") -> torch.Tensor:
    """Fused Winograd forward conv on FP32 CUDA cores, pad 1 stride 1:
    x (C,H,W,N), u (C,4,4,K) -> y (K,H,W,N).  split_c: 0 = the library's choice, else
    force the split-C factor (1, 2, 4, 8) of the warp-specialised kernel
    (``wino_conv2d_f2x3_fwd_split``).  ws: a device workspace of >= conv_workspace_bytes
    bytes enables the stream-K plan (``wino_conv2d_f2x3_fwd_ws``); stream_k = "auto"
    (planner's choice), "off" or "on"."""
    _need_cuda_f32(x, "x", 4)
    _need_cuda_f32(u, "u", 4)
    C, H, W, N = x.shape
    if u.shape[0] != C or tuple(u.shape[1:3]) != (4, 4):
        raise ValueError(f"u must be (C,4,4,K) with C={C}, got {tuple(u.shape)}")
    if u.device != x.device:
        raise ValueError("x and u must be on the same device")
    K = u.shape[3]
    if out is None:
        out = torch.empty((K, H, W, N), dtype=torch.float32, device=x.device)
    _need_cuda_f32(out, "out", 4)
    if tuple(out.shape) != (K, H, W, N):
        raise ValueError("out must be (K,H,W,N)")
    _same_device(x, u=u, out=out)
    _need_ws(ws, x)
    args = (ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(u.data_ptr()), ctypes.c_void_p(out.data_ptr()),
            N, C, H, W, K, 1, 1)
    with torch.cuda.device(x.device):
        if variant != "fp32":
            raise ValueError(f"conv2d runs the FP32 kernel; use conv2d_tc for {variant!r}")
        if ws is not None or stream_k == "on":
            if split_c:
                raise ValueError("split_c and a stream-K workspace are exclusive")
            mode = {"auto": 0, "off": 1, "on": 2}[stream_k]
            wp, wb = (ctypes.c_void_p(ws.data_ptr()), ws.numel() * ws.element_size()) if ws is not None else (None, 0)
            _check(lib().wino_conv2d_f2x3_fwd_ws(*args, mode, wp, wb, _stream_ptr(stream)), "wino_conv2d_f2x3_fwd_ws")
        elif split_c:
            _check(lib().wino_conv2d_f2x3_fwd_split(*args, int(split_c), _stream_ptr(stream)),
                   "wino_conv2d_f2x3_fwd_split")
        else:
            _check(lib().wino_conv2d_f2x3_fwd(*args, _stream_ptr(stream)), "wino_conv2d_f2x3_fwd")
    return out


def _conv_jobs(layers):
    arr = (_ConvJob * len(layers))()
    for i, (x, u, y) in enumerate(layers):
        _need_cuda_f32(x, f"layer {i} x", 4)
        _need_cuda_f32(u, f"layer {i} u", 4)
        _need_cuda_f32(y, f"layer {i} y", 4)
        _same_device(layers[0][0], x=x, u=u, y=y)
        C, H, W, N = x.shape
        K = u.shape[3]
        if tuple(u.shape) != (C, 4, 4, K) or tuple(y.shape) != (K, H, W, N):
            raise ValueError(f"layer {i}: x (C,H,W,N), u (C,4,4,K), y (K,H,W,N) expected")
        arr[i] = _ConvJob(x.data_ptr(), u.data_ptr(), y.data_ptr(), N, C, H, W, K)
    return arr


def conv_multi_workspace_bytes(shapes) -> int:
    """Workspace of conv2d_multi for [(N, C, H, W, K), ...] (wino_conv_multi_workspace_bytes)."""
    arr = (_ConvJob * len(shapes))()
    for i, (N, C, H, W, K) in enumerate(shapes):
        arr[i] = _ConvJob(None, None, None, N, C, H, W, K)
    return int(lib().wino_conv_multi_workspace_bytes(arr, len(shapes)))


def conv_multi_launches(shapes) -> int:
    """Kernel launches of one conv2d_multi call on [(N, C, H, W, K), ...] (wino_conv_multi_launches)."""
    arr = (_ConvJob * len(shapes))()
    for i, (N, C, H, W, K) in enumerate(shapes):
        arr[i] = _ConvJob(None, None, None, N, C, H, W, K)
    n = int(lib().wino_conv_multi_launches(arr, len(shapes)))
    if n < 0:
        raise WinoError(1, f"wino_conv_multi_launches {shapes}")
    return n


def conv2d_multi(layers, ws: torch.Tensor, stream=None, u_ready: torch.cuda.Event | None = None) -> None:
    """Several independent layers [(x (C,H,W,N), u (C,4,4,K), y (K,H,W,N)), ...]: the layers with
    fewer than 64 tiles per SM share one persistent stream-K launch of the warp-specialised FP32
    kernel per group of <= 4, the others run alone through the planner (wino_conv2d_f2x3_fwd_multi).
    ws: a ZERO-FILLED CUDA byte buffer of >= conv_multi_workspace_bytes (calls leave it zeroed).
    u_ready: an event the convolutions wait for (the x-only input transforms of N = 4 / 8 layers
    are queued before the wait), e.g. recorded after filter_transform_multi on another stream."""
    arr = _conv_jobs(layers)
    _need_ws(ws, layers[0][0])
    ev = ctypes.c_void_p(u_ready.cuda_event) if u_ready is not None else None
    with torch.cuda.device(layers[0][0].device):
        _check(lib().wino_conv2d_f2x3_fwd_multi(arr, len(layers), ctypes.c_void_p(ws.data_ptr()),
                                                ws.numel() * ws.element_size(), ev, _stream_ptr(stream)),
               "wino_conv2d_f2x3_fwd_multi")


def filter_transform_kcrs(w_kcrs: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """NEXT row N2 (Sec. 8.4): FTF from PyTorch's conv weight layout w (K,C,3,3) -> u (C,4,4,K)."""
    _need_cuda_f32(w_kcrs, "w_kcrs", 4)
    K, C, r, s = w_kcrs.shape
    if (r, s) != (3, 3):
        raise ValueError(f"w_kcrs must be (K,C,3,3), got {tuple(w_kcrs.shape)}")
    if out is None:
        out = torch.empty((C, 4, 4, K), dtype=torch.float32, device=w_kcrs.device)
    _need_cuda_f32(out, "out", 4)
    if tuple(out.shape) != (C, 4, 4, K):
        raise ValueError("out must be (C,4,4,K)")
    _same_device(w_kcrs, out=out)
    with torch.cuda.device(w_kcrs.device):
        _check(lib().wino_filter_transform_kcrs(ctypes.c_void_p(w_kcrs.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                                C, K, _stream_ptr(stream)), "wino_filter_transform_kcrs")
    return out


def nchw_workspace_bytes(N: int, C: int, H: int, W: int, K: int) -> int:
    """Device workspace of the transpose + CHWN-kernel NCHW path (wino_nchw_workspace_bytes)."""
    return int(lib().wino_nchw_workspace_bytes(N, C, H, W, K))


def conv2d_nchw(x: torch.Tensor, u: torch.Tensor, out: torch.Tensor | None = None, stream=None,
                ws: torch.Tensor | None = None) -> torch.Tensor:
    """NEXT row N2 (Sec. 8.4): fused Winograd conv on NCHW tensors, pad 1 stride 1:
    x (N,C,H,W), u (C,4,4,K) -> y (N,K,H,W) -- torch.nn.functional.conv2d(x, w, padding=1)
    with u = filter_transform_kcrs(w).  ws (>= nchw_workspace_bytes): transpose to CHWN, the
    CHWN fused kernel, transpose back (wino_conv2d_f2x3_fwd_nchw_ws); else the strided kernel."""
    _need_cuda_f32(x, "x", 4)
    _need_cuda_f32(u, "u", 4)
    N, C, H, W = x.shape
    if u.shape[0] != C or tuple(u.shape[1:3]) != (4, 4):
        raise ValueError(f"u must be (C,4,4,K) with C={C}, got {tuple(u.shape)}")
    if u.device != x.device:
        raise ValueError("x and u must be on the same device")
    K = u.shape[3]
    if out is None:
        out = torch.empty((N, K, H, W), dtype=torch.float32, device=x.device)
    _need_cuda_f32(out, "out", 4)
    if tuple(out.shape) != (N, K, H, W):
        raise ValueError("out must be (N,K,H,W)")
    _same_device(x, u=u, out=out)
    _need_ws(ws, x)
    with torch.cuda.device(x.device):
        if ws is not None:
            _check(lib().wino_conv2d_f2x3_fwd_nchw_ws(
                ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(u.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                N, C, H, W, K, 1, 1, ctypes.c_void_p(ws.data_ptr()), ws.numel() * ws.element_size(),
                _stream_ptr(stream)), "wino_conv2d_f2x3_fwd_nchw_ws")
        else:
            _check(lib().wino_conv2d_f2x3_fwd_nchw(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(u.data_ptr()),
                                                   ctypes.c_void_p(out.data_ptr()), N, C, H, W, K, 1, 1,
                                                   _stream_ptr(stream)), "wino_conv2d_f2x3_fwd_nchw")
    return out


def nonfused_workspace_bytes(N: int, C: int, H: int, W: int, K: int) -> int:
    """Device workspace of the non-fused path: V[16][C][NV] + M[16][K][NV] floats."""
    return int(lib().wino_nonfused_workspace_bytes(N, C, H, W, K))


def nonfused_launches() -> int:
    """Kernels one conv2d_nonfused call launches (u arrangement, ITF, GEMM, OTF)."""
    return int(lib().wino_nonfused_launches())


def conv2d_nonfused(x: torch.Tensor, u: torch.Tensor, ws: torch.Tensor, out: torch.Tensor | None = None,
                    stream=None, tf32: bool = False) -> torch.Tensor:
    """NEXT row N3 (Sec. 9): NON-fused Winograd -- ITF kernel to a global workspace,
    16 batched GEMMs on the tcgen05 tensor cores (this library's kernel: 3xTF32, FP32-level accuracy;
    tf32=True: plain TF32), OTF kernel (4 launches, nonfused_launches()).
    x (C,H,W,N), u (C,4,4,K) -> y (K,H,W,N); ws: CUDA byte buffer of >= nonfused_workspace_bytes."""
    _need_cuda_f32(x, "x", 4)
    _need_cuda_f32(u, "u", 4)
    C, H, W, N = x.shape
    if u.shape[0] != C or tuple(u.shape[1:3]) != (4, 4):
        raise ValueError(f"u must be (C,4,4,K) with C={C}, got {tuple(u.shape)}")
    K = u.shape[3]
    _need_ws(ws, x)
    if out is None:
        out = torch.empty((K, H, W, N), dtype=torch.float32, device=x.device)
    _need_cuda_f32(out, "out", 4)
    if tuple(out.shape) != (K, H, W, N):
        raise ValueError("out must be (K,H,W,N)")
    _same_device(x, u=u, out=out)
    fn = "wino_conv2d_f2x3_fwd_nonfused_tf32" if tf32 else "wino_conv2d_f2x3_fwd_nonfused"
    with torch.cuda.device(x.device):
        _check(getattr(lib(), fn)(
            ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(u.data_ptr()), ctypes.c_void_p(out.data_ptr()),
            N, C, H, W, K, 1, 1, ctypes.c_void_p(ws.data_ptr()), ws.numel() * ws.element_size(),
            _stream_ptr(stream)), fn)
    return out


def filter_workspace_bytes_f4(C: int, K: int) -> int:
    return int(lib().wino_filter_workspace_bytes_f4(C, K))


def filter_transform_f4(w: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """NEXT row N1: F(4x4,3x3) filter transform w (C,3,3,K) -> u4 (C,6,6,K) on the GPU."""
    _need_cuda_f32(w, "w", 4)
    C, r, s, K = w.shape
    if (r, s) != (3, 3):
        raise ValueError(f"w must be (C,3,3,K), got {tuple(w.shape)}")
    if out is None:
        out = torch.empty((C, 6, 6, K), dtype=torch.float32, device=w.device)
    _need_cuda_f32(out, "out", 4)
    if tuple(out.shape) != (C, 6, 6, K):
        raise ValueError("out must be (C,6,6,K)")
    _same_device(w, out=out)
    with torch.cuda.device(w.device):
        _check(lib().wino_filter_transform_f4(ctypes.c_void_p(w.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                              C, K, _stream_ptr(stream)), "wino_filter_transform_f4")
    return out


def f4_workspace_bytes(N: int, C: int, H: int, W: int, K: int) -> int:
    """Device workspace that lets ``conv2d_f4`` use the stream-K plan (wino_f4_workspace_bytes)."""
    return int(lib().wino_f4_workspace_bytes(N, C, H, W, K))


def conv2d_f4(x: torch.Tensor, u4: torch.Tensor, out: torch.Tensor | None = None, stream=None,
              ws: torch.Tensor | None = None, stream_k: str = "auto") -> torch.Tensor:
    """NEXT row N1: fused Winograd F(4x4,3x3) forward conv (FP32), pad 1 stride 1:
    x (C,H,W,N), u4 (C,6,6,K) -> y (K,H,W,N); any shape (N % 16 == 0 and K % 4 == 0: TMA path,
    else a cp.async gather path).  ws (>=
    f4_workspace_bytes) enables the stream-K plan (wino_conv2d_f4x3_fwd_ws)."""
    _need_cuda_f32(x, "x", 4)
    _need_cuda_f32(u4, "u4", 4)
    C, H, W, N = x.shape
    if u4.shape[0] != C or tuple(u4.shape[1:3]) != (6, 6):
        raise ValueError(f"u4 must be (C,6,6,K) with C={C}, got {tuple(u4.shape)}")
    if u4.device != x.device:
        raise ValueError("x and u4 must be on the same device")
    K = u4.shape[3]
    if out is None:
        out = torch.empty((K, H, W, N), dtype=torch.float32, device=x.device)
    _need_cuda_f32(out, "out", 4)
    if tuple(out.shape) != (K, H, W, N):
        raise ValueError("out must be (K,H,W,N)")
    _same_device(x, u4=u4, out=out)
    _need_ws(ws, x)
    args = (ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(u4.data_ptr()), ctypes.c_void_p(out.data_ptr()),
            N, C, H, W, K, 1, 1)
    with torch.cuda.device(x.device):
        if ws is not None or stream_k == "on":
            wp, wb = (ctypes.c_void_p(ws.data_ptr()), ws.numel() * ws.element_size()) if ws is not None else (None, 0)
            _check(lib().wino_conv2d_f4x3_fwd_ws(*args, {"auto": 0, "off": 1, "on": 2}[stream_k], wp, wb,
                                                 _stream_ptr(stream)), "wino_conv2d_f4x3_fwd_ws")
        else:
            _check(lib().wino_conv2d_f4x3_fwd(*args, _stream_ptr(stream)), "wino_conv2d_f4x3_fwd")
    return out


def conv2d_host(x_host: torch.Tensor, w_host: torch.Tensor, y_host: torch.Tensor, ws: torch.Tensor,
                stream=None) -> None:
    """End-to-end call on host buffers (x (C,H,W,N), w (C,3,3,K) -> y (K,H,W,N), pinned CPU
    fp32) through ``wino_conv2d_f2x3_fwd_host``; ``ws`` is a CUDA byte buffer of at least
    host_workspace_bytes().  Asynchronous on the stream."""
    for t, n in ((x_host, "x_host"), (w_host, "w_host"), (y_host, "y_host")):
        if t.is_cuda or t.dtype != torch.float32 or not t.is_contiguous() or t.dim() != 4:
            raise ValueError(f"{n} must be a contiguous 4-d float32 CPU tensor")
    _need_ws(ws, ws)
    C, H, W, N = x_host.shape
    K = w_host.shape[3]
    if tuple(y_host.shape) != (K, H, W, N) or tuple(w_host.shape) != (C, 3, 3, K):
        raise ValueError("shape mismatch")
    nbytes = ws.numel() * ws.element_size()
    with torch.cuda.device(ws.device):
        _check(lib().wino_conv2d_f2x3_fwd_host(
            ctypes.c_void_p(x_host.data_ptr()), ctypes.c_void_p(w_host.data_ptr()),
            ctypes.c_void_p(y_host.data_ptr()), N, C, H, W, K, 1, 1,
            ctypes.c_void_p(ws.data_ptr()), nbytes, _stream_ptr(stream)), "wino_conv2d_f2x3_fwd_host")


def _host_layers(layers):
    arr = (_HostLayer * len(layers))()
    for i, (xh, wh, yh) in enumerate(layers):
        for t, n in ((xh, "x_host"), (wh, "w_host"), (yh, "y_host")):
            if t.is_cuda or t.dtype != torch.float32 or not t.is_contiguous() or t.dim() != 4:
                raise ValueError(f"layer {i}: {n} must be a contiguous 4-d float32 CPU tensor")
        C, H, W, N = xh.shape
        K = wh.shape[3]
        if tuple(wh.shape) != (C, 3, 3, K) or tuple(yh.shape) != (K, H, W, N):
            raise ValueError(f"layer {i}: shape mismatch")
        arr[i] = _HostLayer(xh.data_ptr(), wh.data_ptr(), yh.data_ptr(), N, C, H, W, K)
    return arr


def host_multi_workspace_bytes(layers) -> int:
    """Device workspace for conv2d_host_multi over [(x_host, w_host, y_host), ...]."""
    return int(lib().wino_host_multi_workspace_bytes(_host_layers(layers), len(layers)))


def conv2d_host_multi(layers, ws: torch.Tensor, stream=None) -> None:
    """End-to-end multi-layer call on pinned host buffers with H2D / compute / D2H overlap
    (``wino_conv2d_f2x3_fwd_host_multi``); asynchronous on the stream."""
    arr = _host_layers(layers)
    _need_ws(ws, ws)
    with torch.cuda.device(ws.device):
        _check(lib().wino_conv2d_f2x3_fwd_host_multi(arr, len(layers), ctypes.c_void_p(ws.data_ptr()),
                                                     ws.numel() * ws.element_size(), _stream_ptr(stream)),
               "wino_conv2d_f2x3_fwd_host_multi")
