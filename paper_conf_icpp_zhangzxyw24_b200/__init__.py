"""Python binding of the i2cw C ABI (include/i2cw.h) — argument marshalling only.

Every step of the hot path (filter transform, input transform, tcgen05 3xTF32
contraction, output transform) runs in libi2cw.so's CUDA kernels. There is no
CPU fallback: if the extension is missing, or a call fails, this raises.

Tensors: fp32, contiguous, on a CUDA device (except the *_host call).
  conv2d_nhwc(x [N,H,W,C], w [K,R,S,C], pad_h, pad_w) -> y [N,P,Q,K]
  deconv2d_nhwc(x [N,H,W,C], w [C,R,S,K], pad_h, pad_w) -> y [N,P,Q,K]
"""
from __future__ import annotations

import ctypes
import os
from fractions import Fraction

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("I2CW_LIB_EXPERIMENT") or os.path.join(_HERE, "libi2cw.so")  # override: timing experiments only
_lib = None

I2CW_OK, I2CW_EINVAL, I2CW_EUNSUPPORTED, I2CW_ECUDA = 0, -1, -2, -3

#: every symbol include/i2cw.h declares (checked by tests/test_abi.py)
PUBLIC_SYMBOLS = (
    "i2cw_status_string", "i2cw_version", "i2cw_conv2d_nhwc", "i2cw_deconv2d_nhwc", "i2cw_filter_bytes",
    "i2cw_filter_transform", "i2cw_conv2d_nhwc_pretransformed", "i2cw_deconv2d_nhwc_pretransformed",
    "i2cw_conv2d_nhwc_host", "i2cw_set_device", "i2cw_plan", "i2cw_transform_matrices_rational",
    "i2cw_conv3d_ndhwc", "i2cw_deconv3d_ndhwc", "i2cw_conv2d_nchw", "i2cw_deconv2d_nchw",
    "i2cw_conv2d_nhwc_prec",
)

#: precision modes of i2cw_conv2d_nhwc_prec (include/i2cw.h)
PRECISIONS = {"3xtf32": 0, "1xtf32": 1}
#: per-element tolerance (x sum|x||w|) each precision mode guarantees
TOLERANCE = {"3xtf32": 1e-4, "1xtf32": 1e-2}


class I2CWError(RuntimeError):
    def __init__(self, fn, status):
        super().__init__(f"{fn} failed: {status} ({status_string(status)})")
        self.status = status


def lib():
    """Load libi2cw.so (built by __graft_entry__.build() / `make -C paper_conf_icpp_zhangzxyw24_b200`)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built; run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(LIB_PATH)
        I, P, S = ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t
        L.i2cw_status_string.argtypes = [I]
        L.i2cw_status_string.restype = ctypes.c_char_p
        L.i2cw_version.restype = I
        for name in ("i2cw_conv2d_nhwc", "i2cw_deconv2d_nhwc", "i2cw_conv2d_nhwc_pretransformed",
                     "i2cw_deconv2d_nhwc_pretransformed"):
            f = getattr(L, name)
            f.argtypes = [I] * 9 + [P, P, P, P]
            f.restype = I
        L.i2cw_conv2d_nhwc_prec.argtypes = [I] * 11 + [P, P, P, P]
        L.i2cw_conv2d_nhwc_prec.restype = I
        for name in ("i2cw_conv2d_nchw", "i2cw_deconv2d_nchw"):
            f = getattr(L, name)
            f.argtypes = [I] * 9 + [P, P, P, P]
            f.restype = I
        for name in ("i2cw_conv3d_ndhwc", "i2cw_deconv3d_ndhwc"):
            f = getattr(L, name)
            f.argtypes = [I] * 12 + [P, P, P, P]
            f.restype = I
        L.i2cw_filter_bytes.argtypes = [I] * 4
        L.i2cw_filter_bytes.restype = S
        L.i2cw_filter_transform.argtypes = [I] * 5 + [P, P, P]
        L.i2cw_filter_transform.restype = I
        L.i2cw_conv2d_nhwc_host.argtypes = [I] * 10 + [P, P, P, P]
        L.i2cw_conv2d_nhwc_host.restype = I
        L.i2cw_set_device.argtypes = [I]
        L.i2cw_set_device.restype = I
        L.i2cw_plan.argtypes = [I, I, P, P, P]
        L.i2cw_plan.restype = I
        L.i2cw_transform_matrices_rational.argtypes = [I, I, I] + [P] * 6
        L.i2cw_transform_matrices_rational.restype = I
        L.i2cw_debug_conv_simt.argtypes = [I] * 10 + [P, P, P, P]
        L.i2cw_debug_conv_simt.restype = I
        L.i2cw_debug_plan.argtypes = [I] * 10 + [P]
        L.i2cw_debug_plan.restype = I
        if hasattr(L, "i2cw_debug_set_kchunk"):  # test hook (absent from older experiment builds)
            L.i2cw_debug_set_kchunk.argtypes = [I]
            L.i2cw_debug_set_kchunk.restype = I
        if hasattr(L, "i2cw_debug_set_kslices"):
            L.i2cw_debug_set_kslices.argtypes = [I]
            L.i2cw_debug_set_kslices.restype = I
        _lib = L
    return _lib


def status_string(status: int) -> str:
    return lib().i2cw_status_string(status).decode()


def _check(fn, rc):
    if rc != I2CW_OK:
        raise I2CWError(fn, rc)


def _stream_ptr(stream, like=None):
    """The raw cudaStream_t: the given torch stream, else the current stream of like's device
    (the device the library binds for the call), else of the current device."""
    if stream is not None:
        return stream.cuda_stream
    import torch
    dev = like.get_device() if like is not None else torch.cuda.current_device()
    return torch._C._cuda_getCurrentRawStream(dev)


def _check_tensor(t, name):
    import torch
    if not isinstance(t, torch.Tensor) or t.dtype != torch.float32 or not t.is_cuda or not t.is_contiguous():
        raise ValueError(f"{name} must be a contiguous fp32 CUDA tensor")


def _out(out, shp, like):
    """The output tensor: a new one, or the caller's `out` after checking that the kernels may
    write shp's elements into it (the TMA maps and the zeroing kernel use the plan's sizes)."""
    import torch
    if out is None:
        return torch.empty(shp, dtype=torch.float32, device=like.device)
    _check_tensor(out, "out")
    if tuple(out.shape) != tuple(shp) or out.device != like.device:
        raise ValueError(f"out must have shape {tuple(shp)} on {like.device}, got {tuple(out.shape)} on {out.device}")
    return out


def out_shape(kind, N, H, W, K, R, S, pad_h, pad_w):
    if kind == "conv":
        return (N, H + 2 * pad_h - R + 1, W + 2 * pad_w - S + 1, K)
    return (N, H + R - 1 - 2 * pad_h, W + S - 1 - 2 * pad_w, K)


def conv2d_nhwc(x, w, pad_h, pad_w, out=None, stream=None, precision="3xtf32"):
    """y = conv(x, w) (cross-correlation, zero padding); x [N,H,W,C], w [K,R,S,C] -> y [N,P,Q,K].
    precision: "3xtf32" (fp32 accuracy, default) or "1xtf32" (one tf32 product, TOLERANCE)."""
    _check_tensor(x, "x"); _check_tensor(w, "w")
    N, H, W, C = x.shape
    K, R, S, C2 = w.shape
    if C != C2:
        raise ValueError("channel mismatch")
    if w.device != x.device:
        raise ValueError("x and w must be on the same device")
    y = _out(out, out_shape("conv", N, H, W, K, R, S, pad_h, pad_w), x)
    if precision != "3xtf32":
        _check("i2cw_conv2d_nhwc_prec", lib().i2cw_conv2d_nhwc_prec(
            PRECISIONS[precision], 0, N, H, W, C, K, R, S, pad_h, pad_w, x.data_ptr(), w.data_ptr(), y.data_ptr(),
            _stream_ptr(stream, x)))
        return y
    _check("i2cw_conv2d_nhwc", lib().i2cw_conv2d_nhwc(N, H, W, C, K, R, S, pad_h, pad_w, x.data_ptr(), w.data_ptr(),
                                                      y.data_ptr(), _stream_ptr(stream, x)))
    return y


def deconv2d_nhwc(x, w, pad_h, pad_w, out=None, stream=None, precision="3xtf32"):
    """Transposed conv; x [N,H,W,C], w [C,R,S,K] -> y [N,P,Q,K], P = H+R-1-2 pad_h."""
    _check_tensor(x, "x"); _check_tensor(w, "w")
    N, H, W, C = x.shape
    C2, R, S, K = w.shape
    if C != C2:
        raise ValueError("channel mismatch")
    if w.device != x.device:
        raise ValueError("x and w must be on the same device")
    y = _out(out, out_shape("deconv", N, H, W, K, R, S, pad_h, pad_w), x)
    if precision != "3xtf32":
        _check("i2cw_conv2d_nhwc_prec", lib().i2cw_conv2d_nhwc_prec(
            PRECISIONS[precision], 1, N, H, W, C, K, R, S, pad_h, pad_w, x.data_ptr(), w.data_ptr(), y.data_ptr(),
            _stream_ptr(stream, x)))
        return y
    _check("i2cw_deconv2d_nhwc", lib().i2cw_deconv2d_nhwc(N, H, W, C, K, R, S, pad_h, pad_w, x.data_ptr(),
                                                          w.data_ptr(), y.data_ptr(), _stream_ptr(stream, x)))
    return y


def conv2d_nchw(x, w, pad_h, pad_w, out=None, stream=None):
    """NCHW adapter (f4): x [N,C,H,W], w [K,C,R,S] (PyTorch OIHW) -> y [N,K,P,Q]."""
    _check_tensor(x, "x"); _check_tensor(w, "w")
    N, C, H, W = x.shape
    K, C2, R, S = w.shape
    if C != C2 or w.device != x.device:
        raise ValueError("channel or device mismatch")
    _, P, Q, _ = out_shape("conv", N, H, W, K, R, S, pad_h, pad_w)
    y = _out(out, (N, K, P, Q), x)
    _check("i2cw_conv2d_nchw", lib().i2cw_conv2d_nchw(N, C, H, W, K, R, S, pad_h, pad_w, x.data_ptr(), w.data_ptr(),
                                                      y.data_ptr(), _stream_ptr(stream, x)))
    return y


def deconv2d_nchw(x, w, pad_h, pad_w, out=None, stream=None):
    """NCHW adapter (f4): x [N,C,H,W], w [C,K,R,S] (conv_transpose2d weight) -> y [N,K,P,Q]."""
    _check_tensor(x, "x"); _check_tensor(w, "w")
    N, C, H, W = x.shape
    C2, K, R, S = w.shape
    if C != C2 or w.device != x.device:
        raise ValueError("channel or device mismatch")
    _, P, Q, _ = out_shape("deconv", N, H, W, K, R, S, pad_h, pad_w)
    y = _out(out, (N, K, P, Q), x)
    _check("i2cw_deconv2d_nchw", lib().i2cw_deconv2d_nchw(N, C, H, W, K, R, S, pad_h, pad_w, x.data_ptr(),
                                                          w.data_ptr(), y.data_ptr(), _stream_ptr(stream, x)))
    return y


def out_shape3(kind, N, D, H, W, K, T, R, S, pad_d, pad_h, pad_w):
    if kind == "conv":
        return (N, D + 2 * pad_d - T + 1, H + 2 * pad_h - R + 1, W + 2 * pad_w - S + 1, K)
    return (N, D + T - 1 - 2 * pad_d, H + R - 1 - 2 * pad_h, W + S - 1 - 2 * pad_w, K)


def conv3d_ndhwc(x, w, pad_d, pad_h, pad_w, out=None, stream=None):
    """3D conv; x [N,D,H,W,C], w [K,T,R,S,C] -> y [N,OD,P,Q,K]."""
    _check_tensor(x, "x"); _check_tensor(w, "w")
    N, D, H, W, C = x.shape
    K, T, R, S, C2 = w.shape
    if C != C2 or w.device != x.device:
        raise ValueError("channel or device mismatch")
    y = _out(out, out_shape3("conv", N, D, H, W, K, T, R, S, pad_d, pad_h, pad_w), x)
    _check("i2cw_conv3d_ndhwc", lib().i2cw_conv3d_ndhwc(N, D, H, W, C, K, T, R, S, pad_d, pad_h, pad_w, x.data_ptr(),
                                                        w.data_ptr(), y.data_ptr(), _stream_ptr(stream, x)))
    return y


def deconv3d_ndhwc(x, w, pad_d, pad_h, pad_w, out=None, stream=None):
    """3D transposed conv; x [N,D,H,W,C], w [C,T,R,S,K] -> y [N,OD,P,Q,K], OD = D+T-1-2 pad_d."""
    _check_tensor(x, "x"); _check_tensor(w, "w")
    N, D, H, W, C = x.shape
    C2, T, R, S, K = w.shape
    if C != C2 or w.device != x.device:
        raise ValueError("channel or device mismatch")
    y = _out(out, out_shape3("deconv", N, D, H, W, K, T, R, S, pad_d, pad_h, pad_w), x)
    _check("i2cw_deconv3d_ndhwc", lib().i2cw_deconv3d_ndhwc(N, D, H, W, C, K, T, R, S, pad_d, pad_h, pad_w,
                                                            x.data_ptr(), w.data_ptr(), y.data_ptr(),
                                                            _stream_ptr(stream, x)))
    return y


def filter_bytes(K, C, R, S) -> int:
    """Bytes of a pre-transformed filter for a call with K output / C input channels (C ABI order)."""
    return int(lib().i2cw_filter_bytes(K, C, R, S))


def filter_transform(w, is_deconv=False, stream=None):
    """Pre-transform a filter once (the paper's '*' variant). Returns a uint8 CUDA tensor u."""
    import torch
    _check_tensor(w, "w")
    if is_deconv:
        C, R, S, K = w.shape
    else:
        K, R, S, C = w.shape
    nbytes = filter_bytes(K, C, R, S)
    if nbytes == 0:
        raise I2CWError("i2cw_filter_bytes", I2CW_EUNSUPPORTED)
    u = torch.empty(nbytes, dtype=torch.uint8, device=w.device)
    _check("i2cw_filter_transform", lib().i2cw_filter_transform(K, C, R, S, int(bool(is_deconv)), w.data_ptr(),
                                                                u.data_ptr(), _stream_ptr(stream, w)))
    return u


def conv2d_nhwc_pretransformed(x, u, K, R, S, pad_h, pad_w, is_deconv=False, out=None, stream=None):
    """y from a filter pre-transformed by filter_transform() (the paper's '*' variant)."""
    import torch
    _check_tensor(x, "x")
    N, H, W, C = x.shape
    if not isinstance(u, torch.Tensor) or u.dtype != torch.uint8 or not u.is_cuda or not u.is_contiguous() \
            or u.device != x.device:
        raise ValueError("u must be a contiguous uint8 CUDA tensor on x's device (from filter_transform)")
    need = filter_bytes(K, C, R, S)
    if need == 0 or u.numel() < need:
        raise ValueError(f"u holds {u.numel()} bytes, this call needs {need}")
    y = _out(out, out_shape("deconv" if is_deconv else "conv", N, H, W, K, R, S, pad_h, pad_w), x)
    fn = lib().i2cw_deconv2d_nhwc_pretransformed if is_deconv else lib().i2cw_conv2d_nhwc_pretransformed
    _check("i2cw_*_pretransformed", fn(N, H, W, C, K, R, S, pad_h, pad_w, x.data_ptr(), u.data_ptr(), y.data_ptr(),
                                       _stream_ptr(stream, x)))
    return y


def conv2d_nhwc_host(x, w, pad_h, pad_w, is_deconv=False, out=None, stream=None):
    """End-to-end call on HOST tensors (CPU, fp32, contiguous; pinned memory recommended):
    H2D copies, the conv/deconv and the D2H copy all happen inside the C call."""
    import torch
    for t, nm in ((x, "x"), (w, "w")):
        if t.dtype != torch.float32 or t.is_cuda or not t.is_contiguous():
            raise ValueError(f"{nm} must be a contiguous fp32 CPU tensor")
    N, H, W, C = x.shape
    if is_deconv:
        C2, R, S, K = w.shape
    else:
        K, R, S, C2 = w.shape
    if C != C2:
        raise ValueError("channel mismatch")
    shp = out_shape("deconv" if is_deconv else "conv", N, H, W, K, R, S, pad_h, pad_w)
    if out is None:
        y = torch.empty(shp, dtype=torch.float32)
    else:
        if out.dtype != torch.float32 or out.is_cuda or not out.is_contiguous() or tuple(out.shape) != tuple(shp):
            raise ValueError(f"out must be a contiguous fp32 CPU tensor of shape {tuple(shp)}")
        y = out
    dev = torch.cuda.current_device()
    _check("i2cw_set_device", lib().i2cw_set_device(dev))
    _check("i2cw_conv2d_nhwc_host", lib().i2cw_conv2d_nhwc_host(int(bool(is_deconv)), N, H, W, C, K, R, S, pad_h,
                                                                pad_w, x.data_ptr(), w.data_ptr(), y.data_ptr(),
                                                                _stream_ptr(stream)))
    return y


def plan(S, C=64):
    """(m, alpha, point_set) the library uses for filter width S with C input channels."""
    m, a, ps = ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
    _check("i2cw_plan", lib().i2cw_plan(S, C, ctypes.byref(m), ctypes.byref(a), ctypes.byref(ps)))
    return m.value, a.value, ps.value


def transform_matrices(m, r, point_set=0):
    """Exact (AT, G, BT) from the library's host Cook-Toom generator, as lists of Fractions."""
    a = m + r - 1
    bufs = [(ctypes.c_int64 * n)() for n in (m * a, m * a, a * r, a * r, a * a, a * a)]
    _check("i2cw_transform_matrices_rational", lib().i2cw_transform_matrices_rational(
        m, r, point_set, *[ctypes.addressof(b) for b in bufs]))

    def mat(num, den, rows, cols):
        return [[Fraction(num[i * cols + j], den[i * cols + j]) for j in range(cols)] for i in range(rows)]
    return mat(bufs[0], bufs[1], m, a), mat(bufs[2], bufs[3], a, r), mat(bufs[4], bufs[5], a, a)


PLAN_FIELDS = ("P", "Q", "m", "alpha", "NT", "NB", "NCC", "NKS", "T_r", "TS", "SEGS", "ROWS", "PB", "WBOX", "HBOX",
               "tile_blocks", "GP", "NPASS", "NUS", "smem_bytes", "pad_h", "pad_w", "NI", "NFULL", "NITEMS", "pair",
               "NKC", "CPC", "KSL", "NIS", "NOB", "PLANE", "strip", "NSTRIP")


def debug_plan(kind, N, H, W, C, K, R, S, pad_h, pad_w):
    """The host planner's launch plan (test hook, not in the public header)."""
    out = (ctypes.c_int * 40)()
    _check("i2cw_debug_plan", lib().i2cw_debug_plan(int(kind == "deconv"), N, H, W, C, K, R, S, pad_h, pad_w,
                                                    ctypes.addressof(out)))
    return dict(zip(PLAN_FIELDS, list(out)))


def debug_set_kchunk(ksteps: int) -> int:
    """TEST-ONLY: cap on k-steps accumulated in one TMEM accumulator (0 = default); returns the old cap."""
    return int(lib().i2cw_debug_set_kchunk(int(ksteps)))


def debug_set_kslices(n: int) -> int:
    """TEST-ONLY: cap on concurrent K slices for small grids (1 disables, 0 = default 4);
    returns the old setting (-1 = default)."""
    return int(lib().i2cw_debug_set_kslices(int(n)))


def debug_conv_simt(x, w, pad_h, pad_w, is_deconv=False, stream=None):
    """TEST-ONLY: the SIMT stepping-stone kernel on the same plan / U (not the product path)."""
    import torch
    _check_tensor(x, "x"); _check_tensor(w, "w")
    N, H, W, C = x.shape
    if is_deconv:
        _, R, S, K = w.shape
    else:
        K, R, S, _ = w.shape
    shp = out_shape("deconv" if is_deconv else "conv", N, H, W, K, R, S, pad_h, pad_w)
    y = torch.empty(shp, dtype=torch.float32, device=x.device)
    _check("i2cw_debug_conv_simt", lib().i2cw_debug_conv_simt(int(bool(is_deconv)), N, H, W, C, K, R, S, pad_h,
                                                              pad_w, x.data_ptr(), w.data_ptr(), y.data_ptr(),
                                                              _stream_ptr(stream, x)))
    return y
