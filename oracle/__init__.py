"""ORACLE — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg (and its
``--impl reference`` arm) may import, call, link or execute anything under
oracle/. The product path (include/i2cw.h and paper_conf_icpp_zhangzxyw24_b200/)
never imports this package and shares no code with it.

Contents
  * direct_conv.c   — plain fp64 direct NHWC conv / deconv (+ the bound sum|x||w|),
                      the definition Im2col-Winograd reaches exactly
                      (§4.1, Table 1,
                      deconv PAPER.md:538-541, fp64 ground truth PAPER.md:4187-4190).
  * cook_toom.py    — exact-rational Cook–Toom F(m,r) matrices, §5.3 / Fig 5.
  * brute_*         — pure-Python exact-integer loops for tiny shapes.

Pins (tests/test_oracle_*.py, -m "not gpu"): hand-worked examples in
tests/golden/, torch fp64 conv2d / conv_transpose2d (an independent library),
scipy correlate2d, delta inputs, the R=S=1 GEMM reduction, the deconv
flip-transpose and adjoint identities, and the Figure 5 matrices.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile direct_conv.c (2D) and direct_conv3d.c (3D) with gcc -O2 -fopenmp (plain C)."""
    srcs = [os.path.join(_HERE, f) for f in ("direct_conv.c", "direct_conv3d.c")]
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < max(map(os.path.getmtime, srcs)):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", tmp, *srcs, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        I, P, L = ctypes.c_int, ctypes.c_void_p, ctypes.c_int64
        for name in ("oracle_conv2d_nhwc_f64", "oracle_deconv2d_nhwc_f64"):
            f = getattr(lib, name)
            f.argtypes = [I] * 9 + [P, P, P, P]
            f.restype = I
        for name in ("oracle_conv2d_nhwc_f64_points", "oracle_deconv2d_nhwc_f64_points"):
            f = getattr(lib, name)
            f.argtypes = [I] * 9 + [P, P, L, P, P, P]
            f.restype = I
        for name in ("oracle_conv3d_ndhwc_f64", "oracle_deconv3d_ndhwc_f64"):
            f = getattr(lib, name)
            f.argtypes = [I] * 12 + [P, P, P, P]
            f.restype = I
        lib.oracle_num_threads.restype = I
        _lib = lib
    return _lib


def num_threads() -> int:
    return _load().oracle_num_threads()


def _as_f32(a) -> np.ndarray:
    try:
        import torch
        if isinstance(a, torch.Tensor):
            a = a.detach().cpu().numpy()
    except ImportError:  # pragma: no cover
        pass
    return np.ascontiguousarray(a, dtype=np.float32)


def out_shape(kind, N, H, W, C, K, R, S, ph, pw):
    if kind == "conv":
        return N, H + 2 * ph - R + 1, W + 2 * pw - S + 1, K
    return N, H + R - 1 - 2 * ph, W + S - 1 - 2 * pw, K


def conv2d_nhwc(x, w, pad_h, pad_w, with_bound=True):
    """x [N,H,W,C] fp32, w [K,R,S,C] fp32 -> (y, B) fp64 [N,P,Q,K]."""
    x, w = _as_f32(x), _as_f32(w)
    N, H, W, C = x.shape
    K, R, S, C2 = w.shape
    assert C == C2
    shp = out_shape("conv", N, H, W, C, K, R, S, pad_h, pad_w)
    y = np.empty(shp, np.float64)
    b = np.empty(shp, np.float64) if with_bound else None
    rc = _load().oracle_conv2d_nhwc_f64(N, H, W, C, K, R, S, pad_h, pad_w, x.ctypes.data, w.ctypes.data,
                                        y.ctypes.data, b.ctypes.data if b is not None else None)
    if rc != 0:
        raise ValueError("oracle: invalid shape")
    return (y, b) if with_bound else y


def deconv2d_nhwc(x, w, pad_h, pad_w, with_bound=True):
    """x [N,H,W,C] fp32, w [C,R,S,K] fp32 -> (y, B) fp64 [N,P,Q,K]."""
    x, w = _as_f32(x), _as_f32(w)
    N, H, W, C = x.shape
    C2, R, S, K = w.shape
    assert C == C2
    shp = out_shape("deconv", N, H, W, C, K, R, S, pad_h, pad_w)
    y = np.empty(shp, np.float64)
    b = np.empty(shp, np.float64) if with_bound else None
    rc = _load().oracle_deconv2d_nhwc_f64(N, H, W, C, K, R, S, pad_h, pad_w, x.ctypes.data, w.ctypes.data,
                                          y.ctypes.data, b.ctypes.data if b is not None else None)
    if rc != 0:
        raise ValueError("oracle: invalid shape")
    return (y, b) if with_bound else y


def points(kind, x, w, pad_h, pad_w, idx):
    """Sampled oracle outputs. idx: int array [npts, 4] of (n, p, q, k)."""
    x, w = _as_f32(x), _as_f32(w)
    idx = np.ascontiguousarray(idx, dtype=np.int32)
    N, H, W, C = x.shape
    if kind == "conv":
        K, R, S, _ = w.shape
        f = _load().oracle_conv2d_nhwc_f64_points
    else:
        _, R, S, K = w.shape
        f = _load().oracle_deconv2d_nhwc_f64_points
    n = idx.shape[0]
    y = np.empty(n, np.float64)
    b = np.empty(n, np.float64)
    rc = f(N, H, W, C, K, R, S, pad_h, pad_w, x.ctypes.data, w.ctypes.data, n, idx.ctypes.data,
           y.ctypes.data, b.ctypes.data)
    if rc != 0:
        raise ValueError("oracle: invalid shape or index")
    return y, b


def _conv3d(kind, x, w, pd, ph, pw, with_bound):
    x, w = _as_f32(x), _as_f32(w)
    N, D, H, W, C = x.shape
    if kind == "conv":
        K, T, R, S, C2 = w.shape
        shp = (N, D + 2 * pd - T + 1, H + 2 * ph - R + 1, W + 2 * pw - S + 1, K)
        f = _load().oracle_conv3d_ndhwc_f64
    else:
        C2, T, R, S, K = w.shape
        shp = (N, D + T - 1 - 2 * pd, H + R - 1 - 2 * ph, W + S - 1 - 2 * pw, K)
        f = _load().oracle_deconv3d_ndhwc_f64
    assert C == C2
    y = np.empty(shp, np.float64)
    b = np.empty(shp, np.float64) if with_bound else None
    rc = f(N, D, H, W, C, K, T, R, S, pd, ph, pw, x.ctypes.data, w.ctypes.data, y.ctypes.data,
           b.ctypes.data if b is not None else None)
    if rc != 0:
        raise ValueError("oracle: invalid shape")
    return (y, b) if with_bound else y


def conv3d_ndhwc(x, w, pad_d, pad_h, pad_w, with_bound=True):
    """3D conv: x [N,D,H,W,C], w [K,T,R,S,C] fp32 -> (y, B) fp64 [N,OD,P,Q,K]."""
    return _conv3d("conv", x, w, pad_d, pad_h, pad_w, with_bound)


def deconv3d_ndhwc(x, w, pad_d, pad_h, pad_w, with_bound=True):
    """3D transposed conv: x [N,D,H,W,C], w [C,T,R,S,K] fp32 -> (y, B) fp64 [N,OD,P,Q,K]."""
    return _conv3d("deconv", x, w, pad_d, pad_h, pad_w, with_bound)


def brute_conv3d_int(x, w, pd, ph, pw):
    """Exact-integer 3D conv on Python ints (tiny shapes): x [N,D,H,W,C], w [K,T,R,S,C]."""
    x = [[[[[int(v) for v in c] for c in row] for row in plane] for plane in img] for img in np.asarray(x)]
    w = np.asarray(w).astype(np.int64)
    N, D, H, W, C = len(x), len(x[0]), len(x[0][0]), len(x[0][0][0]), len(x[0][0][0][0])
    K, T, R, S, _ = w.shape
    OD, P, Q = D + 2 * pd - T + 1, H + 2 * ph - R + 1, W + 2 * pw - S + 1
    y = np.zeros((N, OD, P, Q, K), dtype=object)
    for n in range(N):
        for d in range(OD):
            for p in range(P):
                for q in range(Q):
                    for k in range(K):
                        acc = 0
                        for t in range(T):
                            for r in range(R):
                                for s in range(S):
                                    i, j, l = d - pd + t, p - ph + r, q - pw + s
                                    if 0 <= i < D and 0 <= j < H and 0 <= l < W:
                                        for c in range(C):
                                            acc += x[n][i][j][l][c] * int(w[k, t, r, s, c])
                        y[n, d, p, q, k] = acc
    return y


# ---------------------------------------------------------------------------
# Pure-Python exact integer brute force (tiny shapes only): same definition,
# evaluated on Python ints so fp64 rounding cannot hide an indexing mistake.
# ---------------------------------------------------------------------------
def brute_conv_int(x, w, ph, pw):
    N, H, W, C = len(x), len(x[0]), len(x[0][0]), len(x[0][0][0])
    K, R, S = len(w), len(w[0]), len(w[0][0])
    P, Q = H + 2 * ph - R + 1, W + 2 * pw - S + 1
    y = [[[[0] * K for _ in range(Q)] for _ in range(P)] for _ in range(N)]
    for n in range(N):
        for p in range(P):
            for q in range(Q):
                for k in range(K):
                    acc = 0
                    for r in range(R):
                        for s in range(S):
                            ih, iw = p - ph + r, q - pw + s
                            if 0 <= ih < H and 0 <= iw < W:
                                for c in range(C):
                                    acc += x[n][ih][iw][c] * w[k][r][s][c]
                    y[n][p][q][k] = acc
    return y


def brute_deconv_int(x, w, ph, pw):
    N, H, W, C = len(x), len(x[0]), len(x[0][0]), len(x[0][0][0])
    R, S, K = len(w[0]), len(w[0][0]), len(w[0][0][0])
    P, Q = H + R - 1 - 2 * ph, W + S - 1 - 2 * pw
    y = [[[[0] * K for _ in range(Q)] for _ in range(P)] for _ in range(N)]
    for n in range(N):
        for p in range(P):
            for q in range(Q):
                for k in range(K):
                    acc = 0
                    for r in range(R):
                        for s in range(S):
                            ih, iw = p + ph - r, q + pw - s
                            if 0 <= ih < H and 0 <= iw < W:
                                for c in range(C):
                                    acc += x[n][ih][iw][c] * w[c][r][s][k]
                    y[n][p][q][k] = acc
    return y
