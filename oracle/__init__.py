"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl reference`
leg may import this package. The product path never imports it (tests/test_isolation.py
checks that), and the two share no code: only the seeded input generators in synth/
serve both.

  oracle/oracle.c   plain C evaluation of the unsplit operator graphs (fp32 DS, fp64
                    accumulation inside conv/subsample nodes), OpenMP over output rows
  oracle/planner.py accounting (Table 1), splitting / halo back-propagation, chunk rule,
                    DFS + next-use transfer scheduling, brute force over schedules

Parity status per function is listed in DESIGN.md ("Oracle pins").
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc -O2 -fopenmp (no intrinsics) into oracle/liboracle.so."""
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-fopenmp",
                               "-o", _SO, src, "-lm"], cwd=_HERE)
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        f32p = ctypes.POINTER(ctypes.c_float)
        i64 = ctypes.c_int64
        L.orc_conv2d_valid.argtypes = [f32p, i64, i64, f32p, ctypes.c_int, ctypes.c_int, f32p]
        L.orc_conv2d_same.argtypes = [f32p, i64, i64, f32p, ctypes.c_int, ctypes.c_int, f32p]
        L.orc_add.argtypes = [f32p, f32p, f32p, i64]
        L.orc_neg.argtypes = [f32p, f32p, i64]
        L.orc_tanh.argtypes = [f32p, f32p, i64]
        L.orc_max_fold.argtypes = [ctypes.POINTER(f32p), ctypes.c_int, f32p, i64]
        L.orc_subsample.argtypes = [f32p, i64, i64, f32p, ctypes.c_int, f32p]
        L.orc_matmul.argtypes = [f32p, f32p, i64, i64, i64, f32p]
        L.orc_edge.argtypes = [f32p, i64, i64, f32p, f32p, ctypes.c_int, f32p, f32p, f32p]
        L.orc_edge.restype = ctypes.c_int
        L.orc_cnn.argtypes = [f32p, i64, i64, i64, ctypes.c_int, ctypes.POINTER(f32p),
                              ctypes.c_int, f32p]
        L.orc_cnn.restype = ctypes.c_int
        L.orc_num_threads.restype = ctypes.c_int
        L.orc_set_num_threads.argtypes = [ctypes.c_int]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    assert a.dtype == np.float32 and a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_float))


def _c(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float32)


def num_threads() -> int:
    return int(lib().orc_num_threads())


def set_num_threads(n: int) -> None:
    lib().orc_set_num_threads(int(n))


def conv2d_valid(x, K) -> np.ndarray:
    x, K = _c(x), _c(K)
    H, W = x.shape
    kh, kw = K.shape
    y = np.empty((H - kh + 1, W - kw + 1), dtype=np.float32)
    lib().orc_conv2d_valid(_p(x), H, W, _p(K), kh, kw, _p(y))
    return y


def conv2d_same(x, K) -> np.ndarray:
    x, K = _c(x), _c(K)
    H, W = x.shape
    kh, kw = K.shape
    y = np.empty((H, W), dtype=np.float32)
    lib().orc_conv2d_same(_p(x), H, W, _p(K), kh, kw, _p(y))
    return y


def add(a, b) -> np.ndarray:
    a, b = _c(a), _c(b)
    y = np.empty_like(a)
    lib().orc_add(_p(a), _p(b), _p(y), a.size)
    return y


def neg(a) -> np.ndarray:
    a = _c(a)
    y = np.empty_like(a)
    lib().orc_neg(_p(a), _p(y), a.size)
    return y


def tanh(a) -> np.ndarray:
    a = _c(a)
    y = np.empty_like(a)
    lib().orc_tanh(_p(a), _p(y), a.size)
    return y


def max_fold(*xs) -> np.ndarray:
    xs = [_c(x) for x in xs]
    y = np.empty_like(xs[0])
    arr = (ctypes.POINTER(ctypes.c_float) * len(xs))(*[_p(x) for x in xs])
    lib().orc_max_fold(arr, len(xs), _p(y), y.size)
    return y


def subsample(x, P) -> np.ndarray:
    x, P = _c(x), _c(P)
    H, W = x.shape
    s = P.shape[0]
    y = np.empty(((H - s) // s + 1, (W - s) // s + 1), dtype=np.float32)
    lib().orc_subsample(_p(x), H, W, _p(P), s, _p(y))
    return y


def matmul(A, B) -> np.ndarray:
    """C = A B with fp64 accumulation (oracle.c orc_matmul)."""
    A, B = _c(A), _c(B)
    M, K = A.shape
    K2, N = B.shape
    assert K == K2
    C = np.empty((M, N), dtype=np.float32)
    lib().orc_matmul(_p(A), _p(B), M, K, N, _p(C))
    return C


def edge(img, K1, K2, return_parts: bool = False):
    """E = max(Im*K1, Im*K2, -(Im*K1), -(Im*K2)). img: [H][W]."""
    img, K1, K2 = _c(img), _c(K1), _c(K2)
    H, W = img.shape
    ks = K1.shape[0]
    E = np.empty((H, W), dtype=np.float32)
    E1 = np.empty((H, W), dtype=np.float32)
    E2 = np.empty((H, W), dtype=np.float32)
    rc = lib().orc_edge(_p(img), H, W, _p(K1), _p(K2), ks, _p(E), _p(E1), _p(E2))
    if rc != 0:
        raise MemoryError(rc)
    return (E, E1, E2) if return_parts else E


def edge_general(img, kernels, combine: str = "max") -> np.ndarray:
    """Edge graph with explicit filters ('combining the results by doing a
    reduction such as addition/max/max absolute value'), node by node: E_i = Im * K_i (SAME);
    max: left fold over E_1..E_k, -E_1..-E_k; sum: left fold of fp32 adds; maxabs: fold over
    |E_i|; maxplain: fold over E_i."""
    E = [conv2d_same(img, K) for K in kernels]
    if combine == "max":
        return max_fold(*(E + [neg(e) for e in E]))
    if combine == "sum":
        s = E[0]
        for e in E[1:]:
            s = add(s, e)
        return s
    if combine == "maxabs":
        return max_fold(*[np.abs(e) for e in E])
    if combine == "maxplain":
        return max_fold(*E)
    raise ValueError(combine)


def rotate_kernel(K, deg: int) -> np.ndarray:
    """A k x k kernel rotated counter-clockwise by `deg` degrees about its centre
    c = ((k-1)/2, (k-1)/2) -- DESIGN.md reading R18 (the paper draws 8 orientations of one
    filter, Fig. 1(b), without a rule for a discrete kernel). Output tap (i, j)
    takes K at the source point
        sr = c + (i - c) cos t + (j - c) sin t,   sc = c - (i - c) sin t + (j - c) cos t,
    read by bilinear interpolation of the four surrounding taps (taps outside K are 0), in
    float64, rounded once to fp32. For multiples of 90 degrees the source point is a tap, so
    the result is an exact permutation (90 degrees: R[i][j] = K[j][k-1-i])."""
    K = np.asarray(K, dtype=np.float64)
    k = K.shape[0]
    deg = deg % 360
    c = (k - 1) / 2.0
    if deg % 90 == 0:                       # cos, sin exactly in {-1, 0, 1}
        cs, sn = [(1, 0), (0, 1), (-1, 0), (0, -1)][deg // 90]
    else:
        t = math.radians(deg)
        cs, sn = math.cos(t), math.sin(t)
    R = np.zeros((k, k), dtype=np.float64)
    for i in range(k):
        for j in range(k):
            sr = c + (i - c) * cs + (j - c) * sn
            sc = c - (i - c) * sn + (j - c) * cs
            r0, q0 = math.floor(sr), math.floor(sc)
            fr, fc = sr - r0, sc - q0
            v = 0.0
            for dr, wr in ((0, 1.0 - fr), (1, fr)):
                for dc, wc in ((0, 1.0 - fc), (1, fc)):
                    rr, cc = r0 + dr, q0 + dc
                    if 0 <= rr < k and 0 <= cc < k:
                        v += wr * wc * K[rr, cc]
            R[i, j] = v
    return R.astype(np.float32)


def find_edges(img, kernel, num_orientations: int = 4, combine: str = "max") -> np.ndarray:
    """find_edges(Image, Kernel, num_orientations, Combine_op): orientations in
    steps of 360/num_orientations degrees; the first half are SAME convolutions of the image
    with the rotated kernel (rotate_kernel), the second half their remaps -E (PAPER.md:627-629,
    reading R3); combine 'max' over all orientations, 'maxabs' = max |E_i| of the
    convolutions, 'sum' = their sum."""
    step = 360 // num_orientations
    Ks = [rotate_kernel(kernel, q * step) for q in range(num_orientations // 2)]
    return edge_general(img, Ks, combine)


def cnn(img, n5: int, params, bias_plane: bool = True) -> np.ndarray:
    """CNN template. img: [n][1][H][W] or [H][W]; params in the
    order K1,B1,P2,K3,B3,P4,K5,B5,K6,B6. Returns [n][9][H6][W6]."""
    img = _c(img)
    if img.ndim == 2:
        img = img[None, None]
    n, _, H, W = img.shape
    h5 = ((((H - 4) - 2) // 2 + 1 - 4) - 2) // 2 + 1 - 4
    w5 = ((((W - 4) - 2) // 2 + 1 - 4) - 2) // 2 + 1 - 4
    prm = [_c(p) for p in params]
    arr = (ctypes.POINTER(ctypes.c_float) * 10)(*[_p(p) for p in prm])
    out = np.empty((n, 9, h5, w5), dtype=np.float32)
    rc = lib().orc_cnn(_p(img), n, H, W, int(n5), arr, 1 if bias_plane else 0, _p(out))
    if rc != 0:
        raise RuntimeError(f"orc_cnn failed: {rc}")
    return out
