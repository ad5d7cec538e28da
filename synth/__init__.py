"""Seeded, counter-based synthetic inputs shared by the oracle tests and the CUDA path.

This module holds NONE of the method's arithmetic (no convolution, tanh, max, subsample,
planning or accounting). It only turns (seed, ds_id, image index, element index) into
numbers, so that any chunk of any input can be regenerated bit-identically on the host
(numpy) or on a device (torch), and both sides of a parity test see the same bits.

Recipe:
  key  = fmix32(seed ^ fmix32(ds_id * 0x9E3779B1 + n * 0x7FEB352D + 0x165667B1))
  bits = fmix32(fmix32(idx) ^ key)                 idx = linear index inside image n
  image   : float32(bits >> 24) / float32(255)    8-bit micrograph-like levels k/255
  uniform : float32((2 * ((bits >> 8) * 2^-24) - 1) * a)   computed in float64, rounded once
All arithmetic on 32-bit words is modulo 2^32.
"""
from __future__ import annotations

import math

import numpy as np

M32 = 0xFFFFFFFF

# data-structure ids (stable: changing one changes every generated input)
DS_IMAGE = 0
DS_EDGE_K1 = 1
DS_EDGE_K2 = 2
DS_CNN = {"K1": 10, "B1": 11, "P2": 12, "K3": 13, "B3": 14, "P4": 15,
          "K5": 16, "B5": 17, "K6": 18, "B6": 19}


def seed_for_config(config_no: int) -> int:
    return (0x5EED0000 + int(config_no)) & M32


def _fmix32_np(h: np.ndarray) -> np.ndarray:
    h = h.astype(np.uint64) & M32
    h ^= h >> 16
    h = (h * 0x85EBCA6B) & M32
    h ^= h >> 13
    h = (h * 0xC2B2AE35) & M32
    h ^= h >> 16
    return h


def _fmix32_int(h: int) -> int:
    h &= M32
    h ^= h >> 16
    h = (h * 0x85EBCA6B) & M32
    h ^= h >> 13
    h = (h * 0xC2B2AE35) & M32
    h ^= h >> 16
    return h


def stream_key(seed: int, ds_id: int, n: int) -> int:
    inner = (ds_id * 0x9E3779B1 + n * 0x7FEB352D + 0x165667B1) & M32
    return _fmix32_int((seed ^ _fmix32_int(inner)) & M32)


def bits_np(seed: int, ds_id: int, n: int, idx: np.ndarray) -> np.ndarray:
    """32-bit words for element indices `idx` (any integer array) of image n of ds_id."""
    key = np.uint64(stream_key(seed, ds_id, n))
    return _fmix32_np(_fmix32_np(np.asarray(idx, dtype=np.uint64)) ^ key)


def image_np(seed: int, ds_id: int, n: int, shape, row0: int = 0, rows: int | None = None) -> np.ndarray:
    """float32 plane(s) of shape [..., H, W] for image n; optionally only rows [row0, row0+rows)
    of a single-plane image (idx = r * W + c)."""
    shape = tuple(int(s) for s in shape)
    if rows is None:
        idx = np.arange(int(np.prod(shape)), dtype=np.uint64).reshape(shape)
    else:
        H, W = shape[-2], shape[-1]
        assert len(shape) == 2 and 0 <= row0 and row0 + rows <= H
        idx = (np.arange(row0, row0 + rows, dtype=np.uint64)[:, None] * np.uint64(W)
               + np.arange(W, dtype=np.uint64)[None, :])
    k = (bits_np(seed, ds_id, n, idx) >> np.uint64(24)).astype(np.float32)
    return k / np.float32(255.0)


def uniform_np(seed: int, ds_id: int, shape, a: float, n: int = 0) -> np.ndarray:
    """float32 uniform(-a, a) tensor of `shape` (idx = C-order linear index)."""
    shape = tuple(int(s) for s in shape)
    total = int(np.prod(shape))
    out = np.empty(total, dtype=np.float32)
    step = 1 << 24
    for s0 in range(0, total, step):      # bounded temporaries for multi-GB parameter sets
        idx = np.arange(s0, min(total, s0 + step), dtype=np.uint64)
        u = (bits_np(seed, ds_id, n, idx) >> np.uint64(8)).astype(np.float64) * (2.0 ** -24)
        out[s0:s0 + idx.size] = ((2.0 * u - 1.0) * float(a)).astype(np.float32)
    return out.reshape(shape)


def images_np(seed: int, n: int, H: int, W: int, n0: int = 0) -> np.ndarray:
    """[n][1][H][W] float32 batch of images n0 .. n0+n-1."""
    out = np.empty((n, 1, H, W), dtype=np.float32)
    for i in range(n):
        out[i, 0] = image_np(seed, DS_IMAGE, n0 + i, (H, W))
    return out


# ---------------------------------------------------------------- template parameters
def edge_filter_np(ks: int = 16) -> tuple[np.ndarray, np.ndarray]:
    """Synthetic antisymmetric oriented edge filter K1 and its 90-degree rotation K2
    (SURVEY §8(c) ambiguity 4: the paper's filter from [7] is not printed)."""
    c = (ks - 1) / 2.0
    K1 = np.empty((ks, ks), dtype=np.float32)
    for i in range(ks):
        for j in range(ks):
            s = 1.0 if j > c else -1.0
            K1[i, j] = np.float32(s * math.exp(-((i - c) ** 2 + (j - c) ** 2) / (2.0 * (ks / 4.0) ** 2)))
    K2 = np.ascontiguousarray(np.rot90(K1))
    return K1, K2


def random_edge_filters_np(seed: int, ks: int = 16) -> tuple[np.ndarray, np.ndarray]:
    """Two independent random ks x ks filters (general, not antisymmetric) for parity tests."""
    K1 = uniform_np(seed, DS_EDGE_K1, (ks, ks), 1.0 / ks)
    K2 = uniform_np(seed, DS_EDGE_K2, (ks, ks), 1.0 / ks)
    return K1, K2


def cnn_dims(H: int, W: int):
    """Plane sizes per level for the reconstructed CNN: valid 5x5 convs,
    2x2/2 subsampling with floor((D-2)/2)+1. Pure shape bookkeeping, no arithmetic on data."""
    h1, w1 = H - 4, W - 4
    h2, w2 = (h1 - 2) // 2 + 1, (w1 - 2) // 2 + 1
    h3, w3 = h2 - 4, w2 - 4
    h4, w4 = (h3 - 2) // 2 + 1, (w3 - 2) // 2 + 1
    h5, w5 = h4 - 4, w4 - 4
    return (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5)


def cnn_params_np(seed: int, n5: int, H: int, W: int, bias_mode: str = "plane") -> list[np.ndarray]:
    """The 10 CNN parameter tensors in the C-ABI order K1,B1,P2,K3,B3,P4,K5,B5,K6,B6.
    Weights uniform +-1/sqrt(fan_in); bias planes per-pixel uniform +-0.1; subsample
    kernels uniform +-0.5."""
    (h1, w1), _, (h3, w3), _, (h5, w5) = cnn_dims(H, W)
    d = DS_CNN
    K1 = uniform_np(seed, d["K1"], (8, 1, 5, 5), 1.0 / math.sqrt(25))
    K3 = uniform_np(seed, d["K3"], (20, 8, 5, 5), 1.0 / math.sqrt(200))
    K5 = uniform_np(seed, d["K5"], (n5, 20, 5, 5), 1.0 / math.sqrt(500))
    K6 = uniform_np(seed, d["K6"], (9, n5, 1, 1), 1.0 / math.sqrt(n5))
    P2 = uniform_np(seed, d["P2"], (8, 2, 2), 0.5)
    P4 = uniform_np(seed, d["P4"], (20, 2, 2), 0.5)
    if bias_mode == "plane":
        B1 = uniform_np(seed, d["B1"], (1, 8, h1, w1), 0.1)
        B3 = uniform_np(seed, d["B3"], (1, 20, h3, w3), 0.1)
        B5 = uniform_np(seed, d["B5"], (1, n5, h5, w5), 0.1)
        B6 = uniform_np(seed, d["B6"], (1, 9, h5, w5), 0.1)
    else:
        B1 = uniform_np(seed, d["B1"], (8,), 0.1)
        B3 = uniform_np(seed, d["B3"], (20,), 0.1)
        B5 = uniform_np(seed, d["B5"], (n5,), 0.1)
        B6 = uniform_np(seed, d["B6"], (9,), 0.1)
    return [K1, B1, P2, K3, B3, P4, K5, B5, K6, B6]


# ---------------------------------------------------------------- device-side generator
def images_torch(seed: int, n: int, H: int, W: int, device, n0: int = 0, out=None):
    """Same bits as images_np, generated with torch int64 ops on `device` (e.g. 'cuda:0')
    so multi-GB inputs need no host round trip. Returns [n][1][H][W] float32."""
    import torch

    def fmix(h):
        h = h & M32
        h = h ^ (h >> 16)
        h = (h * 0x85EBCA6B) & M32
        h = h ^ (h >> 13)
        h = (h * 0xC2B2AE35) & M32
        h = h ^ (h >> 16)
        return h

    if out is None:
        out = torch.empty((n, 1, H, W), dtype=torch.float32, device=device)
    rows_per = max(1, (1 << 25) // max(W, 1))
    for i in range(n):
        key = stream_key(seed, DS_IMAGE, n0 + i)
        for r0 in range(0, H, rows_per):
            r1 = min(H, r0 + rows_per)
            idx = torch.arange(r0 * W, r1 * W, dtype=torch.int64, device=device)
            v = fmix(fmix(idx) ^ key)
            k = (v >> 24).to(torch.float32)
            out[i, 0, r0:r1].copy_((k / 255.0).view(r1 - r0, W))
    return out
