"""Pins for the CNN oracle (oracle.cnn; Fig. 7):
  * an independent float64 torch.nn.functional evaluation of the same layer stack
    (conv2d / grouped stride-2 conv2d / tanh -- library routines), normwise 1e-5;
  * delta-kernel geometry: with delta kernels the network is a pure gather followed by
    five tanh's, so every output equals tanh^5 of ONE input pixel at a closed-form offset
    (exact up to the tanh rounding, which both sides do identically here)."""
import math

import numpy as np
import pytest
import torch
import torch.nn.functional as F

from synth import cnn_params_np, images_np, cnn_dims


def torch_cnn64(img, n5, prm, bias_plane=True):
    t = lambda a: torch.from_numpy(np.asarray(a, np.float64))   # noqa: E731
    K1, B1, P2, K3, B3, P4, K5, B5, K6, B6 = [t(p) for p in prm]
    x = t(img)

    def bias(y, B):
        return y + (B if bias_plane else B.view(1, -1, 1, 1))

    def sub(y, P):
        c = y.shape[1]
        return F.conv2d(y, P.view(c, 1, 2, 2), stride=2, groups=c)

    y = torch.tanh(bias(F.conv2d(x, K1), B1))
    y = torch.tanh(sub(y, P2))
    y = torch.tanh(bias(F.conv2d(y, K3), B3))
    y = torch.tanh(sub(y, P4))
    y = torch.tanh(bias(F.conv2d(y, K5), B5))
    y = bias(F.conv2d(y, K6), B6)
    return y.numpy()


def normwise(g, r):
    g = g.astype(np.float64)
    r = r.astype(np.float64)
    errs = []
    for b in range(r.shape[0]):
        for c in range(r.shape[1]):
            errs.append(np.abs(g[b, c] - r[b, c]).max() / max(np.abs(r[b, c]).max(), 1e-30))
    return max(errs)


@pytest.mark.parametrize("n,H,W,n5,bias", [(2, 64, 72, 20, "plane"), (1, 67, 61, 120, "plane"),
                                            (2, 60, 64, 20, "scalar"), (1, 483 // 5, 643 // 5, 120, "scalar")])
def test_cnn_vs_torch64(orc, n, H, W, n5, bias):
    seed = 0x5EED0003
    img = np.stack([images_np(seed, 1, H, W, n0=i)[0] for i in range(n)])
    prm = cnn_params_np(seed, n5, H, W, bias)
    out = orc.cnn(img, n5, prm, bias_plane=(bias == "plane"))
    ref = torch_cnn64(img, n5, prm, bias == "plane")
    assert out.shape == ref.shape == (n, 9) + cnn_dims(H, W)[4]
    assert normwise(out, ref) < 1e-5
    # a transposed kernel index (K[i][j] for K[j][i]) or a misplaced bias plane fails this
    assert np.abs(ref).max() > 0.05


def _tanh32(v):
    return np.float32(math.tanh(float(v)))


def test_cnn_delta_geometry(orc):
    rng = np.random.default_rng(7)
    H, W, n5 = 83, 91, 20
    (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5) = cnn_dims(H, W)
    x = rng.random((H, W)).astype(np.float32)
    a1 = rng.integers(0, 5, (8, 2))
    p2 = rng.integers(0, 2, (8, 2))
    a3 = rng.integers(0, 5, (20, 2))
    p4 = rng.integers(0, 2, (20, 2))
    a5 = rng.integers(0, 5, (n5, 2))
    K1 = np.zeros((8, 1, 5, 5), np.float32)
    P2 = np.zeros((8, 2, 2), np.float32)
    K3 = np.zeros((20, 8, 5, 5), np.float32)
    P4 = np.zeros((20, 2, 2), np.float32)
    K5 = np.zeros((n5, 20, 5, 5), np.float32)
    K6 = np.zeros((9, n5, 1, 1), np.float32)
    for j in range(8):
        K1[j, 0, a1[j, 0], a1[j, 1]] = 1
        P2[j, p2[j, 0], p2[j, 1]] = 1
    for j in range(20):
        K3[j, j % 8, a3[j, 0], a3[j, 1]] = 1
        P4[j, p4[j, 0], p4[j, 1]] = 1
    for j in range(n5):
        K5[j, j % 20, a5[j, 0], a5[j, 1]] = 1
    for j in range(9):
        K6[j, j % n5, 0, 0] = 1
    zeros = [np.zeros((1, c, h, w), np.float32) for c, (h, w) in
             [(8, (h1, w1)), (20, (h3, w3)), (n5, (h5, w5)), (9, (h5, w5))]]
    prm = [K1, zeros[0], P2, K3, zeros[1], P4, K5, zeros[2], K6, zeros[3]]
    out = orc.cnn(x, n5, prm)[0]
    for j in range(9):
        i = j % n5
        m = i % 20
        l = m % 8
        for r in range(h5):
            for c in range(w5):
                R = 2 * (2 * (r + a5[i, 0]) + p4[m, 0] + a3[m, 0]) + p2[l, 0] + a1[l, 0]
                C = 2 * (2 * (c + a5[i, 1]) + p4[m, 1] + a3[m, 1]) + p2[l, 1] + a1[l, 1]
                v = x[R, C]
                for _ in range(5):
                    v = _tanh32(v)
                assert out[j, r, c] == v, (j, r, c)
