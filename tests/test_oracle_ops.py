"""Pins for the oracle's operators (oracle/oracle.c) against things other than itself:
hand-computed worked examples (tests/golden/hand_examples.json), brute-force gathers with
delta kernels (exact), torch.nn.functional in float64 (a library routine), and
invariants that the paper's graph fixes (remap + max == max(|E1|, |E2|))."""
import json
import math
import os

import numpy as np
import pytest
import torch
import torch.nn.functional as F

import synth

from conftest import GOLDEN

rng = np.random.default_rng(1234)


def f32(a):
    return np.asarray(a, dtype=np.float32)


def hand():
    with open(os.path.join(GOLDEN, "hand_examples.json")) as fh:
        return json.load(fh)


# ---------------------------------------------------------------- worked examples
def test_hand_edge_4x4(orc):
    ex = hand()["edge_4x4"]
    img = f32(ex["image"])
    E, E1, E2 = orc.edge(img, f32(ex["K1"]), f32(ex["K2"]), return_parts=True)
    assert np.array_equal(E1, f32(ex["E1"]))
    assert np.array_equal(E2, f32(ex["E2"]))
    assert np.array_equal(E, f32(ex["E"]))


def test_hand_subsample_5x5(orc):
    ex = hand()["subsample_5x5"]
    y = orc.subsample(f32(ex["x"]), f32(ex["P"]))
    assert np.array_equal(y, f32(ex["y"]))


def test_hand_valid_conv_3x3(orc):
    ex = hand()["valid_3x4"]
    y = orc.conv2d_valid(f32(ex["x"]), f32(ex["K"]))
    assert np.array_equal(y, f32(ex["y"]))


# ---------------------------------------------------------------- library routine pins
def _torch_corr(x, K, padding):
    xt = torch.from_numpy(np.asarray(x, np.float64))[None, None]
    kt = torch.from_numpy(np.asarray(K, np.float64))[None, None]
    return F.conv2d(xt, kt, padding=padding)[0, 0].numpy()


def _ulp_close(a, b, ulps=1):
    a, b = f32(a), f32(b)
    d = np.abs(a.astype(np.float64) - b.astype(np.float64))
    tol = ulps * np.spacing(np.maximum(np.abs(a), np.abs(b)).astype(np.float32)).astype(np.float64)
    return bool(np.all(d <= tol + 1e-45))


@pytest.mark.parametrize("H,W,k", [(7, 9, 3), (12, 10, 5), (20, 23, 16), (16, 16, 16), (5, 31, 4), (3, 3, 5)])
def test_conv_same_vs_torch(orc, H, W, k):
    x = f32(rng.standard_normal((H, W)))
    K = f32(rng.standard_normal((k, k)))
    y = orc.conv2d_same(x, K)
    # torch 'same' pads (k-1)//2 top/left and k//2 bottom/right: the reading R2
    ref = _torch_corr(x, K, "same").astype(np.float32)
    assert y.shape == (H, W)
    assert _ulp_close(y, ref)


@pytest.mark.parametrize("H,W,k", [(9, 9, 5), (100, 100, 5), (13, 17, 1), (30, 11, 5)])
def test_conv_valid_vs_torch(orc, H, W, k):
    x = f32(rng.standard_normal((H, W)))
    K = f32(rng.standard_normal((k, k)))
    y = orc.conv2d_valid(x, K)
    ref = _torch_corr(x, K, 0).astype(np.float32)
    assert y.shape == (H - k + 1, W - k + 1)
    assert _ulp_close(y, ref)


def test_valid_conv_size_p367(orc):
    """100x100 convolved with 5x5 gives 96x96."""
    y = orc.conv2d_valid(np.zeros((100, 100), np.float32), np.ones((5, 5), np.float32))
    assert y.shape == (96, 96)


@pytest.mark.parametrize("H,W", [(6, 8), (7, 9), (483 // 10, 643 // 10), (2, 2)])
def test_subsample_vs_torch(orc, H, W):
    x = f32(rng.standard_normal((H, W)))
    P = f32(rng.standard_normal((2, 2)))
    y = orc.subsample(x, P)
    ref = F.conv2d(torch.from_numpy(x.astype(np.float64))[None, None],
                   torch.from_numpy(P.astype(np.float64))[None, None], stride=2)[0, 0].numpy()
    assert y.shape == ((H - 2) // 2 + 1, (W - 2) // 2 + 1)
    assert _ulp_close(y, ref.astype(np.float32))


def test_tanh_add_neg(orc):
    x = f32(rng.standard_normal(1000) * 3)
    y = f32(rng.standard_normal(1000))
    assert np.array_equal(orc.tanh(x), f32([math.tanh(float(v)) for v in x]))
    assert np.array_equal(orc.add(x, y), x + y)   # one fp32 rounding == numpy fp32 add
    assert np.array_equal(orc.neg(x), -x)


def test_max_fold_order_and_ties(orc):
    a = f32([1, -2, 0.0, 3, -0.0])
    b = f32([2, -3, -0.0, 3, 0.0])
    c = f32([0, -1, 0.0, 1, -1])
    y = orc.max_fold(a, b, c)
    assert np.array_equal(y, f32([2, -1, 0.0, 3, 0.0]))
    # (a > b) ? a : b left fold keeps the FIRST of equal values: sign of zero from a
    assert np.signbit(orc.max_fold(f32([-0.0]), f32([0.0]))[0])


# ---------------------------------------------------------------- exact geometry pins
def test_edge_delta_kernels_are_exact_gathers(orc):
    """K1 = delta(i0,j0) turns C1 into a pure gather E1[r][c] = x~[r+i0-7][c+j0-7]; all 256
    anchors on a 37x41 image (exact, no rounding)."""
    H, W = 37, 41
    x = f32(rng.random((H, W)))
    xp = np.zeros((H + 15, W + 15), np.float32)
    xp[7:7 + H, 7:7 + W] = x                     # zero padding 7 top/left, 8 bottom/right
    for i0 in range(16):
        for j0 in range(16):
            K = np.zeros((16, 16), np.float32)
            K[i0, j0] = 1.0
            E, E1, E2 = orc.edge(x, K, K, return_parts=True)
            ref = xp[i0:i0 + H, j0:j0 + W]
            assert np.array_equal(E1, ref), (i0, j0)
            assert np.array_equal(E, np.abs(ref))


def test_edge_invariant_abs_max(orc):
    """max(E1, E2, -E1, -E2) == max(|E1|, |E2|) (negation and max are exact)."""
    from synth import edge_filter_np
    K1, K2 = edge_filter_np()
    x = f32(rng.random((50, 60)))
    E, E1, E2 = orc.edge(x, K1, K2, return_parts=True)
    assert np.array_equal(E, np.maximum(np.abs(E1), np.abs(E2)))
    # K2 = rot90(K1) and C1, C2 are independent convolutions
    assert np.array_equal(E1, orc.conv2d_same(x, K1))
    assert np.array_equal(E2, orc.conv2d_same(x, K2))


def test_edge_general_reduces_to_pinned_template(orc):
    """edge_general composes pinned operators; with 2 filters and 'max' it IS the 4-orientation
    template, and the other reductions obey their definitions exactly."""
    x = f32(rng.random((40, 52)))
    K = [f32(rng.standard_normal((16, 16))) for _ in range(4)]
    assert np.array_equal(orc.edge_general(x, K[:2], "max"), orc.edge(x, K[0], K[1]))
    E = [orc.conv2d_same(x, k) for k in K]
    assert np.array_equal(orc.edge_general(x, K, "maxabs"), np.max(np.abs(np.stack(E)), axis=0))
    assert np.array_equal(orc.edge_general(x, K, "maxplain"), np.max(np.stack(E), axis=0))
    s = ((E[0] + E[1]) + E[2]) + E[3]          # fp32 left fold
    assert np.array_equal(orc.edge_general(x, K, "sum"), s)
    assert np.array_equal(orc.edge_general(x, K, "max"), np.max(np.abs(np.stack(E)), axis=0))


# ---------------------------------------------------------------- kernel rotation (reading R18)
def test_rotate_kernel_multiples_of_90_are_numpy_rot90(orc):
    """90-degree steps are exact permutations: numpy.rot90 (counter-clockwise), four of them
    the identity, 180 degrees both axes reversed."""
    rs = np.random.default_rng(5)
    for k in (1, 2, 3, 5, 16):
        K = rs.standard_normal((k, k)).astype(np.float32)
        for q in range(4):
            assert np.array_equal(orc.rotate_kernel(K, 90 * q), np.rot90(K, q))
        assert np.array_equal(orc.rotate_kernel(K, 180), K[::-1, ::-1])
        assert np.array_equal(orc.rotate_kernel(K, 360 + 90), np.rot90(K))


def test_rotate_kernel_45_hand_example(orc):
    """3x3 kernel 1..9 rotated by 45 degrees about its centre, worked by hand from R18 with
    a = sqrt(2)/2: the centre tap stays 5; tap (0,1) samples (1-a, 1+a) -> 5 - sqrt(2); tap
    (1,0) samples (1-a, 1-a) -> 5 - 2 sqrt(2); tap (0,0) samples (1-sqrt(2), 1), a row above
    the kernel, half-weight of the outside zero -> (2 - sqrt(2)) * K[0][1] = 4 - 2 sqrt(2)."""
    K = np.arange(1, 10, dtype=np.float32).reshape(3, 3)
    R = orc.rotate_kernel(K, 45).astype(np.float64)
    r2 = np.sqrt(2.0)
    assert R[1, 1] == 5.0
    assert abs(R[0, 1] - (5 - r2)) < 1e-6
    assert abs(R[1, 0] - (5 - 2 * r2)) < 1e-6
    assert abs(R[0, 0] - (4 - 2 * r2)) < 1e-6


def test_rotate_kernel_reproduces_linear_fields(orc):
    """Bilinear interpolation is exact on linear functions: for K[i][j] = al i + be j + ga,
    every tap whose four source taps lie inside K equals the linear function at the source
    point (c + y cos t + x sin t, c - y sin t + x cos t), y = i - c, x = j - c. A transposed
    axis, a flipped sign of t or a wrong centre fails this at every angle."""
    k = 16
    i, j = np.mgrid[0:k, 0:k].astype(np.float64)
    al, be, ga = 0.37, -1.21, 0.5
    K = (al * i + be * j + ga).astype(np.float32)
    c = (k - 1) / 2
    for deg in (30, 45, 60, 135, 200, 315):
        t = np.deg2rad(deg)
        R = orc.rotate_kernel(K, deg).astype(np.float64)
        sr = c + (i - c) * np.cos(t) + (j - c) * np.sin(t)
        sc = c - (i - c) * np.sin(t) + (j - c) * np.cos(t)
        inside = (sr >= 0) & (sr <= k - 1) & (sc >= 0) & (sc <= k - 1)
        want = al * sr + be * sc + ga
        assert inside.sum() > 100
        assert np.abs(R[inside] - want[inside]).max() < 1e-5 * np.abs(want).max()


def test_find_edges_is_the_edge_template_at_4_orientations(orc):
    """find_edges(Im, K, 4, max) is the pinned edge template with K2 = rot90(K1)."""
    img = synth.images_np(3, 1, 40, 37)[0, 0]
    K1, K2 = synth.edge_filter_np()
    assert np.array_equal(orc.find_edges(img, K1, 4, "max"), orc.edge(img, K1, K2))
