"""The shared input generator: host (numpy) and device (torch) generators agree bit-exactly,
row slices regenerate the same bits, and values follow the stated recipe."""
import numpy as np
import torch

import synth


def test_numpy_torch_generators_agree():
    a = synth.images_np(123, 2, 37, 53, n0=5)
    b = synth.images_torch(123, 2, 37, 53, "cpu", n0=5).numpy()
    assert np.array_equal(a, b)


def test_row_slices_regenerate_bits():
    full = synth.image_np(9, synth.DS_IMAGE, 3, (50, 70))
    part = synth.image_np(9, synth.DS_IMAGE, 3, (50, 70), row0=13, rows=20)
    assert np.array_equal(full[13:33], part)


def test_value_recipe():
    x = synth.images_np(1, 1, 64, 64)
    k = np.round(x * 255).astype(np.int64)
    assert np.array_equal((k.astype(np.float32) / np.float32(255)), x)
    assert 0 <= k.min() and k.max() <= 255 and len(np.unique(k)) > 200
    w = synth.uniform_np(1, 10, (1000,), 0.2)
    assert np.abs(w).max() <= 0.2 and w.std() > 0.1
    K1, K2 = synth.edge_filter_np()
    assert np.array_equal(K2, np.rot90(K1)) and np.allclose(K1, -K1[:, ::-1])
