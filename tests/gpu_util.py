"""Helpers for the -m gpu parity tests (test infrastructure)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")


def need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def normwise(g, r):
    """max over planes of max|g - r| / max|r| (R16)."""
    g = np.asarray(g, np.float64)
    r = np.asarray(r, np.float64)
    hw = r.shape[-2] * r.shape[-1]
    g = g.reshape(-1, hw)
    r = r.reshape(-1, hw)
    return float(max(np.abs(g[i] - r[i]).max() / max(np.abs(r[i]).max(), 1e-30) for i in range(r.shape[0])))


def pinned(shape):
    return torch.zeros(shape, dtype=torch.float32).pin_memory()
