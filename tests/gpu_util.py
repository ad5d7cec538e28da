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


GUARD = 1 << 20


def guard_runtime(tg):
    """A tg_runtime whose arena sits between two 1 MiB guard bands of a known byte pattern and
    starts filled with 0xFF bytes (NaN as fp32, as bf16 and as fp16): a kernel that writes
    outside the plan's arena changes a guard band, and one that reads a slot buffer it never
    filled propagates NaN into the outputs (test infrastructure for the slot-layout property
    'every buffer the kernels touch is in the slot')."""

    class GuardRuntime(tg.TorchRuntime):
        def __init__(self):
            super().__init__()
            self.blocks = []

        def _alloc_cb(self, nbytes, dev, ctx):
            t = self._torch.full((int(nbytes) + 2 * GUARD,), 0xA5, dtype=self._torch.uint8, device=f"cuda:{dev}")
            t[GUARD:GUARD + int(nbytes)] = 0xFF
            self._torch.cuda.synchronize()     # the fill runs on torch's stream, the library on its own
            self.blocks.append((t, int(nbytes)))
            self._bufs[t.data_ptr() + GUARD] = t
            return t.data_ptr() + GUARD

        def guards_intact(self) -> bool:
            self._torch.cuda.synchronize()
            return all(bool((t[:GUARD] == 0xA5).all()) and bool((t[GUARD + n:] == 0xA5).all())
                       for t, n in self.blocks)

    return GuardRuntime()
