"""B200-native out-of-core operator-graph executor (Sundaram, Raghunathan & Chakradhar,
IPDPS 2009): the edge-detection and CNN templates executed over data larger than the device
budget with operator splitting, fused offload units and overlapped host<->GPU transfers.

The implementation is libtg.so (C ABI: include/tg.h); `tg` is its ctypes binding."""
from . import tg  # noqa: F401  (raises ImportError if libtg.so is missing: no fallback)

__all__ = ["tg"]
