"""Thin Python binding of include/tg.h (ctypes; argument marshalling only).

Every step of the hot path runs inside libtg.so (planner in C++, copies and fused sm_100a
kernels driven by its stream engine). This module only converts arrays to pointers,
checks status codes and -- when asked -- hands the library PyTorch-owned device memory
and streams through the tg_runtime hooks. There is no fallback: if libtg.so is missing or
fails to load, importing this module raises.

The functions keep the C names (tg_graph_create, tg_input, ..., tg_execute); `Graph` and
`Plan` are small conveniences over them.
"""
from __future__ import annotations

import ctypes
import json
import os
from typing import Sequence

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libtg.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(the CUDA library is the only implementation; there is no CPU fallback)")
_lib = ctypes.CDLL(LIB_PATH)

# ---------------------------------------------------------------------------- constants
TG_OK, TG_E_ARG, TG_E_SHAPE, TG_E_INFEASIBLE, TG_E_CUDA, TG_E_OOM, TG_E_STATE, TG_E_UNSUPPORTED = \
    0, -1, -2, -3, -4, -5, -6, -7
TG_VALID, TG_SAME = 0, 1
TG_ADD, TG_NEG, TG_AFFINE, TG_ABS = 0, 1, 2, 3
TG_MAX, TG_SUM, TG_MAXABS = 0, 1, 2
TG_BIAS_PLANE, TG_BIAS_SCALAR = 0, 1
TG_FP32, TG_BF16_TC, TG_FP32_TC = 0, 1, 2
TG_FUSED, TG_PER_OP, TG_BASELINE = 0, 1, 2
TG_OPLIB_CONV, TG_OPLIB_ELEM, TG_OPLIB_SUB, TG_OPLIB_MATMUL = 0, 1, 2, 3

_STATUS = {v: k for k, v in dict(TG_E_ARG=-1, TG_E_SHAPE=-2, TG_E_INFEASIBLE=-3, TG_E_CUDA=-4,
                                   TG_E_OOM=-5, TG_E_STATE=-6, TG_E_UNSUPPORTED=-7).items()}


class TGError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{_STATUS.get(code, code)}: {msg}")
        self.code = code


# ---------------------------------------------------------------------------- prototypes
c_i32, c_i64, c_u64, c_sz = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_size_t
vp = ctypes.c_void_p
P_id = ctypes.POINTER(c_i32)

ALLOC_FN = ctypes.CFUNCTYPE(vp, c_sz, c_i32, vp)
FREE_FN = ctypes.CFUNCTYPE(None, vp, c_i32, vp)
STREAM_FN = ctypes.CFUNCTYPE(vp, c_i32, c_i32, vp)


class tg_runtime(ctypes.Structure):
    _fields_ = [("alloc", ALLOC_FN), ("free", FREE_FN), ("stream", STREAM_FN), ("ctx", vp)]


class tg_oplib_seg(ctypes.Structure):
    _fields_ = [("p", ctypes.c_void_p), ("r0", ctypes.c_int64), ("r1", ctypes.c_int64)]


class tg_oplib_view(ctypes.Structure):
    _fields_ = [("seg", tg_oplib_seg * 8), ("nseg", ctypes.c_int32)]


class tg_oplib_op(ctypes.Structure):
    """One operator piece for tg_oplib_run (include/tg.h "operator library")."""
    _fields_ = [("kind", ctypes.c_int32), ("nin", ctypes.c_int32), ("in_", tg_oplib_view * 16),
                ("in_dims", (ctypes.c_int64 * 4) * 16), ("y", ctypes.c_void_p), ("y_dims", ctypes.c_int64 * 4),
                ("r0", ctypes.c_int64), ("r1", ctypes.c_int64), ("pad", ctypes.c_int32), ("elem", ctypes.c_int32),
                ("s", ctypes.c_int32), ("a", ctypes.c_float), ("b", ctypes.c_float)]


class tg_plan_stats(ctypes.Structure):
    _fields_ = [("h2d_bytes", c_u64), ("d2h_bytes", c_u64), ("io_lower_bound_bytes", c_u64),
                ("total_temp_bytes", c_u64), ("peak_device_bytes", c_u64 * 8), ("n_chunks", c_i64),
                ("n_units", c_i64), ("n_ops_fig7", c_i64), ("n_ds_fig7", c_i64),
                ("chunk_begin", c_i64), ("chunk_end", c_i64), ("host_registered_bytes", c_u64),
                ("h2d_bytes_steady", c_u64), ("io_lower_bound_data_bytes", c_u64)]


class tg_timing(ctypes.Structure):
    _fields_ = [("launches", c_i64), ("executions", c_i64), ("kernel_ms", ctypes.c_double * 4),
                ("unit_launches", c_i64 * 4), ("h2d_ms", ctypes.c_double), ("d2h_ms", ctypes.c_double)]


class tg_trace_rec(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("kind", ctypes.c_int32), ("chunk", ctypes.c_int64),
                ("t0_ms", ctypes.c_double), ("t1_ms", ctypes.c_double)]


_PROTOS = {
    "tg_graph_create": (c_i32, [ctypes.POINTER(vp)]),
    "tg_graph_destroy": (None, [vp]),
    "tg_input": (c_i32, [vp, c_i64, c_i64, c_i64, c_i64, vp, P_id]),
    "tg_input_device": (c_i32, [vp, c_i64, c_i64, c_i64, c_i64, vp, P_id]),
    "tg_param": (c_i32, [vp, c_i64, c_i64, c_i64, c_i64, vp, P_id]),
    "tg_conv2d": (c_i32, [vp, c_i32, c_i32, c_i32, c_i32, P_id]),
    "tg_elementwise": (c_i32, [vp, c_i32, P_id, c_i32, ctypes.c_float, ctypes.c_float, P_id]),
    "tg_tanh": (c_i32, [vp, c_i32, P_id]),
    "tg_max_combine": (c_i32, [vp, P_id, c_i32, P_id]),
    "tg_subsample": (c_i32, [vp, c_i32, c_i32, c_i32, P_id]),
    "tg_matmul": (c_i32, [vp, c_i32, c_i32, P_id]),
    "tg_output": (c_i32, [vp, c_i32, vp]),
    "tg_output_device": (c_i32, [vp, c_i32, vp]),
    "tg_shape": (c_i32, [vp, c_i32, ctypes.POINTER(c_i64)]),
    "tg_find_edges": (c_i32, [vp, c_i32, c_i32, c_i32, c_i32, P_id]),
    "tg_cnn": (c_i32, [vp, c_i32, c_i32, P_id, c_i32, P_id]),
    "tg_set_devices": (c_i32, [vp, P_id, c_i32]),
    "tg_set_device_budget": (c_i32, [vp, c_u64]),
    "tg_set_precision": (c_i32, [vp, c_i32]),
    "tg_set_chunking": (c_i32, [vp, c_i64, c_i32]),
    "tg_set_shard": (c_i32, [vp, c_i32, c_i32]),
    "tg_set_runtime": (c_i32, [vp, ctypes.POINTER(tg_runtime)]),
    "tg_plan_create": (c_i32, [vp, c_i32, ctypes.POINTER(vp)]),
    "tg_plan_stats_get": (c_i32, [vp, ctypes.POINTER(tg_plan_stats)]),
    "tg_plan_dump_json": (c_i32, [vp, ctypes.c_char_p, c_sz, ctypes.POINTER(c_sz)]),
    "tg_plan_codegen": (c_i32, [vp, ctypes.c_char_p, c_sz, ctypes.POINTER(c_sz)]),
    "tg_oplib_run": (c_i32, [vp, vp]),
    "tg_execute": (c_i32, [vp]),
    "tg_execute_async": (c_i32, [vp]),
    "tg_execute_on": (c_i32, [vp, vp, c_i32]),
    "tg_plan_set_graph": (c_i32, [vp, c_i32]),
    "tg_probe_fp32_peak": (c_i32, [c_i32, ctypes.POINTER(ctypes.c_double)]),
    "tg_plan_set_profiling": (c_i32, [vp, c_i32]),
    "tg_plan_timing_get": (c_i32, [vp, ctypes.POINTER(tg_timing)]),
    "tg_plan_trace_get": (c_i32, [vp, ctypes.POINTER(tg_trace_rec), c_sz, ctypes.POINTER(c_sz)]),
    "tg_plan_launch_count": (c_i64, [vp]),
    "tg_plan_invalidate_params": (c_i32, [vp]),
    "tg_plan_destroy": (None, [vp]),
    "tg_sched_create": (c_i32, [ctypes.POINTER(vp)]),
    "tg_sched_destroy": (None, [vp]),
    "tg_sched_add_ds": (c_i32, [vp, c_u64, c_i32, P_id]),
    "tg_sched_add_op": (c_i32, [vp, P_id, c_i32, P_id, c_i32, P_id]),
    "tg_sched_dfs_order": (c_i32, [vp, P_id]),
    "tg_sched_transfers": (c_i32, [vp, P_id, c_u64, ctypes.POINTER(c_u64), P_id, c_i64, ctypes.POINTER(c_i64)]),
    "tg_sched_optimal": (c_i32, [vp, c_u64, c_u64, P_id, ctypes.POINTER(c_u64), ctypes.POINTER(c_u64),
                                 ctypes.POINTER(c_u64)]),
    "tg_last_error": (ctypes.c_char_p, []),
    "tg_version": (ctypes.c_char_p, []),
}
for _name, (_res, _args) in _PROTOS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_PROTOS)


def last_error() -> str:
    return (_lib.tg_last_error() or b"").decode()


def _ck(st: int) -> None:
    if st != TG_OK:
        raise TGError(st, last_error())


def _ptr(a) -> int:
    """Address of a C-contiguous float32 numpy array or torch tensor (host or device)."""
    if isinstance(a, np.ndarray):
        if a.dtype != np.float32 or not a.flags["C_CONTIGUOUS"]:
            raise TypeError("arrays must be C-contiguous float32")
        return a.ctypes.data
    import torch
    if isinstance(a, torch.Tensor):
        if a.dtype != torch.float32 or not a.is_contiguous():
            raise TypeError("tensors must be contiguous float32")
        return a.data_ptr()
    raise TypeError(f"unsupported buffer type {type(a)}")


def _dims4(shape) -> tuple[int, int, int, int]:
    shape = tuple(int(s) for s in shape)
    if len(shape) > 4:
        raise ValueError("at most 4 dims")
    return (1,) * (4 - len(shape)) + shape


# ---------------------------------------------------------------------------- C-named API
def tg_graph_create() -> int:
    h = vp()
    _ck(_lib.tg_graph_create(ctypes.byref(h)))
    return h.value


def tg_graph_destroy(g: int) -> None:
    _lib.tg_graph_destroy(g)


def _id_call(fn, *args) -> int:
    out = c_i32()
    _ck(fn(*args, ctypes.byref(out)))
    return out.value


def tg_input(g, n, c, h, w, host_ptr) -> int:
    return _id_call(_lib.tg_input, g, n, c, h, w, host_ptr)


def tg_input_device(g, n, c, h, w, dev_ptr) -> int:
    return _id_call(_lib.tg_input_device, g, n, c, h, w, dev_ptr)


def tg_param(g, d0, d1, d2, d3, host_ptr) -> int:
    return _id_call(_lib.tg_param, g, d0, d1, d2, d3, host_ptr)


def tg_conv2d(g, x, k, bias, pad) -> int:
    return _id_call(_lib.tg_conv2d, g, x, k, bias, pad)


def tg_elementwise(g, op, xs: Sequence[int], a=1.0, b=0.0) -> int:
    arr = (c_i32 * len(xs))(*xs)
    return _id_call(_lib.tg_elementwise, g, op, arr, len(xs), a, b)


def tg_tanh(g, x) -> int:
    return _id_call(_lib.tg_tanh, g, x)


def tg_max_combine(g, xs: Sequence[int]) -> int:
    arr = (c_i32 * len(xs))(*xs)
    return _id_call(_lib.tg_max_combine, g, arr, len(xs))


def tg_subsample(g, x, p, s=2) -> int:
    return _id_call(_lib.tg_subsample, g, x, p, s)


def tg_matmul(g, a, b) -> int:
    return _id_call(_lib.tg_matmul, g, a, b)


def tg_output(g, y, host_ptr) -> None:
    _ck(_lib.tg_output(g, y, host_ptr))


def tg_output_device(g, y, dev_ptr) -> None:
    _ck(_lib.tg_output_device(g, y, dev_ptr))


def tg_shape(g, y) -> tuple[int, int, int, int]:
    d = (c_i64 * 4)()
    _ck(_lib.tg_shape(g, y, d))
    return tuple(d)


def tg_find_edges(g, img, kernel, num_orientations=4, combine_op=TG_MAX) -> int:
    return _id_call(_lib.tg_find_edges, g, img, kernel, num_orientations, combine_op)


def tg_cnn(g, img, n5, params: Sequence[int], bias_mode=TG_BIAS_PLANE) -> int:
    arr = (c_i32 * 10)(*params)
    return _id_call(_lib.tg_cnn, g, img, n5, arr, bias_mode)


def tg_set_devices(g, ordinals: Sequence[int]) -> None:
    arr = (c_i32 * len(ordinals))(*ordinals)
    _ck(_lib.tg_set_devices(g, arr, len(ordinals)))


def tg_set_device_budget(g, nbytes: int) -> None:
    _ck(_lib.tg_set_device_budget(g, int(nbytes)))


def tg_set_precision(g, prec: int) -> None:
    _ck(_lib.tg_set_precision(g, prec))


def tg_set_chunking(g, max_chunk_px: int, depth: int) -> None:
    _ck(_lib.tg_set_chunking(g, int(max_chunk_px), int(depth)))


def tg_set_shard(g, rank: int, world: int) -> None:
    _ck(_lib.tg_set_shard(g, rank, world))


def tg_set_runtime(g, rt) -> None:
    _ck(_lib.tg_set_runtime(g, ctypes.byref(rt) if rt is not None else None))


def tg_plan_create(g, mode=TG_FUSED) -> int:
    h = vp()
    _ck(_lib.tg_plan_create(g, mode, ctypes.byref(h)))
    return h.value


def tg_plan_stats_get(p) -> dict:
    s = tg_plan_stats()
    _ck(_lib.tg_plan_stats_get(p, ctypes.byref(s)))
    d = {k: getattr(s, k) for k, _ in tg_plan_stats._fields_}
    d["peak_device_bytes"] = list(s.peak_device_bytes)
    return d


def tg_plan_dump_json(p) -> dict:
    need = c_sz()
    _lib.tg_plan_dump_json(p, None, 0, ctypes.byref(need))
    buf = ctypes.create_string_buffer(need.value)
    _ck(_lib.tg_plan_dump_json(p, buf, need.value, ctypes.byref(need)))
    return json.loads(buf.value.decode())


def tg_oplib_run(op: "tg_oplib_op", stream=None) -> None:
    """Run one operator piece on the device (device pointers in `op`)."""
    _ck(_lib.tg_oplib_run(ctypes.byref(op), stream))


def tg_plan_codegen(p) -> str:
    """C source replaying the plan (tg_plan_codegen)."""
    need = c_sz(0)
    _lib.tg_plan_codegen(p, None, 0, ctypes.byref(need))
    if need.value == 0:
        raise TGError(TG_E_UNSUPPORTED, last_error())
    buf = ctypes.create_string_buffer(need.value)
    _ck(_lib.tg_plan_codegen(p, buf, need.value, ctypes.byref(need)))
    return buf.value.decode()


def tg_execute(p) -> None:
    _ck(_lib.tg_execute(p))


def tg_execute_async(p) -> None:
    _ck(_lib.tg_execute_async(p))


def tg_execute_on(p, stream, blocking: bool = True) -> None:
    """stream: a cudaStream_t handle (int) or None (legacy default stream)."""
    _ck(_lib.tg_execute_on(p, stream, 1 if blocking else 0))


def tg_plan_set_graph(p, on: bool) -> None:
    _ck(_lib.tg_plan_set_graph(p, 1 if on else 0))


def tg_probe_fp32_peak(device: int = 0) -> float:
    """Measured FP32 FFMA peak (TFLOP/s) of the device."""
    v = ctypes.c_double(0.0)
    _ck(_lib.tg_probe_fp32_peak(device, ctypes.byref(v)))
    return v.value


def tg_plan_set_profiling(p, on) -> None:
    """on: 0 off, 1 (True) kernels and copies, 2 kernels only."""
    _ck(_lib.tg_plan_set_profiling(p, int(on)))


def tg_plan_timing_get(p) -> dict:
    t = tg_timing()
    _ck(_lib.tg_plan_timing_get(p, ctypes.byref(t)))
    return {"launches": t.launches, "executions": t.executions, "kernel_ms": list(t.kernel_ms),
            "unit_launches": list(t.unit_launches), "h2d_ms": t.h2d_ms, "d2h_ms": t.d2h_ms}


TRACE_KINDS = {0: "edge", 1: "U1", 2: "U2", 3: "U3", 10: "h2d", 11: "d2h"}


def tg_plan_trace_get(p) -> list[dict]:
    n = c_sz(0)
    _ck(_lib.tg_plan_trace_get(p, None, 0, ctypes.byref(n)))
    buf = (tg_trace_rec * max(1, n.value))()
    _ck(_lib.tg_plan_trace_get(p, buf, n.value, ctypes.byref(n)))
    return [{"device": r.device, "kind": TRACE_KINDS.get(r.kind, str(r.kind)), "chunk": r.chunk,
             "t0_ms": r.t0_ms, "t1_ms": r.t1_ms} for r in buf[:n.value]]


def tg_plan_launch_count(p) -> int:
    return int(_lib.tg_plan_launch_count(p))


def tg_plan_invalidate_params(p) -> None:
    _ck(_lib.tg_plan_invalidate_params(p))


def tg_plan_destroy(p) -> None:
    _lib.tg_plan_destroy(p)


TG_DS_INPUT, TG_DS_PARAM, TG_DS_TEMP, TG_DS_OUTPUT = 0, 1, 2, 3


class Sched:
    """The paper's DFS + latest-time-of-use scheduler (tg_sched_*) over an abstract graph."""

    def __init__(self):
        h = vp()
        _ck(_lib.tg_sched_create(ctypes.byref(h)))
        self.h = h.value
        self.n_ops = 0

    def __del__(self):
        if getattr(self, "h", None):
            _lib.tg_sched_destroy(self.h)
            self.h = None

    def add_ds(self, size: int, kind: int) -> int:
        return _id_call(_lib.tg_sched_add_ds, self.h, int(size), int(kind))

    def add_op(self, ins: Sequence[int], outs: Sequence[int]) -> int:
        a = (c_i32 * max(1, len(ins)))(*ins)
        b = (c_i32 * max(1, len(outs)))(*outs)
        self.n_ops += 1
        return _id_call(_lib.tg_sched_add_op, self.h, a, len(ins), b, len(outs))

    def dfs_order(self) -> list[int]:
        o = (c_i32 * max(1, self.n_ops))()
        _ck(_lib.tg_sched_dfs_order(self.h, o))
        return list(o)[: self.n_ops]

    def transfers(self, order: Sequence[int], capacity: int, trace: bool = False):
        o = (c_i32 * max(1, len(order)))(*order)
        moved = c_u64()
        n = c_i64()
        _ck(_lib.tg_sched_transfers(self.h, o, int(capacity), ctypes.byref(moved), None, 0, ctypes.byref(n)))
        if not trace:
            return moved.value
        buf = (c_i32 * (2 * max(1, n.value)))()
        _ck(_lib.tg_sched_transfers(self.h, o, int(capacity), ctypes.byref(moved), buf, n.value, ctypes.byref(n)))
        return moved.value, [(buf[2 * i], buf[2 * i + 1]) for i in range(n.value)]

    def optimal(self, capacity: int, max_orders: int = 10 ** 7):
        """Exhaustive optimum over all dependence-respecting operator orders (tg_sched_optimal):
        (moved, lexicographically smallest optimal order, orders enumerated, optimal orders)."""
        o = (c_i32 * max(1, self.n_ops))()
        moved, n, nb = c_u64(), c_u64(), c_u64()
        _ck(_lib.tg_sched_optimal(self.h, int(capacity), int(max_orders), o, ctypes.byref(moved), ctypes.byref(n),
                                  ctypes.byref(nb)))
        return moved.value, list(o)[: self.n_ops], n.value, nb.value


def tg_version() -> str:
    return _lib.tg_version().decode()


# ---------------------------------------------------------------------------- torch runtime
class TorchRuntime:
    """tg_runtime backed by PyTorch: the arena comes from the caching allocator
    (torch.empty(uint8)), the three streams are torch.cuda.Stream objects (non-blocking),
    so callers can order torch work / CUDA events against the library's compute stream."""

    def __init__(self):
        import torch
        self._torch = torch
        self._bufs: dict[int, object] = {}
        self._streams: dict[tuple[int, int], object] = {}
        self._alloc = ALLOC_FN(self._alloc_cb)
        self._free = FREE_FN(self._free_cb)
        self._stream = STREAM_FN(self._stream_cb)
        self.struct = tg_runtime(self._alloc, self._free, self._stream, None)

    def _alloc_cb(self, nbytes, dev, ctx):
        try:
            t = self._torch.empty(int(nbytes), dtype=self._torch.uint8, device=f"cuda:{dev}")
        except Exception:  # noqa: BLE001 - reported to the library as NULL (TG_E_OOM)
            return None
        # the caching allocator orders a block's reuse on the allocating (current) stream only;
        # the library's streams are others, so wait once here for work still pending on the block
        self._torch.cuda.current_stream(dev).synchronize()
        self._bufs[t.data_ptr()] = t
        return t.data_ptr()

    def _free_cb(self, ptr, dev, ctx):
        self._bufs.pop(int(ptr or 0), None)

    def _stream_cb(self, dev, which, ctx):
        key = (int(dev), int(which))
        if key not in self._streams:
            self._streams[key] = self._torch.cuda.Stream(device=f"cuda:{dev}")
        return self._streams[key].cuda_stream

    def stream(self, dev: int = 0, which: int = 1):
        """The torch.cuda.Stream the library uses for `which` (0 H2D, 1 compute, 2 D2H)."""
        key = (int(dev), int(which))
        if key not in self._streams:
            self._streams[key] = self._torch.cuda.Stream(device=f"cuda:{dev}")
        return self._streams[key]


# ---------------------------------------------------------------------------- conveniences
class Graph:
    """Owns a tg_graph and keeps every buffer handed to the library alive."""

    def __init__(self):
        self.h = tg_graph_create()
        self._keep = []
        self.runtime = None
        self.device_io = False

    def __del__(self):
        # (at interpreter exit the module's functions may already be torn down)
        if getattr(self, "h", None) and callable(tg_graph_destroy):
            tg_graph_destroy(self.h)
            self.h = None

    def input(self, a, device: bool = False) -> int:
        self._keep.append(a)
        self.device_io = self.device_io or device
        n, c, h, w = _dims4(a.shape)
        return (tg_input_device if device else tg_input)(self.h, n, c, h, w, _ptr(a))

    def param(self, a) -> int:
        a = np.ascontiguousarray(a, dtype=np.float32) if isinstance(a, np.ndarray) else a
        self._keep.append(a)
        return tg_param(self.h, *_dims4(a.shape), _ptr(a))

    def output(self, y: int, a, device: bool = False) -> None:
        self._keep.append(a)
        (tg_output_device if device else tg_output)(self.h, y, _ptr(a))

    def shape(self, y: int):
        return tg_shape(self.h, y)

    def find_edges(self, img: int, kernel: int, num_orientations=4, combine_op=TG_MAX) -> int:
        return tg_find_edges(self.h, img, kernel, num_orientations, combine_op)

    def cnn(self, img: int, n5: int, params: Sequence[int], bias_mode=TG_BIAS_PLANE) -> int:
        return tg_cnn(self.h, img, n5, params, bias_mode)

    def conv2d(self, x, k, bias=-1, pad=TG_VALID):
        return tg_conv2d(self.h, x, k, bias, pad)

    def neg(self, x):
        return tg_elementwise(self.h, TG_NEG, [x])

    def elementwise(self, op, xs, a=1.0, b=0.0):
        return tg_elementwise(self.h, op, list(xs), a, b)

    def tanh(self, x):
        return tg_tanh(self.h, x)

    def subsample(self, x, p, s=2):
        return tg_subsample(self.h, x, p, s)

    def matmul(self, a, b):
        return tg_matmul(self.h, a, b)

    def max_combine(self, xs):
        return tg_max_combine(self.h, xs)

    def set(self, budget: int | None = None, precision: int | None = None, devices=None,
            max_chunk_px: int | None = None, depth: int | None = None, shard=None,
            torch_runtime: bool = False):
        if budget is not None:
            tg_set_device_budget(self.h, budget)
        if precision is not None:
            tg_set_precision(self.h, precision)
        if devices is not None:
            tg_set_devices(self.h, list(devices))
        if max_chunk_px is not None or depth is not None:
            tg_set_chunking(self.h, max_chunk_px or (1 << 25), depth or 3)
        if shard is not None:
            tg_set_shard(self.h, *shard)
        if torch_runtime:
            self.runtime = TorchRuntime()
            tg_set_runtime(self.h, self.runtime.struct)
        return self

    def plan(self, mode=TG_FUSED) -> "Plan":
        return Plan(self, tg_plan_create(self.h, mode))


class Plan:
    def __init__(self, graph: Graph, h: int):
        self.graph = graph
        self.h = h

    def __del__(self):
        if getattr(self, "h", None) and callable(tg_plan_destroy):
            tg_plan_destroy(self.h)
            self.h = None

    def stats(self) -> dict:
        return tg_plan_stats_get(self.h)

    def json(self) -> dict:
        return tg_plan_dump_json(self.h)

    def codegen(self) -> str:
        return tg_plan_codegen(self.h)

    def execute(self, blocking: bool = True, stream=None) -> None:
        """stream: a torch.cuda.Stream (or raw cudaStream_t) to order the execution against
        (tg_execute_on); by default device-resident plans order against the legacy default
        stream and, when PyTorch is loaded, against torch's current stream."""
        if stream is None and self.graph.device_io:
            import torch
            stream = torch.cuda.current_stream()
        if stream is not None:
            tg_execute_on(self.h, getattr(stream, "cuda_stream", stream), blocking)
        else:
            (tg_execute if blocking else tg_execute_async)(self.h)

    def use_graph(self, on: bool = True) -> None:
        """Replay executions as one captured CUDA graph (tg_plan_set_graph)."""
        tg_plan_set_graph(self.h, on)

    def profiling(self, on: bool = True, copies: bool = True) -> None:
        """Per-launch CUDA-event timing; copies=False leaves the copy streams untouched."""
        tg_plan_set_profiling(self.h, 0 if not on else (1 if copies else 2))

    def timing(self) -> dict:
        return tg_plan_timing_get(self.h)

    def launches(self) -> int:
        return tg_plan_launch_count(self.h)

    def trace(self) -> list[dict]:
        """Timeline of the profiled copies and kernel launches (tg_plan_trace_get)."""
        return tg_plan_trace_get(self.h)

    def invalidate_params(self) -> None:
        tg_plan_invalidate_params(self.h)

    def compute_stream(self, dev: int = 0):
        if self.graph.runtime is None:
            raise RuntimeError("compute_stream needs set(torch_runtime=True)")
        return self.graph.runtime.stream(dev, 1)


def edge_graph(img, K1, K2=None, out=None, device: bool = False) -> tuple[Graph, int]:
    """Edge template graph. With K2=None it is find_edges(img, K1, 4, TG_MAX) (K2 = rot90
    K1); otherwise the same graph built from primitives with two given kernels."""
    g = Graph()
    x = g.input(img, device=device)
    k1 = g.param(np.asarray(K1, np.float32).reshape(1, 1, *np.shape(K1)[-2:]))
    if K2 is None:
        e = g.find_edges(x, k1)
    else:
        k2 = g.param(np.asarray(K2, np.float32).reshape(1, 1, *np.shape(K2)[-2:]))
        e1 = g.conv2d(x, k1, -1, TG_SAME)
        e2 = g.conv2d(x, k2, -1, TG_SAME)
        e = g.max_combine([e1, e2, g.neg(e1), g.neg(e2)])
    if out is not None:
        g.output(e, out, device=device)
    return g, e


def edge_graph_general(img, kernels, combine: str = "max", out=None, device: bool = False) -> tuple[Graph, int]:
    """Edge graph from primitives with explicit filters: len(kernels) SAME convolutions combined
    by 'max' (responses and their remaps), 'sum', 'maxabs' or 'maxplain'."""
    g = Graph()
    x = g.input(img, device=device)
    resp = []
    for K in kernels:
        k = g.param(np.asarray(K, np.float32).reshape(1, 1, *np.shape(K)[-2:]))
        resp.append(g.conv2d(x, k, -1, TG_SAME))
    if combine == "max":
        e = g.max_combine(resp + [g.neg(r) for r in resp])
    elif combine == "sum":
        e = tg_elementwise(g.h, TG_ADD, resp)
    elif combine == "maxabs":
        e = g.max_combine([tg_elementwise(g.h, TG_ABS, [r]) for r in resp])
    elif combine == "maxplain":
        e = g.max_combine(resp)
    else:
        raise ValueError(combine)
    if out is not None:
        g.output(e, out, device=device)
    return g, e


def find_edges_graph(img, kernel, num_orientations: int = 4, combine_op: int = TG_MAX, out=None,
                     device: bool = False) -> tuple[Graph, int]:
    """find_edges(Image, Kernel, num_orientations, Combine_op)."""
    g = Graph()
    x = g.input(img, device=device)
    k = g.param(np.asarray(kernel, np.float32).reshape(1, 1, *np.shape(kernel)[-2:]))
    e = g.find_edges(x, k, num_orientations, combine_op)
    if out is not None:
        g.output(e, out, device=device)
    return g, e


def cnn_graph(img, n5: int, params, out=None, bias_mode=TG_BIAS_PLANE, device: bool = False) -> tuple[Graph, int]:
    g = Graph()
    x = g.input(img, device=device)
    ids = [g.param(p) for p in params]
    y = g.cnn(x, n5, ids, bias_mode)
    if out is not None:
        g.output(y, out, device=device)
    return g, y
