#!/usr/bin/env python
"""Benchmark of the hot path: a template executed over data larger than the device budget
(BASELINE.json configs[1] by default: the edge-detection template on 15 x 10000x10000 fp32
images = 6.0 GB per GPU, 768 MiB device budget), plus one line per other BASELINE config.

One JSON line (rank 0):
  value     Mpixels/s with inputs already resident in HBM (device-resident plan, uncapped),
            CUDA events on the library's compute stream, max over ranks
  e2e       the same metric through the C ABI with HOST buffers: pinned input -> H2D -> fused
            kernels -> D2H -> pinned output inside the timed region, at the config's budget
            (streamed); `e2e.uncapped` the same without a budget
  roofline  the dominant kernel against its roofline (FP32 peak MEASURED by the FFMA2 probe of
            the library, or the measured bf16 tensor / HBM peaks of MEASURED_PEAKS.json)
  cpu_baseline  the CPU oracle on a bounded sample of the same workload
  per_template  one entry per other config / precision (configs[0], [2], [3](a), [3](b))
Multi-GPU (torchrun): ONE global workload of N x the per-GPU images; every rank executes its
shard of the global chunk list (tg_set_shard) from NUMA-local pinned buffers holding only its
share, no collective on the data path; per-chunk output digests are gathered to show that
every chunk's output is identical for every N.
Usage: python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]
       [--template edge|edge256|cnn4|cnn26|cnn3|cnn3s|cnn3b] [--precision fp32|bf16_tc|fp32_tc]
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "Mpixels/s end-to-end per template at 1/2/4/8 B200; % HBM / host-link roofline"
PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
SMS, FP32_LANES = 148, 128


def derived_fp32_peak_tflops(sm_mhz: float) -> float:
    """Unit-count FP32 peak: 148 SMs x 128 lanes x 2 flop x f_SM (context for the measured one)."""
    return SMS * FP32_LANES * 2 * sm_mhz * 1e6 / 1e12


def measured_peaks() -> dict:
    return json.load(open(PEAKS_FILE)) if os.path.exists(PEAKS_FILE) else {}


# ------------------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks and throttle reasons sampled every 50 ms (20 Hz) during a timed region."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, dev: int):
        self.dev = dev
        self.proc = None
        self.lines: list[str] = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.dev), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except (OSError, FileNotFoundError):
            self.proc = None
        time.sleep(0.2)
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.1)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self) -> dict:
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx = float(parts[1])
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm), "hz": 20}


def merge_clocks(*cs) -> dict:
    sm = [c["sm_mhz"] for c in cs if c and c.get("sm_mhz")]
    return {"sm_mhz": min(sm) if sm else None, "sm_max_mhz": next((c["sm_max_mhz"] for c in cs if c), None),
            "reasons": sorted(set().union(*[set(c["reasons"]) for c in cs if c])),
            "samples": sum(c["samples"] for c in cs if c), "hz": 20,
            "regions": [{"sm_mhz": c["sm_mhz"], "samples": c["samples"]} for c in cs if c]}


# ------------------------------------------------------------------------------ dist
def dist_setup():
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch.distributed as dist
        # TG_BENCH_DIST_BACKEND=gloo with more ranks than GPUs runs the multi-rank code path on
        # one GPU (a functional check of the sharding, NUMA binding, digests and reductions --
        # its timings mean nothing); the measured runs are one rank per GPU over NCCL
        backend = os.environ.get("TG_BENCH_DIST_BACKEND", "nccl")
        local = local % max(1, torch.cuda.device_count())
        torch.cuda.set_device(local)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local}"))
        else:
            dist.init_process_group(backend)
    elif torch.cuda.is_available():
        torch.cuda.set_device(0)
    return rank, world, local


def barrier(world):
    import torch
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    if torch.cuda.is_available():
        torch.cuda.synchronize()


def _reduce_device():
    import torch.distributed as dist
    return "cuda" if dist.get_backend() == "nccl" else "cpu"


def max_over_ranks(x: float, world: int) -> float:
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=_reduce_device())
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def min_over_ranks(x: float, world: int) -> float:
    return -max_over_ranks(-x, world)


def gather_objects(obj, world: int) -> list:
    if world == 1:
        return [obj]
    import torch.distributed as dist
    out = [None] * world
    dist.all_gather_object(out, obj)
    return out


# ------------------------------------------------------------------------------ NUMA
def numa_bind(dev: int) -> dict:
    """Bind this process to the CPUs of its GPU's NUMA node (sysfs numa_node of the GPU's PCI
    function) BEFORE any host buffer is allocated: pinned buffers are then first-touched on the
    node next to the GPU's PCIe root port."""
    import torch
    info = {"node": None, "cpus": None, "bdf": None}
    try:
        pr = torch.cuda.get_device_properties(dev)
        bdf = f"{pr.pci_domain_id:04x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
        info["bdf"] = bdf
        node = int(open(f"/sys/bus/pci/devices/{bdf}/numa_node").read().strip())
        info["node"] = node
        if node >= 0:
            cpus = set()
            for part in open(f"/sys/devices/system/node/node{node}/cpulist").read().strip().split(","):
                a, _, b = part.partition("-")
                cpus.update(range(int(a), int(b or a) + 1))
            cpus &= os.sched_getaffinity(0) or cpus
            if cpus:
                os.sched_setaffinity(0, cpus)
                info["cpus"] = len(cpus)
    except (OSError, ValueError, AttributeError) as e:
        info["error"] = str(e)[:120]
    return info


# ------------------------------------------------------------------------------ workloads
def workload(name: str) -> dict:
    """Per-GPU share of each BASELINE config (weak scaling: N GPUs run N x these images as ONE
    global workload)."""
    import synth
    if name == "edge":       # configs[1]: ~6 GB of large images, 768 MB budget, then uncapped
        return dict(name=name, config="configs[1]", template="edge", n=15, H=10000, W=10000, budget=768 << 20,
                    uncapped=True, seed=synth.seed_for_config(2),
                    desc="edge-detection template (16x16 filter, 4 orientations, max)")
    if name == "edge256":    # configs[0]: one 256x256 image, no splitting (launch-latency bound)
        return dict(name=name, config="configs[0]", template="edge", n=1, H=256, W=256, budget=0, uncapped=False,
                    seed=synth.seed_for_config(1), desc="edge-detection template on one 256x256 image, no split")
    if name == "cnn4":       # configs[3](a) paper-literal: large CNN, one 6400x4800 image, 1.5 GB budget
        return dict(name=name, config="configs[3](a)", template="cnn", n=1, H=4800, W=6400, n5=120,
                    budget=1536 << 20, uncapped=True, bias="plane", seed=synth.seed_for_config(4),
                    desc="large CNN (n5=120) on one 6400x4800 image (17.66e9-float footprint, PAPER.md:745)")
    if name == "cnn26":      # configs[3](b) byte-literal: large CNN, 26 x 480x640 (16.96 GB fp32 footprint)
        return dict(name=name, config="configs[3](b)", template="cnn", n=26, H=480, W=640, n5=120,
                    budget=1536 << 20, uncapped=True, bias="plane", seed=synth.seed_for_config(4),
                    desc="large CNN (n5=120) on 26 x 480x640 (16.96 GB fp32 footprint at Fig. 7 granularity)")
    if name in ("cnn3", "cnn3s", "cnn3b"):  # configs[2]: CNN in-core on a batch
        n5 = 20 if name == "cnn3s" else 120
        bias = "scalar" if name == "cnn3b" else "plane"
        return dict(name=name, config="configs[2]", template="cnn", n=64, H=480, W=640, n5=n5, budget=0,
                    uncapped=False, bias=bias, seed=synth.seed_for_config(3),
                    desc=f"{'large' if n5 == 120 else 'small'} CNN (n5={n5}, bias {bias}), batch of 64 x 480x640")
    raise ValueError(name)


def host_link_peak(dev: int) -> dict:
    """Pinned host <-> device copy rates, best of 5: H2D alone, D2H alone, and both
    directions at once on two streams -- as one 1 GiB copy each, and as 4 x 256 MiB copies each
    interleaved on the two streams (the two directions' start skew then matters less); the
    concurrent figure is the better of the two. Called by every rank at once under torchrun, so
    at N GPUs it measures the concurrent link."""
    import torch
    n = 1 << 28
    h1 = torch.empty(n, dtype=torch.float32).pin_memory()
    h2 = torch.empty(n, dtype=torch.float32).pin_memory()
    d1 = torch.empty(n, dtype=torch.float32, device=f"cuda:{dev}")
    d2 = torch.empty(n, dtype=torch.float32, device=f"cuda:{dev}")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    best = {"h2d": 0.0, "d2h": 0.0, "bidir_each": 0.0}
    for _ in range(5):
        for mode in ("h2d", "d2h", "bidir", "bidir4"):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            s1.wait_event(e0)
            s2.wait_event(e0)
            parts = 4 if mode == "bidir4" else 1
            q = n // parts
            for i in range(parts):
                if mode in ("h2d", "bidir", "bidir4"):
                    with torch.cuda.stream(s1):
                        d1[i * q:(i + 1) * q].copy_(h1[i * q:(i + 1) * q], non_blocking=True)
                if mode in ("d2h", "bidir", "bidir4"):
                    with torch.cuda.stream(s2):
                        h2[i * q:(i + 1) * q].copy_(d2[i * q:(i + 1) * q], non_blocking=True)
            cur = torch.cuda.current_stream()
            cur.wait_stream(s1)
            cur.wait_stream(s2)
            e1.record()
            torch.cuda.synchronize()
            gbs = n * 4 / (e0.elapsed_time(e1) / 1e3) / 1e9
            key = "bidir_each" if mode.startswith("bidir") else mode
            best[key] = max(best[key], gbs)
    del h1, h2, d1, d2
    return best


def out_shape(wl, n):
    import synth
    if wl["template"] == "edge":
        return (n, 1, wl["H"], wl["W"])
    h5, w5 = synth.cnn_dims(wl["H"], wl["W"])[4]
    return (n, 9, h5, w5)


def params_of(wl):
    import synth
    if wl["template"] == "edge":
        return [synth.edge_filter_np()[0]]
    return synth.cnn_params_np(wl["seed"], wl["n5"], wl["H"], wl["W"], wl["bias"])


def make_graph(tg, wl, n, x_ptr, y_ptr, device, params, *, budget=0, prec=None, shard=None, chunking=None):
    """The template graph over n images bound to raw input/output pointers (the C ABI calls;
    host pointers may be a shard's base: only its chunks' rows are touched)."""
    import numpy as np
    g = tg.Graph()
    H, W = wl["H"], wl["W"]
    x = (tg.tg_input_device if device else tg.tg_input)(g.h, n, 1, H, W, x_ptr)
    g.device_io = device
    if wl["template"] == "edge":
        k = g.param(np.asarray(params[0], np.float32).reshape(1, 1, 16, 16))
        y = g.find_edges(x, k, 4, tg.TG_MAX)
    else:
        ids = [g.param(p) for p in params]
        y = g.cnn(x, wl["n5"], ids, tg.TG_BIAS_PLANE if wl["bias"] == "plane" else tg.TG_BIAS_SCALAR)
    (tg.tg_output_device if device else tg.tg_output)(g.h, y, y_ptr)
    g.set(budget=budget, torch_runtime=True, precision=prec, shard=shard,
          max_chunk_px=(chunking or {}).get("max_chunk_px"), depth=(chunking or {}).get("depth"))
    return g


def unit_flops_per_px(wl, precision: str) -> dict:
    """Algorithmic flops per pixel of each unit's OUTPUT level, and which of
    them run on the tensor cores in this precision."""
    if wl["template"] == "edge":
        return {0: (2 * 2 * 256, False)}
    n5 = wl["n5"]
    tc = precision in ("bf16_tc", "fp32_tc")
    u3 = n5 * 500 * 2 + 9 * n5 * 2
    if precision == "fp32_tc":
        u3 = n5 * 500 * 2          # C5 on the tensor cores; the 1x1 C6 on the CUDA cores
    elif precision == "bf16_tc":
        u3 = n5 * 500 * 2 + 9 * n5 * 2
    return {1: (4 * 8 * 25 * 2, False), 2: (4 * 20 * 200 * 2, tc), 3: (u3, tc)}


def unit_bytes(wl, n, precision: str) -> dict:
    """Algorithmic HBM bytes of each unit for n images: inputs read once, bias
    planes once (shared by every image of the batch), outputs written once; T2/T4 in the layout
    the precision path keeps between units (fp32 planes, or bf16 channel blocks)."""
    if wl["template"] == "edge":
        return {0: n * wl["H"] * wl["W"] * 8}
    import synth
    (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5) = synth.cnn_dims(wl["H"], wl["W"])
    bf = precision == "bf16_tc"
    pl = wl["bias"] == "plane"
    t2 = n * h2 * w2 * (16 if bf else 32)
    t4 = n * h4 * w4 * (48 if bf else 96 if precision == "fp32_tc" else 80)
    return {1: n * wl["H"] * wl["W"] * 4 + (8 * h1 * w1 * 4 if pl else 0) + t2,
            2: t2 + (20 * h3 * w3 * 4 if pl else 0) + t4,
            3: t4 + ((wl["n5"] + 9) * h5 * w5 * 4 if pl else 0) + n * 9 * h5 * w5 * 4}


def unit_out_px(wl, n) -> dict:
    import synth
    if wl["template"] == "edge":
        return {0: n * wl["H"] * wl["W"]}
    (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5) = synth.cnn_dims(wl["H"], wl["W"])
    return {1: n * h2 * w2, 2: n * h4 * w4, 3: n * h5 * w5}


KERNEL_NAMES = {0: "edge_fused_kernel (K1)", 1: "cnn_u1_kernel (U1: C1 T S2 T)", 2: "cnn_u2_kernel (U2: C3 T S4 T)",
                3: "cnn_u3_kernel (U3: C5 T C6)"}


def piece_digest(arr, pos0: int, plane_stride: int) -> list:
    """Two 64-bit sums over the output words of one piece of an image's output, arr =
    [planes][rows][w] starting at flat position pos0 of the image's output, planes plane_stride
    apart: sum(v) and sum(v * (pos mod 65521 + 1)). Both are additive over the pieces of an
    image, so an image's digest does not depend on how it was chunked or sharded, and equal
    digests mean bit-identical outputs with overwhelming probability."""
    import numpy as np
    planes, rows, w = arr.shape
    v = np.ascontiguousarray(arr).view(np.uint32).astype(np.uint64)
    pos = (pos0 + np.arange(planes, dtype=np.uint64)[:, None, None] * np.uint64(plane_stride)
           + np.arange(rows * w, dtype=np.uint64).reshape(1, rows, w))
    wgt = pos % np.uint64(65521) + np.uint64(1)
    return [int(v.sum(dtype=np.uint64)), int((v * wgt).sum(dtype=np.uint64))]


def time_steps(fn, stream, steps, flush=None):
    """Device time of `steps` calls of fn with CUDA events on `stream` (L2 flushed between steps
    when `flush` is given: a 512 MB write on the stream, outside the per-step events)."""
    import torch
    if flush is None:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(steps):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / steps
    evs = []
    for _ in range(steps):
        with torch.cuda.stream(stream):
            flush.zero_()
        ea, eb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ea.record(stream)
        fn()
        eb.record(stream)
        evs.append((ea, eb))
    torch.cuda.synchronize()
    return sum(a.elapsed_time(b) for a, b in evs) / steps


def repeats_summary(values, steps_each):
    """Five repeats of a timed measurement: the values, their median and best."""
    return {"n": len(values), "steps_each": steps_each, "values": values,
            "median": statistics.median(values), "best": max(values)}


def auto_steps(fn, stream, floor_steps, min_s):
    """Enough steps for a timed region of at least min_s seconds (clock evidence, stability)."""
    import torch
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(2):
        fn()
    e1.record(stream)
    torch.cuda.synchronize()
    per = max(e0.elapsed_time(e1) / 2 / 1e3, 1e-6)
    return max(floor_steps, int(math.ceil(min_s / per)))


# ------------------------------------------------------------------------------ one config
def run_line(args, ctx, wl_name: str, precision: str, headline: bool) -> dict:
    import numpy as np
    import torch

    import synth
    from paper_conf_ipps_sundaramrc09_b200 import tg

    rank, world, local = ctx["rank"], ctx["world"], ctx["local"]
    wl = workload(wl_name)
    prec_code = {"fp32": tg.TG_FP32, "bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}[precision]
    H, W = wl["H"], wl["W"]
    n_glob = wl["n"] * world
    dev = torch.device(f"cuda:{local}")
    params = params_of(wl)
    chunking = {"max_chunk_px": args.max_chunk_px, "depth": args.depth} if headline else None
    os_ = out_shape(wl, 1)
    out_img = os_[1] * os_[2] * os_[3]

    # ---- the global streamed plan, sharded: which images does this rank touch?
    g0 = make_graph(tg, wl, n_glob, 0x1000, 0x2000, False, params, budget=wl["budget"], prec=prec_code,
                    shard=(rank, world), chunking=chunking)
    j0 = g0.plan().json()
    _, _, c0, c1 = j0["shard"]
    mine = j0["chunks"][c0:c1]
    i0 = min(ch["img"] for ch in mine)
    i1 = max(ch["img"] + ch["nimg"] for ch in mine)
    n_loc = i1 - i0
    px_loc = sum(ch["nimg"] for ch in mine if ch["out"][0] == 0) * H * W   # images this rank completes
    # shards of the global list start on image boundaries here (N x the per-GPU images, the
    # same chunk count per image), so the ranks' image ranges do not overlap
    del g0

    # ---- value: device-resident, uncapped, over this rank's images
    x_dev = synth.images_torch(wl["seed"], n_loc, H, W, dev, n0=i0)
    y_dev = torch.empty(out_shape(wl, n_loc), dtype=torch.float32, device=dev)
    g = make_graph(tg, wl, n_loc, x_dev.data_ptr(), y_dev.data_ptr(), True, params, prec=prec_code)
    g._keep += [x_dev, y_dev]
    p = g.plan()
    cs = p.compute_stream(local)
    run_dev = lambda: p.execute(blocking=False)   # noqa: E731
    for _ in range(args.warmup):
        p.execute()
    px = n_loc * H * W
    flush = torch.empty(128 << 20, dtype=torch.float32, device=dev) if px * 4 < (252 << 20) else None
    steps = args.steps if headline else auto_steps(run_dev, cs, max(args.steps, 20), 0.5)
    if flush is not None and not headline:
        steps = min(steps, max(args.steps, 2000))   # each step also writes the 512 MB flush
    # the timed pass replays each execution as one captured CUDA graph (tg_plan_set_graph: one
    # host call per step; what bounds the launch-latency-bound configs[0]); a second, profiled
    # pass of direct executions gives the per-unit kernel times (events on the compute stream)
    p.use_graph(True)
    p.execute()
    l0 = p.launches()
    barrier(world)
    with ClockSampler(local) as clk_v:
        ms = time_steps(run_dev, cs, steps, flush)
    launches = p.launches() - l0
    p.use_graph(False)
    p.profiling(True, copies=False)
    ms_prof = time_steps(run_dev, cs, steps, flush)
    tim = p.timing()
    p.profiling(False)
    px_all = sum(gather_objects(px, world))
    # SURVEY §8(d) "five repeats: median and best": 5 more graph-replay runs of steps / 5 steps each
    p.use_graph(True)
    p.execute()   # (re-)capture the graph outside the timed repeats
    rep_each = max(1, steps // 5)
    value_repeats = repeats_summary([px_all / (max_over_ranks(time_steps(run_dev, cs, rep_each, flush), world) / 1e3)
                                     / 1e6 for _ in range(5)], rep_each)
    p.use_graph(False)
    del flush
    ms_max = max_over_ranks(ms, world)
    value = px_all / (ms_max / 1e3) / 1e6

    # ---- roofline of the dominant kernel and of every unit
    peaks = measured_peaks()
    bf16_peak = float(peaks.get("bf16_tflops", 1590.0))
    hbm_peak = float(peaks.get("hbm_gbs", 6549.0))
    fp32_peak = ctx["fp32_peak_tflops"]
    fl, ub, opx = unit_flops_per_px(wl, precision), unit_bytes(wl, n_loc, precision), unit_out_px(wl, n_loc)
    units = {}
    compute_ms_at_peak = 0.0
    for u, (fpx, on_tc) in fl.items():
        ms_u = tim["kernel_ms"][u] / steps
        pk = bf16_peak if on_tc else fp32_peak
        t_flop = fpx * opx[u] / (pk * 1e12) * 1e3
        t_byte = ub[u] / (hbm_peak * 1e9) * 1e3
        compute_ms_at_peak += max(t_flop, t_byte)
        if ms_u <= 0:
            continue
        tf = fpx * opx[u] / (ms_u / 1e3) / 1e12
        gbs = ub[u] / (ms_u / 1e3) / 1e9
        units[KERNEL_NAMES[u]] = {"ms": ms_u, "launches_per_step": tim["unit_launches"][u] / steps,
                                  "tflops": tf, "flop_frac": tf / pk, "flop_bound": "tensor" if on_tc else "alu",
                                  "gbs": gbs, "hbm_frac": gbs / hbm_peak,
                                  "bound": "hbm" if t_byte > t_flop else ("tensor" if on_tc else "alu")}
    k = max(fl, key=lambda u: tim["kernel_ms"][u])
    nl = max(1, tim["unit_launches"][k])
    kern_ms = tim["kernel_ms"][k] / nl
    fpx, on_tc = fl[k]
    flops_per_launch = fpx * opx[k] * steps / nl
    bytes_per_launch = ub[k] * steps / nl
    achieved_tf = flops_per_launch / (kern_ms / 1e3) / 1e12
    hbm_gbs = bytes_per_launch / (kern_ms / 1e3) / 1e9
    if on_tc:
        peak_tf = bf16_peak
        peak_basis = ("bf16 dense, measured cuBLAS burst (MEASURED_PEAKS.json)" if "bf16_tflops" in peaks
                      else "bf16 dense fallback 1.59 PFLOP/s (B200_PROFILING.md)")
        if precision == "fp32_tc":
            peak_basis = ("fp16 dense = the measured bf16 burst rate (same kind::f16 MMA); 3xFP16 issues 3 MMAs "
                          "per product, so its algorithmic ceiling is 1/3 of this peak")
    else:
        peak_tf = fp32_peak
        peak_basis = (f"FP32 FFMA peak MEASURED in this run by tg_probe_fp32_peak (FFMA2 chains on every SM) "
                      f"at {ctx['fp32_probe_clocks'].get('sm_mhz')} MHz; unit-count peak at 1965 MHz "
                      f"{derived_fp32_peak_tflops(1965.0):.2f}")
    traffic = None
    tf_file = os.path.join(ROOT, "profiles", "traffic.json")
    ncu = json.load(open(tf_file)) if os.path.exists(tf_file) else {}
    tkey = "edge" if wl["template"] == "edge" else wl["name"]
    tr = ncu.get(f"{tkey}:{precision}:{KERNEL_NAMES[k]}")
    if tr and wl["name"] in ("edge", "cnn3", "cnn3s"):   # the captured workloads (tools/update_traffic.py)
        traffic = tr["dram_bytes_per_out_px"] * opx[k] * steps / nl
    for u in fl:    # ncu pipe utilisation of each unit on the captured workload, when there is one
        e = ncu.get(f"{tkey}:{precision}:{KERNEL_NAMES[u]}")
        if e and KERNEL_NAMES[u] in units:
            units[KERNEL_NAMES[u]]["ncu_captured"] = {k2: v for k2, v in e.items() if k2 != "note"} | {
                "workload": "cnn3 (64 x 480x640, n5 120)" if tkey.startswith("cnn") else "edge 15 x 10000^2"}
    if bytes_per_launch / (hbm_peak * 1e9) > flops_per_launch / (peak_tf * 1e12):
        roofline = {"bound": "hbm", "achieved": hbm_gbs, "peak": hbm_peak, "unit": "GB/s", "frac": hbm_gbs / hbm_peak,
                    "peak_basis": "HBM copy bandwidth, measured (MEASURED_PEAKS.json)",
                    "compute": {"achieved": achieved_tf, "peak": peak_tf, "unit": "TFLOP/s",
                                "frac": achieved_tf / peak_tf, "basis": peak_basis}}
    else:
        roofline = {"bound": "tensor" if on_tc else "alu", "achieved": achieved_tf, "peak": peak_tf,
                    "unit": "TFLOP/s", "frac": achieved_tf / peak_tf, "peak_basis": peak_basis,
                    "hbm": {"achieved": hbm_gbs, "peak": hbm_peak, "unit": "GB/s", "frac": hbm_gbs / hbm_peak}}
    roofline.update({"traffic": traffic, "kernel": KERNEL_NAMES[k], "kernel_ms_per_launch": kern_ms,
                     "algorithmic_flop_per_launch": flops_per_launch, "algorithmic_bytes_per_launch": bytes_per_launch,
                     "kernel_share_of_step": tim["kernel_ms"][k] / steps / ms_prof, "units": units,
                     "profiled_pass_ms_per_step": ms_prof,
                     "compute_ms_per_step_at_peak": compute_ms_at_peak})
    y_first, y_last = y_dev[0].clone(), y_dev[-1].clone()
    del p, g, y_dev

    # ---- e2e: the global plan's shard, NUMA-local pinned host buffers holding only this share
    x_host = torch.empty((n_loc, 1, H, W), dtype=torch.float32).pin_memory()
    x_host.copy_(x_dev)
    del x_dev
    y_host = torch.empty(out_shape(wl, n_loc), dtype=torch.float32).pin_memory()
    xb = x_host.data_ptr() - i0 * H * W * 4
    yb = y_host.data_ptr() - i0 * out_img * 4

    def e2e_pass(budget, timed_steps, profile):
        g2 = make_graph(tg, wl, n_glob, xb, yb, False, params, budget=budget, prec=prec_code,
                        shard=(rank, world), chunking=chunking)
        g2._keep += [x_host, y_host]
        p2 = g2.plan()
        st, js = p2.stats(), p2.json()
        cs2 = p2.compute_stream(local)
        for _ in range(args.warmup):
            p2.execute()
        torch.cuda.synchronize()
        n_steps = timed_steps or auto_steps(lambda: p2.execute(blocking=False), cs2, max(args.steps, 20), 0.5)
        l2 = p2.launches()
        barrier(world)
        with ClockSampler(local) as clk:
            t0 = time.perf_counter()
            ms2 = time_steps(lambda: p2.execute(blocking=False), cs2, n_steps)
            wall = (time.perf_counter() - t0) / n_steps * 1e3
        res = {"ms": ms2, "wall_ms": wall, "steps": n_steps, "launches": p2.launches() - l2, "stats": st,
               "json": js, "clocks": clk.summary()}
        if profile:   # SURVEY §8(d) "five repeats: median and best": 5 more timed runs of n_steps / 5 steps
            each = max(1, n_steps // 5)
            p2.execute()
            res["repeats_ms"] = [max_over_ranks(time_steps(lambda: p2.execute(blocking=False), cs2, each), world)
                                 for _ in range(5)]
            res["repeat_steps"] = each
        if profile and st["n_chunks"] <= js["depth"]:
            # a plan of at most `depth` chunks has no copy/compute overlap within an execution:
            # also time it as one CUDA-graph replay per step (tg_plan_set_graph; executions then
            # serialise, but each costs one host call)
            p2.use_graph(True)
            p2.execute()
            res["graph_ms"] = max_over_ranks(time_steps(lambda: p2.execute(blocking=False), cs2, n_steps), world)
            p2.use_graph(False)
        if profile:
            # kernel busy time in a second pass with events on the compute stream only (no
            # events on the copy streams, which would perturb the copy engines)
            p2.profiling(True, copies=False)
            res["prof_ms"] = time_steps(lambda: p2.execute(blocking=False), cs2, n_steps)
            tim2 = p2.timing()
            p2.profiling(False)
            res["kernel_ms"] = sum(tim2["kernel_ms"]) / n_steps
        del p2, g2
        return res

    cap = e2e_pass(wl["budget"], args.steps if headline else None, True)
    torch.cuda.synchronize()
    # the streamed result equals the device-resident one bit for bit (same kernels, same order)
    same = torch.equal(y_host[0].to(dev), y_first) and torch.equal(y_host[-1].to(dev), y_last)
    assert same, "streamed != resident"
    del y_first, y_last
    ms2_max = max_over_ranks(cap["ms"], world)
    px_glob = sum(gather_objects(px_loc, world))
    e2e_value = px_glob / (ms2_max / 1e3) / 1e6
    st, js = cap["stats"], cap["json"]
    h2d, d2h = st["h2d_bytes_steady"], st["d2h_bytes"]
    # the I/O lower bound of a steady step of THIS shard: its images in and outputs out once,
    # plus, when the plan streams the bias planes with the chunks, the streamed planes once
    streamed_param = (st["io_lower_bound_bytes"] - st["io_lower_bound_data_bytes"]) - js["h2d_param_bytes"]
    lb_steady = n_loc * (H * W + out_img) * 4 + (streamed_param if js["bias"] == "streamed" else 0)
    link = ctx["link"]
    # streamed roofline = max(link time, compute at peak). The link time is a lower
    # bound from the rates measured in this run (every rank at once): the bytes both directions
    # can overlap move at the concurrent-bidirectional rate, the rest of the busier direction
    # at its solo rate (with one direction dominant -- the CNN's 2.2 B/px out vs 4+ in -- the
    # concurrent rate alone would overstate the time)
    both = min(h2d, d2h)
    t_link = (both / (link["bidir_each"] * 1e9)
              + (h2d - both) / (link["h2d"] * 1e9) + (d2h - both) / (link["d2h"] * 1e9)) * 1e3
    t_h2d = h2d / (link["h2d"] * 1e9) * 1e3
    t_d2h = d2h / (link["d2h"] * 1e9) * 1e3
    t_cmp = compute_ms_at_peak
    t_roof = max(t_link, t_cmp)
    s_copy = t_link                 # copy busy time at the measured link rates
    s_kern = cap["kernel_ms"]
    e2e = {"value": e2e_value, "unit": "Mpixels/s", "ms_per_step": ms2_max, "steps": cap["steps"],
           "wall_ms_per_step": cap["wall_ms"], "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
           "lower_bound_bytes_per_step": lb_steady,
           "bytes_vs_lower_bound": (h2d + d2h) / lb_steady,
           "bytes_vs_lower_bound_def": "steady-state step (resident parameters uploaded by the first execution) "
                                       "H2D + D2H over this shard's images in + outputs out once, plus the bias "
                                       "planes once when the plan streams them with the chunks (like for like)",
           "first_execution_bytes_vs_lower_bound": (st["h2d_bytes"] + d2h) / (lb_steady + js["h2d_param_bytes"]),
           "budget_bytes": wl["budget"], "arena_bytes": st["peak_device_bytes"][0], "chunks": st["n_chunks"],
           "shard_chunks": [st["chunk_begin"], st["chunk_end"]], "split": js["split"], "bias": js["bias"],
           "gpu_launches": cap["launches"], "host_registered_bytes": st["host_registered_bytes"],
           "kernel_ms_per_step": s_kern, "kernel_profiled_pass_ms_per_step": cap["prof_ms"],
           "copy_ms_per_step_at_link_rate": s_copy,
           "overlap": (s_copy + s_kern - cap["ms"]) / max(min(s_copy, s_kern), 1e-9),
           "overlap_def": ("(copy busy + kernel busy - timed step) / min(copy busy, kernel busy); step from the "
                           "timed pass (no profiling), kernel busy from a kernels-only profiled pass (events on "
                           "the compute stream only), copy busy = the step's bytes at the link rates measured "
                           "in this run (streamed_roofline.link_ms); 1 = the shorter is fully hidden; "
                           "meaningless for launch-latency-bound steps"),
           "streamed_roofline": {"time_ms": t_roof, "frac": t_roof / cap["ms"], "link_ms": t_link,
                                 "h2d_alone_ms": t_h2d, "d2h_alone_ms": t_d2h, "compute_ms_at_peak": t_cmp,
                                 "bound": "link" if t_link >= t_cmp else "compute",
                                 "def": "max(link, compute at peak) / measured step (SURVEY §8(d)); link = "
                                        "min(H2D, D2H) at the concurrent-bidirectional rate + the rest of "
                                        "the busier direction at its solo rate (rates measured in this run)"},
           "host_link": {"peak_h2d_gbs": link["h2d"], "peak_d2h_gbs": link["d2h"],
                         "peak_bidir_each_gbs": link["bidir_each"],
                         "achieved_h2d_gbs": (h2d / 1e9) / (cap["ms"] / 1e3),
                         "achieved_d2h_gbs": (d2h / 1e9) / (cap["ms"] / 1e3)}}
    if "repeats_ms" in cap:
        e2e["repeats"] = repeats_summary([px_glob / (r / 1e3) / 1e6 for r in cap["repeats_ms"]], cap["repeat_steps"])
    if "graph_ms" in cap:
        e2e["graph_replay"] = {"value": px_glob / (cap["graph_ms"] / 1e3) / 1e6, "ms_per_step": cap["graph_ms"],
                               "what": "the same e2e step replayed as one captured CUDA graph (tg_plan_set_graph)"}
    clocks = [clk_v.summary(), cap["clocks"]]
    # per-image output digests (additive over the pieces of an image), gathered in image order:
    # the first per-GPU share of images is the N = 1 workload, so its digest must equal N = 1's
    M64 = (1 << 64) - 1
    h_o, w_o = os_[2], os_[3]
    dig = {}
    for ch in mine:
        r0, r1 = ch["out"]
        for b in range(ch["img"], ch["img"] + ch["nimg"]):
            a, c = piece_digest(y_host[b - i0, :, r0:r1].numpy(), r0 * w_o, h_o * w_o)
            o = dig.setdefault(b, [0, 0])
            o[0], o[1] = (o[0] + a) & M64, (o[1] + c) & M64
    per_img = {}
    for part in gather_objects(dig, world):
        for b, (a, c) in part.items():
            o = per_img.setdefault(b, [0, 0])
            o[0], o[1] = (o[0] + a) & M64, (o[1] + c) & M64

    def fold(ds):
        h = 1469598103934665603
        for a, b in ds:
            h = ((h ^ a) * 1099511628211 + b) & M64
        return f"{h:016x}"

    ordered = [per_img[b] for b in sorted(per_img)]
    checksum = {"images": len(ordered), "digest_all": fold(ordered), "digest_first_share": fold(ordered[:wl["n"]]),
                "first_share_images": wl["n"],
                "def": "FNV fold, in image order, of per-image (sum, position-weighted sum) of the output words "
                       "(additive over chunks, so independent of chunking and sharding); digest_first_share "
                       "covers the first per-GPU share of images (the N=1 workload) and must equal the N=1 "
                       "run's digest_all"}
    if wl["uncapped"]:
        unc = e2e_pass(0, args.steps if headline else None, False)
        ms_u = max_over_ranks(unc["ms"], world)
        su = unc["stats"]
        e2e["uncapped"] = {"value": px_glob / (ms_u / 1e3) / 1e6, "ms_per_step": ms_u, "steps": unc["steps"],
                           "chunks": su["n_chunks"], "arena_bytes": su["peak_device_bytes"][0],
                           "split": unc["json"]["split"], "bias": unc["json"]["bias"],
                           "h2d_bytes_per_step": su["h2d_bytes_steady"], "d2h_bytes_per_step": su["d2h_bytes"],
                           "bytes_vs_lower_bound": (su["h2d_bytes_steady"] + su["d2h_bytes"])
                           / (n_loc * (H * W + out_img) * 4), "gpu_launches": unc["launches"]}
        clocks.append(unc["clocks"])
    # ---- verification against the oracle in the same run (rank 0, N = 1): one image
    verified = None
    if rank == 0 and world == 1 and not args.no_verify:
        verified = verify_against_oracle(ctx, wl, precision, y_host)
    l2 = {"l2": f"inputs {px * 4 / 1e9:.3f} GB per step" + (" >> 126 MB L2 (no flush needed)" if px * 4 >= (252 << 20)
                                                              else ": L2 flushed (512 MB write) before every "
                                                                   "device-resident timed step")}
    config = config_of(wl, precision, world) | l2
    return {"value": value, "value_repeats": value_repeats, "ms_per_step": ms_max, "steps": steps,
            "clocks": merge_clocks(*clocks),
            "gpu_launches": launches, "roofline": roofline, "e2e": e2e, "config": config, "checksum": checksum,
            "verified": verified, "y_host": y_host if (headline and rank == 0) else None}


def config_of(wl, precision, world) -> dict:
    n = wl["n"]
    desc = (f"{wl['desc']}; {n} x {wl['H']}x{wl['W']} fp32 images ({n * wl['H'] * wl['W'] * 4 / 1e9:.2f} GB) per GPU"
            f"{' x ' + str(world) + ' GPUs = one global workload' if world > 1 else ''}; value: device-resident, "
            f"uncapped; e2e: pinned host buffers, "
            f"{'uncapped' if not wl['budget'] else str(wl['budget'] >> 20) + ' MiB device budget'}, streamed")
    return {"workload": desc, "baseline_config": wl["config"], "template": wl["template"], "images_per_gpu": n,
            "H": wl["H"], "W": wl["W"], "n5": wl.get("n5"), "bias": wl.get("bias"),
            "budget_bytes_e2e": wl["budget"], "precision": precision}


_ORACLE_CACHE: dict = {}


def _normwise(g, r) -> float:
    """max over output planes of max|g - r| / max|r| (R16)."""
    import numpy as np
    g = np.asarray(g, np.float64).reshape(-1, r.shape[-2] * r.shape[-1])
    r = np.asarray(r, np.float64).reshape(-1, r.shape[-2] * r.shape[-1])
    return float(max(np.abs(g[i] - r[i]).max() / max(np.abs(r[i]).max(), 1e-30) for i in range(r.shape[0])))


def verify_against_oracle(ctx, wl, precision, y_host) -> dict:
    """The oracle's output for the first image of the workload (cached across precisions) vs
    this run's streamed GPU output of that image."""
    import oracle
    import synth
    oracle.build()
    key = (wl["template"], wl["seed"], wl["H"], wl["W"], wl.get("n5"), wl.get("bias"))
    t0 = time.perf_counter()
    if key not in _ORACLE_CACHE:
        img = synth.image_np(wl["seed"], synth.DS_IMAGE, 0, (wl["H"], wl["W"]))
        if wl["template"] == "edge":
            K1, K2 = synth.edge_filter_np()
            _ORACLE_CACHE[key] = oracle.edge(img, K1, K2)[None]
        else:
            _ORACLE_CACHE[key] = oracle.cnn(img, wl["n5"], params_of(wl), bias_plane=wl["bias"] == "plane")[0]
    ref = _ORACLE_CACHE[key]
    err = _normwise(y_host[0].numpy(), ref)
    tol = 2e-2 if precision == "bf16_tc" else 1e-5
    return {"images": 1, "max_normwise_err": err, "tol": tol, "ok": err <= tol,
            "oracle_s": round(time.perf_counter() - t0, 2),
            "what": "the oracle's output of the workload's first image vs this run's streamed GPU output"}


# ------------------------------------------------------------------------------ CPU leg
def _cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_oracle_sample(template: str = "edge", target_s: float = 12.0) -> dict:
    """The CPU oracle (as it stands) on a bounded sample of the workload: whole images of the
    workload until ~target_s of CPU work (edge: 10000x10000 images of configs[1]; CNN: images
    of the workload). Reports input Mpx/s, and the same oracle on ONE core on a crop."""
    import oracle
    import synth
    oracle.build()
    wl = workload(template)
    H, W = wl["H"], wl["W"]
    done_px, t_tot, imgs = 0, 0.0, 0
    while (t_tot < target_s or imgs == 0) and imgs < wl["n"]:
        img = synth.image_np(wl["seed"], synth.DS_IMAGE, imgs, (H, W))
        t0 = time.perf_counter()
        if wl["template"] == "edge":
            oracle.edge(img, *synth.edge_filter_np())
        else:
            oracle.cnn(img, wl["n5"], params_of(wl), bias_plane=wl["bias"] == "plane")
        t_tot += time.perf_counter() - t0
        done_px += H * W
        imgs += 1
    out = {"value": done_px / t_tot / 1e6, "unit": "Mpixels/s", "cores": oracle.num_threads(), "kind": "oracle",
           "sample": f"oracle on {imgs} whole {H}x{W} image(s) of the workload ({t_tot:.1f} s)",
           "nproc": os.cpu_count(), "cpu_model": _cpu_model()}
    nt = oracle.num_threads()
    oracle.set_num_threads(1)
    try:
        img = synth.image_np(wl["seed"], synth.DS_IMAGE, 0, (H, W))
        crop = img[:min(H, 1000 if wl["template"] == "edge" else 480), :min(W, 10000 if wl["template"] == "edge" else 640)]
        crop = crop.copy()
        t0 = time.perf_counter()
        if wl["template"] == "edge":
            oracle.edge(crop, *synth.edge_filter_np())
        else:
            wl2 = dict(wl, H=crop.shape[0], W=crop.shape[1])
            oracle.cnn(crop[None, None], wl["n5"], params_of(wl2), bias_plane=wl["bias"] == "plane")
        t1 = time.perf_counter() - t0
        out["single_core"] = {"value": crop.size / t1 / 1e6, "unit": "Mpixels/s",
                              "sample": f"oracle on a {crop.shape[0]}x{crop.shape[1]} crop ({t1:.1f} s)"}
    finally:
        oracle.set_num_threads(nt)
    return out


def run_reference(args):
    """The reference arm: the CPU oracle (as it stands) on the host cores, each step ONE whole
    image of the workload (a bounded sample), timed per step; same config keys as our arm."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    import synth
    oracle.build()
    wl = workload(args.template)
    H, W = wl["H"], wl["W"]
    prm = params_of(wl) if wl["template"] == "cnn" else None

    def step(i):
        img = synth.image_np(wl["seed"], synth.DS_IMAGE, i % wl["n"], (H, W))
        t0 = time.perf_counter()
        if wl["template"] == "edge":
            oracle.edge(img, *synth.edge_filter_np())
        else:
            oracle.cnn(img, wl["n5"], prm, bias_plane=wl["bias"] == "plane")
        return time.perf_counter() - t0

    for i in range(args.warmup):
        step(i)
    ts = [step(args.warmup + i) for i in range(args.steps)]
    t_med = statistics.median(ts)
    v = H * W / t_med / 1e6
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "Mpixels/s",
            "n_gpus": int(args.gpus), "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": t_med * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32 (fp64 accumulation)", "data": "synthetic",
            "config": config_of(wl, args.precision, 1),
            "sample_per_step": f"one whole {H}x{W} image of the workload per step (a bounded sample of the "
                               f"{wl['n']}-image workload); ms_per_step = the median time of one such step",
            "ms_per_workload_extrapolated": t_med * 1e3 * wl["n"],
            "best_step_ms": min(ts) * 1e3,
            "cpu_baseline": {"kind": "oracle", "cores": oracle.num_threads(), "value": v, "nproc": os.cpu_count(),
                             "cpu_model": _cpu_model(),
                             "sample": f"{args.steps} steps of one {H}x{W} image each (median {t_med:.2f} s)"},
            "e2e": {"value": v, "unit": "Mpixels/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------ main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--template", default="edge", choices=["edge", "edge256", "cnn4", "cnn26", "cnn3", "cnn3s", "cnn3b"])
    ap.add_argument("--precision", default="fp32", choices=["fp32", "bf16_tc", "fp32_tc"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-verify", action="store_true", help="skip the in-run oracle verification")
    ap.add_argument("--depth", type=int, default=None, help="pipeline slots of the headline e2e plan")
    ap.add_argument("--max-chunk-px", type=int, default=None, help="chunk cap of the headline e2e plan")
    ap.add_argument("--per-template", default=None,
                    help="extra name:precision lines under per_template (default with --template edge: every "
                         "other BASELINE config; 'none' skips them)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        run_reference(args)
        return
    from paper_conf_ipps_sundaramrc09_b200 import tg
    rank, world, local = dist_setup()
    numa = numa_bind(local)
    import torch
    # measured denominators, every rank at once: the FP32 FFMA peak and the concurrent host link
    with ClockSampler(local) as clk_p:
        fp32_peak = tg.tg_probe_fp32_peak(local)
    fp32_peak = min_over_ranks(fp32_peak, world)
    barrier(world)
    link = host_link_peak(local)
    link = {k: min_over_ranks(v, world) for k, v in link.items()}
    numas = gather_objects(numa, world)
    ctx = {"rank": rank, "world": world, "local": local, "fp32_peak_tflops": fp32_peak,
           "fp32_probe_clocks": clk_p.summary(), "link": link}
    res = run_line(args, ctx, args.template, args.precision, headline=True)
    line = None
    if rank == 0:
        line = {"metric": METRIC, "value": res["value"], "unit": "Mpixels/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms_per_step"],
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
                "dtype": {"fp32": "f32", "bf16_tc": "bf16 (fp32 accumulate)",
                          "fp32_tc": "f32 (3xFP16 tensor cores, fp32 accumulate)"}[args.precision],
                "data": "synthetic (counter-based generator synth/, 8-bit levels k/255)",
                "value_repeats": res["value_repeats"],
                "config": res["config"], "roofline": res["roofline"], "e2e": res["e2e"], "clocks": res["clocks"],
                "gpu_launches": res["gpu_launches"], "checksum": res["checksum"], "verified": res["verified"],
                "measured_peaks": {"fp32_tflops": fp32_peak, "fp32_probe_clocks": ctx["fp32_probe_clocks"],
                                   "fp32_unit_count_tflops_at_1965": derived_fp32_peak_tflops(1965.0),
                                   "host_link_gbs": link},
                "numa": numas, "dist_backend": os.environ.get("TG_BENCH_DIST_BACKEND", "nccl") if world > 1 else None}
        if args.template == "edge":
            line["paper_context"] = {"mpx_s": 24.3, "what": "edge 10000x10000, Tesla C870, host-to-host, no overlap "
                                                            "(PAPER.md:753); 25.5 on 8800 GTX"}
        if world == 1 and not args.no_cpu:
            line["cpu_baseline"] = cpu_oracle_sample(args.template)
    del res
    extra = args.per_template
    if extra is None:
        extra = ("edge256:fp32,cnn4:fp32,cnn4:fp32_tc,cnn4:bf16_tc,cnn26:fp32_tc,cnn26:bf16_tc,"
                 "cnn3:fp32,cnn3:fp32_tc,cnn3:bf16_tc,cnn3s:bf16_tc,cnn3b:bf16_tc"
                 if args.template == "edge" else "none")
    per = []
    for item in ([] if extra == "none" else extra.split(",")):
        name, pr = item.split(":")
        r2 = run_line(args, ctx, name, pr, headline=False)
        if rank == 0:
            ent = {"template": name, "baseline_config": r2["config"]["baseline_config"], "precision": pr,
                   "steps": r2["steps"], "workload": r2["config"]["workload"], "value": r2["value"],
                   "value_repeats": r2["value_repeats"],
                   "unit": "Mpixels/s", "ms_per_step": r2["ms_per_step"],
                   "e2e": {k: r2["e2e"].get(k) for k in ("value", "ms_per_step", "steps", "h2d_bytes_per_step",
                                                         "d2h_bytes_per_step", "bytes_vs_lower_bound", "overlap",
                                                         "chunks", "split", "bias", "uncapped", "repeats")}
                   | {"streamed_roofline_frac": r2["e2e"]["streamed_roofline"]["frac"],
                      "link_ms": r2["e2e"]["streamed_roofline"]["link_ms"],
                      "streamed_roofline_bound": r2["e2e"]["streamed_roofline"]["bound"]},
                   "roofline": {k: r2["roofline"].get(k) for k in ("bound", "achieved", "peak", "unit", "frac",
                                                                    "kernel", "units")},
                   "gpu_launches": r2["gpu_launches"], "clocks": r2["clocks"], "checksum": r2["checksum"],
                   "verified": r2["verified"]}
            if name == "edge256":
                ent["us_per_step_device"] = r2["ms_per_step"] * 1e3
                ent["us_per_step_e2e"] = r2["e2e"]["ms_per_step"] * 1e3
                if "graph_replay" in r2["e2e"]:
                    ent["us_per_step_e2e_graph"] = r2["e2e"]["graph_replay"]["ms_per_step"] * 1e3
                    ent["e2e"]["graph_replay"] = r2["e2e"]["graph_replay"]
                ent["kernel_us_per_launch"] = r2["roofline"]["kernel_ms_per_launch"] * 1e3
            per.append(ent)
        del r2
    if rank == 0:
        if per:
            line["per_template"] = per
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
