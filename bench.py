#!/usr/bin/env python
"""Benchmark of the hot path: a template executed over data larger than the device budget
(BASELINE.json configs[1] by default: the edge-detection template on 15 x 10000x10000 fp32
images = 6.0 GB per GPU, 768 MiB device budget).

One JSON line (rank 0):
  value  Mpixels/s with inputs already resident in HBM (device-resident plan, uncapped),
         CUDA events on the library's compute stream, max over ranks
  e2e    the same metric through the C ABI with HOST buffers: pinned input -> H2D -> fused
         kernels -> D2H -> pinned output inside the timed region, 768 MiB budget (streamed)
  roofline  the dominant kernel (K1) against the FP32 FFMA peak (ALU-bound)
  cpu_baseline  the CPU oracle on a bounded sample of the same workload
Usage: python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]
       [--template edge|cnn] (multi-GPU: torchrun ... bench.py --gpus N)
"""
from __future__ import annotations

import argparse
import json
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
# FP32 FFMA peak derived from unit counts and clocks:
# 148 SMs x 128 FP32 lanes x 2 flop x f_SM
SMS, FP32_LANES = 148, 128


def fp32_peak_tflops(sm_mhz: float) -> float:
    return SMS * FP32_LANES * 2 * sm_mhz * 1e6 / 1e12


# ------------------------------------------------------------------------------ clocks
class ClockSampler:
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
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except (OSError, FileNotFoundError):
            self.proc = None
        time.sleep(0.3)
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.15)
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
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------ dist
def dist_setup(args):
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch.distributed as dist
        # TG_BENCH_DIST_BACKEND=gloo with more ranks than GPUs runs the multi-rank code path on
        # one GPU (a functional check of the sharding, barriers and reductions -- its timings
        # mean nothing); the measured runs are one rank per GPU over NCCL
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


def sum_over_ranks(x: float, world: int) -> float:
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=_reduce_device())
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


# ------------------------------------------------------------------------------ workloads
def workload(name: str, rank: int) -> dict:
    """Per-GPU workloads (weak scaling: every rank processes its own images)."""
    import synth
    if name == "edge":       # configs[1]: ~6 GB of large images, 768 MB budget
        return dict(template="edge", n=15, H=10000, W=10000, budget=768 << 20, seed=synth.seed_for_config(2),
                    n0=15 * rank, desc="edge-detection template (16x16 filter, 4 orientations, max)")
    if name == "cnn4":       # configs[3] paper-literal: large CNN, one 6400x4800 image, 1.5 GB budget
        return dict(template="cnn", n=1, H=4800, W=6400, n5=120, budget=1536 << 20, seed=synth.seed_for_config(4),
                    n0=rank, desc="large CNN (n5=120, 7500 ops / 11334 DS at Fig. 7 granularity; 17.66e9-float "
                                  "footprint, PAPER.md:745)")
    if name in ("cnn3", "cnn3s"):  # configs[2]: CNN in-core on a batch
        n5 = 120 if name == "cnn3" else 20
        return dict(template="cnn", n=64, H=480, W=640, n5=n5, budget=0, seed=synth.seed_for_config(3),
                    n0=64 * rank, desc=f"{'large' if n5 == 120 else 'small'} CNN (n5={n5}), batch of 64 x 480x640")
    raise ValueError(name)


def host_link_peak(dev: int) -> dict:
    """Pinned 1 GiB H2D, D2H, and both concurrently on two streams, best of 5.
    Called by every rank at once under torchrun, so at N GPUs it measures the concurrent link."""
    import torch
    n = 1 << 28
    h1 = torch.empty(n, dtype=torch.float32).pin_memory()
    h2 = torch.empty(n, dtype=torch.float32).pin_memory()
    d1 = torch.empty(n, dtype=torch.float32, device=f"cuda:{dev}")
    d2 = torch.empty(n, dtype=torch.float32, device=f"cuda:{dev}")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    best = {"h2d": 0.0, "d2h": 0.0, "bidir_each": 0.0}
    for _ in range(5):
        for mode in ("h2d", "d2h", "bidir"):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            s1.wait_event(e0)
            s2.wait_event(e0)
            if mode in ("h2d", "bidir"):
                with torch.cuda.stream(s1):
                    d1.copy_(h1, non_blocking=True)
            if mode in ("d2h", "bidir"):
                with torch.cuda.stream(s2):
                    h2.copy_(d2, non_blocking=True)
            cur = torch.cuda.current_stream()
            cur.wait_stream(s1)
            cur.wait_stream(s2)
            e1.record()
            torch.cuda.synchronize()
            gbs = n * 4 / (e0.elapsed_time(e1) / 1e3) / 1e9
            key = "bidir_each" if mode == "bidir" else mode
            best[key] = max(best[key], gbs)
    del h1, h2, d1, d2
    return best


def build_graph(tg, wl, x, out, device: bool, params):
    if wl["template"] == "edge":
        g, _ = tg.edge_graph(x, params[0], out=out, device=device)
    else:
        g, _ = tg.cnn_graph(x, wl["n5"], params, out=out, device=device)
    return g


def unit_flops_per_px(wl) -> dict:
    """Algorithmic flops per pixel of each unit's OUTPUT level."""
    if wl["template"] == "edge":
        return {0: 2 * 2 * 256}
    n5 = wl["n5"]
    return {1: 4 * 8 * 25 * 2, 2: 4 * 20 * 200 * 2, 3: n5 * 500 * 2 + 9 * n5 * 2}


def unit_bytes(wl, precision: str) -> dict:
    """Algorithmic HBM bytes of each unit for the whole batch: inputs read
    once, bias planes once (shared by every image of the batch), outputs written once; T2/T4 in
    the layout the precision path keeps between units (fp32 planes, or bf16 channel blocks)."""
    n = wl["n"]
    if wl["template"] == "edge":
        return {0: n * wl["H"] * wl["W"] * 8}
    import synth
    (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5) = synth.cnn_dims(wl["H"], wl["W"])
    bf = precision == "bf16_tc"
    t2 = n * h2 * w2 * (16 if bf else 32)
    t4 = n * h4 * w4 * (48 if bf else 96 if precision == "fp32_tc" else 80)
    return {1: n * wl["H"] * wl["W"] * 4 + 8 * h1 * w1 * 4 + t2,
            2: t2 + 20 * h3 * w3 * 4 + t4,
            3: t4 + (wl["n5"] + 9) * h5 * w5 * 4 + n * 9 * h5 * w5 * 4}


def unit_out_px(wl) -> dict:
    import synth
    if wl["template"] == "edge":
        return {0: wl["n"] * wl["H"] * wl["W"]}
    (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5) = synth.cnn_dims(wl["H"], wl["W"])
    return {1: wl["n"] * h2 * w2, 2: wl["n"] * h4 * w4, 3: wl["n"] * h5 * w5}


KERNEL_NAMES = {0: "edge_fused_kernel (K1)", 1: "cnn_u1_kernel (U1: C1 T S2 T)", 2: "cnn_u2_kernel (U2: C3 T S4 T)",
                3: "cnn_u3_kernel (U3: C5 T C6)"}


def run(args, rank, world, local):
    import numpy as np
    import torch

    import synth
    from paper_conf_ipps_sundaramrc09_b200 import tg

    wl = workload(args.template, rank)
    n, H, W = wl["n"], wl["H"], wl["W"]
    px = n * H * W
    dev = torch.device(f"cuda:{local}")
    if wl["template"] == "edge":
        params = [synth.edge_filter_np()[0]]
        out_shape = (n, 1, H, W)
    else:
        params = synth.cnn_params_np(wl["seed"], wl["n5"], H, W)
        h5, w5 = synth.cnn_dims(H, W)[4]
        out_shape = (n, 9, h5, w5)
    x_dev = synth.images_torch(wl["seed"], n, H, W, dev, n0=wl["n0"])
    y_dev = torch.empty(out_shape, dtype=torch.float32, device=dev)

    # ---- value: device-resident, uncapped
    g = build_graph(tg, wl, x_dev, y_dev, True, params)
    g.set(torch_runtime=True, precision=args.precision_code)
    p = g.plan()
    cs = p.compute_stream(local)
    for _ in range(args.warmup):
        p.execute()
    p.profiling(True)
    l0 = p.launches()
    barrier(world)
    # inputs smaller than 2x the 126 MB L2: flush L2 between timed steps (a 512 MB write on the
    # compute stream, outside the per-step events); larger inputs stream through L2 anyway
    flush = torch.empty(128 << 20, dtype=torch.float32, device=dev) if px * 4 < (252 << 20) else None
    with ClockSampler(local) as clk:
        if flush is None:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(cs)
            for _ in range(args.steps):
                p.execute(blocking=False)
            e1.record(cs)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / args.steps
        else:
            evs = []
            for _ in range(args.steps):
                with torch.cuda.stream(cs):
                    flush.zero_()
                ea, eb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                ea.record(cs)
                p.execute(blocking=False)
                eb.record(cs)
                evs.append((ea, eb))
            torch.cuda.synchronize()
            ms = sum(a.elapsed_time(b) for a, b in evs) / args.steps
    del flush
    launches = p.launches() - l0
    tim = p.timing()
    ms_max = max_over_ranks(ms, world)
    value = world * px / (ms_max / 1e3) / 1e6
    clocks = clk.summary()
    # dominant kernel: the unit with the largest summed time
    fl, opx = unit_flops_per_px(wl), unit_out_px(wl)
    k = max(fl, key=lambda u: tim["kernel_ms"][u])
    nl = max(1, tim["unit_launches"][k])
    kern_ms = tim["kernel_ms"][k] / nl
    flops_per_launch = fl[k] * opx[k] * args.steps / nl
    achieved_tf = flops_per_launch / (kern_ms / 1e3) / 1e12
    tensor = args.precision in ("bf16_tc", "fp32_tc") and k in (2, 3)
    if tensor and args.precision == "fp32_tc":
        # 3xFP16 C3 / C5 on tcgen05 against the fp16 dense peak (= the measured bf16 peak: same
        # kind::f16 rate); three MMAs per product, so the algorithmic ceiling is 1/3 of it
        peaks = json.load(open(PEAKS_FILE)) if os.path.exists(PEAKS_FILE) else {}
        peak_tf = float(peaks.get("bf16_tflops", 1590.0))
        peak_basis = ("fp16 dense = measured bf16 burst (MEASURED_PEAKS.json); 3xFP16 issues 3 MMAs "
                      "per product: algorithmic ceiling = peak / 3")
        fl = dict(fl)
        fl[3] = wl["n5"] * 500 * 2  # C5 (C6 runs on the CUDA cores on this path); C3 in U2
        flops_per_launch = fl[k] * opx[k] * args.steps / nl
        achieved_tf = flops_per_launch / (kern_ms / 1e3) / 1e12
    elif tensor:
        # C3 / C5 on tcgen05: bf16 dense peak MEASURED on this pool (MEASURED_PEAKS.json, burst:
        # the kernel is timed on its own launches); algorithmic flops exclude K/N padding
        peaks = json.load(open(PEAKS_FILE)) if os.path.exists(PEAKS_FILE) else {}
        peak_tf = float(peaks.get("bf16_tflops", 1590.0))
        peak_basis = ("bf16 dense, measured cuBLAS burst (MEASURED_PEAKS.json)" if "bf16_tflops" in peaks
                      else "bf16 dense fallback 1.59 PFLOP/s (B200_PROFILING.md)")
        fl = dict(fl)
        # the tensor-core part of each unit: C3 (U2); C5 and the 1x1 C6 (U3)
        fl[2], fl[3] = 4 * 20 * 200 * 2, wl["n5"] * 500 * 2 + 9 * wl["n5"] * 2
        flops_per_launch = fl[k] * opx[k] * args.steps / nl
        achieved_tf = flops_per_launch / (kern_ms / 1e3) / 1e12
    else:
        peak_tf = fp32_peak_tflops(1965.0)
        peak_basis = "FP32 FFMA: 148 SM x 128 lanes x 2 flop x 1965 MHz (clocks.max.sm)"
    # the same kernel against the HBM roofline (measured copy bandwidth): bias planes make the
    # single-image CNN units (cnn4) as byte-heavy as they are flop-heavy
    peaks = json.load(open(PEAKS_FILE)) if os.path.exists(PEAKS_FILE) else {}
    hbm_peak = float(peaks.get("hbm_gbs", 6549.0))
    bytes_per_launch = unit_bytes(wl, args.precision)[k] * args.steps / nl
    hbm_gbs = bytes_per_launch / (kern_ms / 1e3) / 1e9
    traffic = None
    tf_file = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tf_file):
        tr = json.load(open(tf_file)).get(f"{args.template}:{args.precision}:{KERNEL_NAMES[k]}")
        if tr:
            traffic = tr["dram_bytes_per_out_px"] * opx[k] * args.steps / nl
    if bytes_per_launch / (hbm_peak * 1e9) > flops_per_launch / (peak_tf * 1e12):
        # HBM is the binding roofline of this kernel at this workload
        roofline = {"bound": "hbm", "achieved": hbm_gbs, "peak": hbm_peak, "unit": "GB/s", "frac": hbm_gbs / hbm_peak,
                    "peak_basis": "HBM copy bandwidth, measured (MEASURED_PEAKS.json)" if "hbm_gbs" in peaks
                    else "HBM fallback 6549 GB/s", "compute": {"achieved": achieved_tf, "peak": peak_tf,
                                                              "unit": "TFLOP/s", "frac": achieved_tf / peak_tf,
                                                              "basis": peak_basis}}
    else:
        roofline = {"bound": "tensor" if tensor else "alu", "achieved": achieved_tf, "peak": peak_tf,
                    "unit": "TFLOP/s", "frac": achieved_tf / peak_tf, "peak_basis": peak_basis,
                    "hbm": {"achieved": hbm_gbs, "peak": hbm_peak, "unit": "GB/s", "frac": hbm_gbs / hbm_peak}}
    roofline.update({"traffic": traffic, "kernel": KERNEL_NAMES[k], "kernel_ms_per_launch": kern_ms,
                     "algorithmic_flop_per_launch": flops_per_launch,
                     "algorithmic_bytes_per_launch": bytes_per_launch,
                     "kernel_share_of_step": tim["kernel_ms"][k] / args.steps / ms,
                     "units_ms_per_step": {KERNEL_NAMES[u]: tim["kernel_ms"][u] / args.steps for u in fl}})
    # every unit of the step against both rooflines (algorithmic flops and bytes per step)
    ub, uf = unit_bytes(wl, args.precision), unit_flops_per_px(wl)
    units = {}
    for u in uf:
        ms_u = tim["kernel_ms"][u] / args.steps
        if ms_u <= 0:
            continue
        tens_u = args.precision in ("bf16_tc", "fp32_tc") and u in (2, 3)
        if tens_u and args.precision == "fp32_tc":  # C3 / C5 (3xFP16; C6 on the CUDA cores)
            fpx = 4 * 20 * 200 * 2 if u == 2 else wl["n5"] * 500 * 2
        elif tens_u:  # the tensor-core part: C3 (U2); C5 and C6 (U3)
            fpx = 4 * 20 * 200 * 2 if u == 2 else wl["n5"] * 500 * 2 + 9 * wl["n5"] * 2
        else:
            fpx = uf[u]
        f_u = fpx * opx[u] / (ms_u / 1e3) / 1e12
        pk_u = (float(peaks.get("bf16_tflops", 1590.0)) if tens_u
                else fp32_peak_tflops(1965.0))
        units[KERNEL_NAMES[u]] = {"ms": ms_u, "tflops": f_u, "flop_frac": f_u / pk_u,
                                  "flop_bound": "tensor" if tens_u else "alu",
                                  "gbs": ub[u] / (ms_u / 1e3) / 1e9, "hbm_frac": ub[u] / (ms_u / 1e3) / 1e9 / hbm_peak}
    roofline["units"] = units
    y_ref = [y_dev[0].clone(), y_dev[-1].clone()]
    del p, g, y_dev

    # ---- e2e: host pinned buffers through the C ABI, capped budget, streamed
    x_host = torch.empty((n, 1, H, W), dtype=torch.float32).pin_memory()
    x_host.copy_(x_dev)
    del x_dev
    y_host = torch.empty(out_shape, dtype=torch.float32).pin_memory()
    g2 = build_graph(tg, wl, x_host, y_host, False, params)
    g2.set(budget=wl["budget"], torch_runtime=True, precision=args.precision_code,
           max_chunk_px=args.max_chunk_px, depth=args.depth)
    p2 = g2.plan()
    st = p2.stats()
    js = p2.json()
    cs2 = p2.compute_stream(local)
    for _ in range(args.warmup):
        p2.execute()
    torch.cuda.synchronize()
    # the streamed result equals the device-resident one bit for bit (same kernels, same order)
    assert torch.equal(y_host[0].to(dev), y_ref[0]) and torch.equal(y_host[-1].to(dev), y_ref[1]), \
        "streamed != resident"
    del y_ref
    # the e2e number is timed with the library's per-launch profiling OFF (its events cost up to
    # 25 % of a streamed step); a second, profiled pass of the same steps gives the breakdown
    # (kernel / copy busy times, overlap) reported beside it
    l2 = p2.launches()
    barrier(world)
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    f0.record(cs2)
    for _ in range(args.steps):
        p2.execute(blocking=False)
    f1.record(cs2)
    torch.cuda.synchronize()
    wall = (time.perf_counter() - t0) / args.steps
    ms2 = f0.elapsed_time(f1) / args.steps
    launches2 = p2.launches() - l2
    ms2_max = max_over_ranks(ms2, world)
    p2.profiling(True)
    g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    g0.record(cs2)
    for _ in range(args.steps):
        p2.execute(blocking=False)
    g1.record(cs2)
    torch.cuda.synchronize()
    ms2_prof = g0.elapsed_time(g1) / args.steps
    tim2 = p2.timing()
    p2.profiling(False)
    e2e_value = world * px / (ms2_max / 1e3) / 1e6
    # parameters stay resident after the first execution: a timed step moves the images,
    # the streamed bias rows (if any) and the outputs
    h2d, d2h = st["h2d_bytes_steady"], st["d2h_bytes"]
    e2e = {"value": e2e_value, "unit": "Mpixels/s", "ms_per_step": ms2_max, "wall_ms_per_step": wall * 1e3,
           "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
           "io_lower_bound_bytes": st["io_lower_bound_bytes"],
           "bytes_vs_lower_bound": (h2d + d2h) / st["io_lower_bound_bytes"],
           "budget_bytes": wl["budget"], "arena_bytes": st["peak_device_bytes"][0], "chunks": st["n_chunks"],
           "split": js["split"], "bias": js["bias"], "gpu_launches": launches2,
           "profiled_ms_per_step": ms2_prof,
           "kernel_ms_per_step": sum(tim2["kernel_ms"]) / args.steps,
           "h2d_ms_per_step": tim2["h2d_ms"] / args.steps, "d2h_ms_per_step": tim2["d2h_ms"] / args.steps}
    # SURVEY 8(d) overlap = (sum copy + sum kernel - wall) / min(sum copy, sum kernel), with the copy
    # time taken per direction (the two copy engines run concurrently): 1 = the shorter of {busier
    # copy direction, kernels} is completely hidden behind the longer, 0 = fully serialised
    s_copy = max(tim2["h2d_ms"], tim2["d2h_ms"]) / args.steps
    s_kern = sum(tim2["kernel_ms"]) / args.steps
    e2e["overlap"] = (s_copy + s_kern - ms2_prof) / max(min(s_copy, s_kern), 1e-9)
    e2e["overlap_def"] = ("(max(H2D, D2H) busy + kernel busy - step) / min(max(H2D, D2H) busy, kernel busy), "
                          "all from the profiled pass")
    # every rank measures its link at the same time (the concurrent figure is the one that
    # bounds a multi-GPU streamed run: host DRAM and root-complex bandwidth are shared); the
    # denominator is the slowest rank's
    barrier(world)
    link = host_link_peak(local)
    link = {k: min_over_ranks(v, world) for k, v in link.items()}
    if rank == 0:
        # link roofline: each direction at its solo peak, both together at the measured
        # concurrent (bidirectional) rate
        t_link = max(h2d / (link["h2d"] * 1e9), d2h / (link["d2h"] * 1e9),
                     (h2d + d2h) / (2 * link["bidir_each"] * 1e9))
        e2e["host_link"] = {"peak_h2d_gbs": link["h2d"], "peak_d2h_gbs": link["d2h"],
                            "peak_bidir_each_gbs": link["bidir_each"],
                            "achieved_h2d_gbs": (h2d / 1e9) / (ms2 / 1e3),
                            "achieved_d2h_gbs": (d2h / 1e9) / (ms2 / 1e3),
                            "roofline_time_ms": t_link * 1e3, "roofline_frac": t_link / (ms2 / 1e3)}
    desc = (f"{wl['desc']}, {n} x {H}x{W} fp32 images ({px * 4 / 1e9:.2f} GB) per GPU; value: device-resident, "
            f"uncapped; e2e: pinned host buffers, "
            f"{'uncapped' if not wl['budget'] else str(wl['budget'] >> 20) + ' MiB device budget'}, streamed")
    config = {"workload": desc, "template": wl["template"], "images_per_gpu": n, "H": H, "W": W,
              "n5": wl.get("n5"), "budget_bytes_e2e": wl["budget"], "precision": args.precision,
              "l2": f"inputs {px * 4 / 1e9:.2f} GB per step" + (" >> 126 MB L2 (no flush needed)" if px * 4 >= (252 << 20)
                                                               else ": L2 flushed (512 MB write) before every timed step")}
    return {"value": value, "ms_per_step": ms_max, "clocks": clocks, "gpu_launches": launches,
            "roofline": roofline, "e2e": e2e, "config": config, "y_host": y_host}


# ------------------------------------------------------------------------------ CPU leg
def _normwise(g, r) -> float:
    """max over output planes of max|g - r| / max|r| (R16)."""
    import numpy as np
    g = np.asarray(g, np.float64).reshape(-1, r.shape[-2] * r.shape[-1])
    r = np.asarray(r, np.float64).reshape(-1, r.shape[-2] * r.shape[-1])
    return float(max(np.abs(g[i] - r[i]).max() / max(np.abs(r[i]).max(), 1e-30) for i in range(r.shape[0])))


def _cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_oracle_sample(template: str = "edge", target_s: float = 12.0, gpu_out=None, tol: float = 1e-5) -> dict:
    """The CPU oracle (as it stands) on a bounded sample of the workload: for the edge
    template whole 10000x10000 images of configs[1]; for the CNN one image of the workload.
    Reports input Mpx/s. With gpu_out (the GPU run's host output, [n][c][h][w]) the sampled
    images' oracle outputs are also compared with it: outputs verified in the same run."""
    import oracle
    import synth
    oracle.build()
    if template == "edge":
        W = 10000
        seed = synth.seed_for_config(2)
        K1, K2 = synth.edge_filter_np()
        done_px, t_tot, imgs, err = 0, 0.0, 0, 0.0
        while t_tot < target_s and imgs < 15:
            img = synth.image_np(seed, synth.DS_IMAGE, imgs, (10000, W))
            t0 = time.perf_counter()
            E = oracle.edge(img, K1, K2)
            t_tot += time.perf_counter() - t0
            if gpu_out is not None:
                err = max(err, _normwise(gpu_out[imgs, 0], E))
            done_px += img.size
            imgs += 1
        sample = f"oracle.edge on {imgs} whole 10000x10000 images of configs[1] ({t_tot:.1f} s)"
    else:
        wl = workload(template, 0)
        H, W, n5 = wl["H"], wl["W"], wl["n5"]
        prm = synth.cnn_params_np(wl["seed"], n5, H, W)
        img = synth.image_np(wl["seed"], synth.DS_IMAGE, 0, (H, W))
        t0 = time.perf_counter()
        ref = oracle.cnn(img, n5, prm)
        t_tot = time.perf_counter() - t0
        err = _normwise(gpu_out[0:1], ref) if gpu_out is not None else 0.0
        imgs = 1
        done_px = H * W
        sample = f"oracle.cnn on one {H}x{W} image of the workload ({t_tot:.1f} s)"
    out = {"value": done_px / t_tot / 1e6, "unit": "Mpixels/s", "cores": oracle.num_threads(), "kind": "oracle",
           "sample": sample, "nproc": os.cpu_count(), "cpu_model": _cpu_model()}
    # the same oracle on ONE core (SURVEY 8(d) "and once on 1 core"), on a small crop of the sample
    nt = oracle.num_threads()
    oracle.set_num_threads(1)
    try:
        if template == "edge":
            crop = synth.image_np(seed, synth.DS_IMAGE, 0, (10000, W))[:1000]
            t0 = time.perf_counter()
            oracle.edge(crop, K1, K2)
            t1 = time.perf_counter() - t0
            what = "oracle.edge on the first 1000 rows of one 10000x10000 image"
        else:
            crop = img[:min(H, 480), :min(W, 640)].copy()
            cprm = synth.cnn_params_np(wl["seed"], n5, crop.shape[0], crop.shape[1])
            t0 = time.perf_counter()
            oracle.cnn(crop[None, None], n5, cprm)
            t1 = time.perf_counter() - t0
            what = f"oracle.cnn on a {crop.shape[0]}x{crop.shape[1]} crop"
        out["single_core"] = {"value": crop.size / t1 / 1e6, "unit": "Mpixels/s", "sample": f"{what} ({t1:.1f} s)"}
    finally:
        oracle.set_num_threads(nt)
    if gpu_out is not None:
        out["verified"] = {"images": imgs, "max_normwise_err": err, "tol": tol, "ok": err <= tol,
                           "what": "the sampled images' oracle outputs vs this run's streamed GPU outputs"}
    return out


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    wl = workload(args.template, 0)
    for _ in range(min(args.warmup, 1)):
        cpu_oracle_sample(args.template, 1.0)
    vals = [cpu_oracle_sample(args.template, 8.0) for _ in range(args.steps)]
    v = statistics.median([x["value"] for x in vals])
    px = wl["n"] * wl["H"] * wl["W"]
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "Mpixels/s",
            "n_gpus": int(args.gpus), "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": px / (v * 1e6) * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32 (fp64 accumulation)", "data": "synthetic",
            "config": {"workload": f"{wl['desc']}, {wl['n']} x {wl['H']}x{wl['W']} per GPU; the CPU oracle "
                                   f"(oracle/oracle.c, OpenMP) timed on a bounded sample of it",
                       "template": wl["template"]},
            "cpu_baseline": {"kind": "oracle", "cores": vals[0]["cores"], "sample": vals[-1]["sample"], "value": v},
            "e2e": {"value": v, "unit": "Mpixels/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--template", default="edge", choices=["edge", "cnn4", "cnn3", "cnn3s"])
    ap.add_argument("--precision", default="fp32", choices=["fp32", "bf16_tc", "fp32_tc"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--depth", type=int, default=None,
                    help="pipeline slots of the e2e plan (tg_set_chunking; default: the library's 3)")
    ap.add_argument("--max-chunk-px", type=int, default=None,
                    help="chunk cap of the e2e plan (tg_set_chunking; default: the library's 2^25)")
    ap.add_argument("--per-template", default=None,
                    help="extra template:precision runs reported under per_template (default with --template "
                         "edge: cnn4 and cnn3 in fp32, fp32_tc and bf16_tc; 'none' skips them)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        run_reference(args)
        return
    from paper_conf_ipps_sundaramrc09_b200 import tg
    args.precision_code = {"fp32": tg.TG_FP32, "bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}[args.precision]
    rank, world, local = dist_setup(args)
    res = run(args, rank, world, local)
    if rank == 0:
        line = {"metric": METRIC, "value": res["value"], "unit": "Mpixels/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms_per_step"],
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
                "dtype": {"fp32": "f32", "bf16_tc": "bf16 (fp32 accumulate)",
                          "fp32_tc": "f32 (3xFP16 tensor cores, fp32 accumulate)"}[args.precision],
                "data": "synthetic (counter-based generator synth/, 8-bit levels k/255)",
                "config": res["config"], "roofline": res["roofline"], "e2e": res["e2e"], "clocks": res["clocks"],
                "gpu_launches": res["gpu_launches"]}
        if args.template == "edge":
            line["paper_context"] = {"mpx_s": 24.3, "what": "edge 10000x10000, Tesla C870, host-to-host, no overlap "
                                                            "(PAPER.md:753); 25.5 on 8800 GTX"}
        if world == 1 and not args.no_cpu:
            line["cpu_baseline"] = cpu_oracle_sample(args.template, gpu_out=res["y_host"].numpy(),
                                                     tol=2e-2 if args.precision == "bf16_tc" else 1e-5)
    del res
    # the metric is per template: the CNN template's configs (configs[3] cnn4, configs[2] cnn3) in
    # both precisions, measured in the same run (value / e2e / roofline of each; full lines come
    # from `--template cnn4 --precision ...`)
    extra = args.per_template
    if extra is None:
        extra = ("cnn4:fp32,cnn4:fp32_tc,cnn4:bf16_tc,cnn3:fp32,cnn3:fp32_tc,cnn3:bf16_tc"
                 if args.template == "edge" else "none")
    per = []
    for item in ([] if extra == "none" else extra.split(",")):
        t, pr = item.split(":")
        a2 = argparse.Namespace(**vars(args))
        a2.template, a2.precision = t, pr
        # the CNN batch steps are ~1-2 ms: time at least 20 of them so one host hiccup does not
        # decide the figure (the headline line above keeps exactly --steps)
        a2.steps = max(args.steps, 20)
        a2.precision_code = {"fp32": tg.TG_FP32, "bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}[pr]
        r2 = run(a2, rank, world, local)
        per.append({"template": t, "precision": pr, "steps": a2.steps, "workload": r2["config"]["workload"],
                    "value": r2["value"],
                    "unit": "Mpixels/s", "ms_per_step": r2["ms_per_step"],
                    "e2e": {k: r2["e2e"].get(k) for k in ("value", "ms_per_step", "h2d_bytes_per_step",
                                                         "d2h_bytes_per_step", "bytes_vs_lower_bound", "overlap")}
                           | {"link_roofline_frac": r2["e2e"].get("host_link", {}).get("roofline_frac")},
                    "roofline": {k: r2["roofline"].get(k) for k in ("bound", "achieved", "peak", "unit", "frac",
                                                                     "kernel")},
                    "gpu_launches": r2["gpu_launches"], "clocks": r2["clocks"]})
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
