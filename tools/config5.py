"""configs[4] of BASELINE.json -- CNN + edge detection over ~400 GB of host-resident input, split
chunks sharded over 8 B200 -- run as rank `--rank` of `--world` of the GLOBAL workload.

The global workloads are 1000 x 10000x10000 edge images (400 GB in, 400 GB out) and 3256 x
6400x4800 large-CNN tiles (400 GB in, ~223 GB out), each ONE plan over all images. Every GPU
executes its contiguous range of the global chunk list (tg_set_shard(rank, world))
with no collective. This process is one of those ranks: it binds to its GPU's NUMA node, pins
host buffers holding ONLY its shard's images (the library touches nothing else of the nominal
400 GB arrays: tg.h tg_set_shard), streams them through the fused units with an uncapped
budget, and reports host RAM, the pinning cost and the bytes moved against the lower bound.
Bias planes are shared by all tiles and resident on the GPU.

Outputs are checked, without the oracle (tools may not use it), against a device-resident
unsplit run of the shard's first and last image through the same library: split/streamed ==
unsplit, bit for bit.

  python tools/config5.py [--rank 0] [--world 8] [--total-gb 400] [--precision fp32|fp32_tc|bf16_tc]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import psutil  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402  (NUMA binding and graph building helpers; no oracle)
import synth  # noqa: E402
from paper_conf_ipps_sundaramrc09_b200 import tg  # noqa: E402


def run_template(name, total_gb, rank, world, precision, steps, dev):
    if name == "edge":
        wl = dict(template="edge", H=10000, W=10000, seed=synth.seed_for_config(5))
        out_per_img = wl["H"] * wl["W"] * 4
    else:
        wl = dict(template="cnn", H=4800, W=6400, n5=120, bias="plane", seed=synth.seed_for_config(5) + 1)
        h5, w5 = synth.cnn_dims(wl["H"], wl["W"])[4]
        out_per_img = 9 * h5 * w5 * 4
    H, W = wl["H"], wl["W"]
    in_per_img = H * W * 4
    n_glob = int(round(total_gb * 1e9 / in_per_img))
    params = bench.params_of(wl)
    # the global plan and this rank's shard of it
    g0 = bench.make_graph(tg, wl, n_glob, 0x1000, 0x2000, False, params, prec=precision, shard=(rank, world))
    j0 = g0.plan().json()
    _, _, c0, c1 = j0["shard"]
    mine = j0["chunks"][c0:c1]
    i0 = min(c["img"] for c in mine)
    i1 = max(c["img"] + c["nimg"] for c in mine)
    n = i1 - i0
    vm = psutil.virtual_memory()
    need = n * (in_per_img + out_per_img)
    if need > 0.85 * vm.available:
        raise SystemExit(f"host RAM: the shard needs {need / 1e9:.1f} GB pinned, {vm.available / 1e9:.1f} GB available")
    t0 = time.perf_counter()
    x = torch.empty((n, 1, H, W), dtype=torch.float32).pin_memory()
    oshape = (n, 1, H, W) if name == "edge" else (n, 9, h5, w5)
    y = torch.empty(oshape, dtype=torch.float32).pin_memory()
    pin_s = time.perf_counter() - t0
    t0 = time.perf_counter()
    B = 4
    for i in range(0, n, B):
        k = min(B, n - i)
        x[i:i + k].copy_(synth.images_torch(wl["seed"], k, H, W, dev, n0=i0 + i))
    torch.cuda.synchronize()
    gen_s = time.perf_counter() - t0
    xb = x.data_ptr() - i0 * in_per_img
    yb = y.data_ptr() - i0 * out_per_img
    g = bench.make_graph(tg, wl, n_glob, xb, yb, False, params, prec=precision, shard=(rank, world))
    g._keep += [x, y]
    p = g.plan()
    st, js = p.stats(), p.json()
    assert js["chunks"] == j0["chunks"]
    cs = p.compute_stream(dev.index or 0)
    t0 = time.perf_counter()
    p.execute()  # first execution: parameters go resident (bias planes: 2.6 GB for the CNN)
    torch.cuda.synchronize()
    first_s = time.perf_counter() - t0
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with bench.ClockSampler(dev.index or 0) as clk:
        t0 = time.perf_counter()
        e0.record(cs)
        for _ in range(steps):
            p.execute(blocking=False)
        e1.record(cs)
        torch.cuda.synchronize()
        wall = (time.perf_counter() - t0) / steps
    ms = e0.elapsed_time(e1) / steps
    # split/streamed == unsplit device-resident, bit for bit, on the shard's first and last image
    ok = True
    for i in (0, n - 1):
        xd = x[i:i + 1].to(dev)
        yd = torch.empty((1,) + tuple(y.shape[1:]), dtype=torch.float32, device=dev)
        gd = bench.make_graph(tg, wl, 1, xd.data_ptr(), yd.data_ptr(), True, params, prec=precision)
        gd._keep += [xd, yd]
        gd.plan().execute()
        torch.cuda.synchronize()
        ok &= bool(torch.equal(yd.cpu(), y[i:i + 1]))
    h2d, d2h = st["h2d_bytes_steady"], st["d2h_bytes"]
    px = n * H * W
    res = {"template": name, "global_images": n_glob, "global_input_gb": n_glob * in_per_img / 1e9,
           "global_chunks": st["n_chunks"], "rank": rank, "world": world,
           "shard_chunks": [st["chunk_begin"], st["chunk_end"]], "shard_images": [i0, i1],
           "input_gb": n * in_per_img / 1e9, "output_gb": n * out_per_img / 1e9,
           "host_ram_total_gb": vm.total / 1e9, "host_ram_available_gb": vm.available / 1e9,
           "pinned_gb": need / 1e9, "pin_s": pin_s, "pin_gbs": need / 1e9 / max(pin_s, 1e-9),
           "generate_s": gen_s, "first_execution_s": first_s,
           "value_mpx_s": px / (ms / 1e3) / 1e6, "ms_per_step": ms, "wall_ms_per_step": wall * 1e3,
           "h2d_gbs": h2d / 1e9 / (ms / 1e3), "d2h_gbs": d2h / 1e9 / (ms / 1e3),
           "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
           "io_lower_bound_data_bytes_shard": n * (in_per_img + out_per_img),
           "bytes_vs_lower_bound": (h2d + d2h) / (n * (in_per_img + out_per_img)),
           "host_registered_bytes": st["host_registered_bytes"],
           "split": js["split"], "bias": js.get("bias"), "arena_bytes": st["peak_device_bytes"][0],
           "gpu_launches_per_step": None, "clocks": clk.summary(),
           "split_equals_unsplit_first_last_image": ok}
    del p, g, x, y
    torch.cuda.empty_cache()
    if hasattr(torch._C, "_host_emptyCache"):
        torch._C._host_emptyCache()  # release the cached pinned host blocks for the next template
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rank", type=int, default=0)
    ap.add_argument("--world", type=int, default=8)
    ap.add_argument("--total-gb", type=float, default=400.0)
    ap.add_argument("--precision", default="fp32", choices=["fp32", "fp32_tc", "bf16_tc"])
    ap.add_argument("--steps", type=int, default=1)
    ap.add_argument("--templates", default="edge,cnn")
    args = ap.parse_args()
    torch.cuda.set_device(0)
    numa = bench.numa_bind(0)
    dev = torch.device("cuda:0")
    prec = {"fp32": tg.TG_FP32, "fp32_tc": tg.TG_FP32_TC, "bf16_tc": tg.TG_BF16_TC}[args.precision]
    link = bench.host_link_peak(0)
    out = {"config": "configs[4]: CNN + edge over ~400 GB host-resident input, split chunks sharded over 8 B200",
           "run": f"rank {args.rank} of {args.world} of the global {args.total_gb:g} GB workload per template "
                  f"(tg_set_shard), uncapped budget, precision {args.precision}",
           "gpu": torch.cuda.get_device_name(0), "numa": numa, "host_link_gbs": link, "results": []}
    for t in args.templates.split(","):
        out["results"].append(run_template(t, args.total_gb, args.rank, args.world, prec, args.steps, dev))
        print(json.dumps(out["results"][-1]), file=sys.stderr, flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
