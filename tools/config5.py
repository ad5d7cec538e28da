"""configs[4] of BASELINE.json -- CNN + edge detection over ~400 GB of host-resident input, split
chunks sharded over 8 B200 -- run as ONE GPU's share.

The 8-GPU run partitions the global chunk list into contiguous ranges, one per GPU, with no
collective (tg_set_shard / tg_set_devices). Every GPU's share is an independent
out-of-core problem of 400/G GB input, so this driver runs the share of one GPU at G = 8
(--share 8, the default): 50 GB of 10000x10000 images through the edge template, then 50 GB of
6400x4800 tiles through the large CNN (bias planes shared by all tiles, resident on the GPU),
one after the other. Host RAM bounds the share: if in + out does not fit
in ~85 % of the available memory the image count is scaled down and the JSON says so.

Outputs are checked, without the oracle (tools may not use it), against a device-resident
unsplit run of the first and last image through the same library: split/streamed == unsplit,
bit for bit.

  python tools/config5.py [--share 8] [--total-gb 400] [--precision fp32|fp32_tc|bf16_tc] [--steps 1]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import psutil  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_sundaramrc09_b200 import tg  # noqa: E402


def run_template(name, total_gb, share, precision, steps, dev):
    if name == "edge":
        H, W, seed = 10000, 10000, synth.seed_for_config(5)
        out_per_img = H * W * 4
        params = [synth.edge_filter_np()[0]]
    else:
        H, W, seed = 4800, 6400, synth.seed_for_config(5) + 1
        h5, w5 = synth.cnn_dims(H, W)[4]
        out_per_img = 9 * h5 * w5 * 4
        params = synth.cnn_params_np(seed, 120, H, W)
    in_per_img = H * W * 4
    n_full = int(round(total_gb * 1e9 / share / in_per_img))
    avail = psutil.virtual_memory().available
    n = min(n_full, int(0.85 * avail // (in_per_img + out_per_img)))
    x = torch.empty((n, 1, H, W), dtype=torch.float32).pin_memory()
    y = torch.empty((n, 1, H, W) if name == "edge" else (n, 9, h5, w5), dtype=torch.float32).pin_memory()
    t0 = time.perf_counter()
    B = 4
    for i in range(0, n, B):
        k = min(B, n - i)
        x[i:i + k].copy_(synth.images_torch(seed, k, H, W, dev, n0=i))
    torch.cuda.synchronize()
    gen_s = time.perf_counter() - t0

    def graph(xx, yy, device):
        if name == "edge":
            return tg.edge_graph(xx, params[0], out=yy, device=device)[0]
        return tg.cnn_graph(xx, 120, params, out=yy, device=device)[0]

    g = graph(x, y, False)
    g.set(budget=0, torch_runtime=True, precision=precision)
    p = g.plan()
    st, js = p.stats(), p.json()
    cs = p.compute_stream(dev.index or 0)
    p.execute()  # warm-up: parameters go resident, kernels configured
    torch.cuda.synchronize()
    p.profiling(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record(cs)
    for _ in range(steps):
        p.execute(blocking=False)
    e1.record(cs)
    torch.cuda.synchronize()
    wall = (time.perf_counter() - t0) / steps
    ms = e0.elapsed_time(e1) / steps
    tim = p.timing()
    # split/streamed == unsplit device-resident, bit for bit, on the first and last image
    ok = True
    for i in (0, n - 1):
        xd = x[i:i + 1].to(dev)
        yd = torch.empty((1,) + tuple(y.shape[1:]), dtype=torch.float32, device=dev)
        gd = graph(xd, yd, True)
        gd.set(torch_runtime=True, precision=precision)
        gd.plan().execute()
        torch.cuda.synchronize()
        ok &= bool(torch.equal(yd.cpu(), y[i:i + 1]))
    h2d, d2h = st["h2d_bytes_steady"], st["d2h_bytes"]
    px = n * H * W
    res = {"template": name, "images": n, "images_full_share": n_full, "H": H, "W": W,
           "input_gb": n * in_per_img / 1e9, "output_gb": n * out_per_img / 1e9,
           "scaled_to_host_ram": n < n_full, "host_ram_available_gb": avail / 1e9,
           "value_mpx_s": px / (ms / 1e3) / 1e6, "ms_per_step": ms, "wall_ms_per_step": wall * 1e3,
           "h2d_gbs": h2d / 1e9 / (ms / 1e3), "d2h_gbs": d2h / 1e9 / (ms / 1e3),
           "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
           "bytes_vs_lower_bound": (h2d + d2h) / st["io_lower_bound_bytes"],
           "chunks": st["n_chunks"], "split": js["split"], "bias": js.get("bias"),
           "kernel_ms_per_step": sum(tim["kernel_ms"]) / steps, "h2d_ms_per_step": tim["h2d_ms"] / steps,
           "d2h_ms_per_step": tim["d2h_ms"] / steps, "generate_s": gen_s,
           "split_equals_unsplit_first_last_image": ok}
    del p, g, x, y
    torch.cuda.empty_cache()
    if hasattr(torch._C, "_host_emptyCache"):
        torch._C._host_emptyCache()  # release the cached pinned host blocks for the next template
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--share", type=int, default=8, help="G: this process runs 1/G of the images")
    ap.add_argument("--total-gb", type=float, default=400.0)
    ap.add_argument("--precision", default="fp32", choices=["fp32", "fp32_tc", "bf16_tc"])
    ap.add_argument("--steps", type=int, default=1)
    ap.add_argument("--templates", default="edge,cnn")
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    prec = {"fp32": tg.TG_FP32, "fp32_tc": tg.TG_FP32_TC, "bf16_tc": tg.TG_BF16_TC}[args.precision]
    out = {"config": "configs[4]: CNN + edge over ~400 GB host-resident input, split chunks sharded over 8 B200",
           "run": f"one GPU's share (1/{args.share}) of {args.total_gb:g} GB per template, uncapped budget, "
                  f"precision {args.precision}", "gpu": torch.cuda.get_device_name(0), "results": []}
    for t in args.templates.split(","):
        out["results"].append(run_template(t, args.total_gb, args.share, prec, args.steps, dev))
        print(json.dumps(out["results"][-1]), file=sys.stderr, flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
