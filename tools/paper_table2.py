"""Table 2 of the paper re-run on one B200: host-resident input -> host
output, seconds per template instance, for the three execution modes of the library:
  baseline  TG_BASELINE (per operator copy in / run / copy out)
  per_op    TG_PER_OP   (the paper's framework: per-operator units, DFS + latest-time-of-use)
  fused     TG_FUSED    (this build: fused offload units, overlapped streaming)
Prints one JSON line per row; the paper's C870 numbers are quoted beside them (context)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_sundaramrc09_b200 import tg  # noqa: E402

PAPER_C870 = {("edge", 1000, 1000): (0.28, 0.036), ("edge", 10000, 10000): (None, 4.12),
              ("small", 480, 640): (1.70, 0.62), ("small", 480, 6400): (6.96, 2.06),
              ("small", 4800, 6400): (54.00, 16.66), ("large", 480, 640): (4.29, 2.57),
              ("large", 480, 6400): (15.71, 6.62), ("large", 4800, 6400): (262.45, 112.99)}


def time_plan(p, reps=3):
    p.execute()
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(reps):
        t0 = time.perf_counter()
        p.execute()
        torch.cuda.synchronize()
        best = min(best, time.perf_counter() - t0)
    return best


def row(kind, H, W):
    seed = 11
    img = torch.empty((1, 1, H, W), dtype=torch.float32).pin_memory()
    img.copy_(synth.images_torch(seed, 1, H, W, "cuda").cpu())
    res = {"template": kind, "H": H, "W": W}
    if kind == "edge":
        K1, _ = synth.edge_filter_np()
        out = torch.empty_like(img).pin_memory()
        build = lambda: tg.edge_graph(img, K1, out=out)[0]  # noqa: E731
    else:
        n5 = 20 if kind == "small" else 120
        prm = synth.cnn_params_np(seed, n5, H, W)
        h5, w5 = synth.cnn_dims(H, W)[4]
        out = torch.empty((1, 9, h5, w5), dtype=torch.float32).pin_memory()
        build = lambda: tg.cnn_graph(img, n5, prm, out=out)[0]  # noqa: E731
    for name, mode in (("baseline", tg.TG_BASELINE), ("per_op", tg.TG_PER_OP), ("fused", tg.TG_FUSED)):
        g = build()
        g.set(torch_runtime=True)
        try:
            p = g.plan(mode)
            s = p.stats()
            res[name] = {"s": time_plan(p), "floats_moved": (s["h2d_bytes"] + s["d2h_bytes"]) // 4}
        except tg.TGError as e:
            res[name] = {"error": str(e)[:120]}
        del g
    res["io_lower_bound_floats"] = s["io_lower_bound_bytes"] // 4
    key = ("edge" if kind == "edge" else kind, H, W)
    res["paper_c870_s"] = {"baseline": PAPER_C870[key][0], "optimized": PAPER_C870[key][1]}
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    torch.cuda.set_device(0)
    for kind, H, W in [("edge", 1000, 1000), ("edge", 10000, 10000), ("small", 480, 640), ("small", 480, 6400),
                       ("small", 4800, 6400), ("large", 480, 640), ("large", 480, 6400), ("large", 4800, 6400)]:
        row(kind, H, W)
