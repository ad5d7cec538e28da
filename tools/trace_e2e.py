"""Timeline of the streamed (host pinned) execution of a bench workload, from tg_plan_trace_get:
per stream busy time and idle gaps, pipelined back-to-back executions. Writes the records to
gpurun_out/trace_<template>_<precision>.json and prints a summary."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_ipps_sundaramrc09_b200 import tg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--template", default="cnn3")
ap.add_argument("--precision", default="bf16_tc")
ap.add_argument("--execs", type=int, default=3)
ap.add_argument("--depth", type=int, default=None)
ap.add_argument("--max-chunk-px", type=int, default=None)
ap.add_argument("--device", action="store_true", help="device-resident I/O instead of pinned host")
ap.add_argument("--tag", default="")
ap.add_argument("--n", type=int, default=None, help="override the number of images")
a = ap.parse_args()
torch.cuda.set_device(0)
wl = bench.workload(a.template)
n, H, W = a.n or wl["n"], wl["H"], wl["W"]
params = bench.params_of(wl)
if wl["template"] == "edge":
    out_shape = (n, 1, H, W)
else:
    out_shape = (n, 9) + tuple(synth.cnn_dims(H, W)[4])
if a.device:
    x = synth.images_torch(wl["seed"], n, H, W, "cuda")
    y = torch.empty(out_shape, dtype=torch.float32, device="cuda")
else:
    x = torch.empty((n, 1, H, W), dtype=torch.float32).pin_memory()
    x.copy_(synth.images_torch(wl["seed"], n, H, W, "cuda").cpu())
    y = torch.empty(out_shape, dtype=torch.float32).pin_memory()
g = bench.make_graph(tg, wl, n, x.data_ptr(), y.data_ptr(), a.device, params,
                     budget=0 if a.device else wl["budget"],
                     prec={"fp32": tg.TG_FP32, "fp32_tc": tg.TG_FP32_TC, "bf16_tc": tg.TG_BF16_TC}[a.precision],
                     chunking={"max_chunk_px": a.max_chunk_px, "depth": a.depth})
g._keep += [x, y]
p = g.plan()
for _ in range(3):
    p.execute()
p.profiling(True)
for _ in range(a.execs):
    p.execute(blocking=False)
torch.cuda.synchronize()
tr = p.trace()
# executions are enqueued in order: number the records of each (kind, chunk) by execution
seen = {}
for r in tr:
    k = (r["kind"], r["chunk"])
    r["exec"] = seen.get(k, 0)
    seen[k] = r["exec"] + 1
os.makedirs("gpurun_out", exist_ok=True)
json.dump(tr, open(f"gpurun_out/trace_{a.template}_{a.precision}{a.tag}.json", "w"))
t_end = max(r["t1_ms"] for r in tr)
print(json.dumps({"chunks": p.stats()["n_chunks"], "execs": a.execs, "span_ms": t_end,
                  "ms_per_exec": t_end / a.execs}))
for kind in sorted({r["kind"] for r in tr}):
    iv = sorted((r["t0_ms"], r["t1_ms"]) for r in tr if r["kind"] == kind)
    busy = sum(b - a_ for a_, b in iv)
    gaps = [round(b[0] - a_[1], 3) for a_, b in zip(iv, iv[1:])]
    print(kind, "n", len(iv), "busy_ms", round(busy, 3), "first", round(iv[0][0], 3), "last_end",
          round(iv[-1][1], 3), "max_gap", max(gaps) if gaps else 0, "gaps", gaps[:24])
