"""e2e step time of a bench workload with and without the library's profiling events, and the
host time spent enqueueing one step (is the streamed pipeline host-bound?)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_ipps_sundaramrc09_b200 import tg  # noqa: E402

torch.cuda.set_device(0)
template = sys.argv[1] if len(sys.argv) > 1 else "cnn3"
for prec_name in sys.argv[2:] or ["bf16_tc", "fp32_tc"]:
    prec = {"fp32": tg.TG_FP32, "fp32_tc": tg.TG_FP32_TC, "bf16_tc": tg.TG_BF16_TC}[prec_name]
    wl = bench.workload(template, 0)
    n, H, W = wl["n"], wl["H"], wl["W"]
    if wl["template"] == "edge":
        params = [synth.edge_filter_np()[0]]
        out_shape = (n, 1, H, W)
    else:
        params = synth.cnn_params_np(wl["seed"], wl["n5"], H, W)
        out_shape = (n, 9) + tuple(synth.cnn_dims(H, W)[4])
    x = torch.empty((n, 1, H, W), dtype=torch.float32).pin_memory()
    x.copy_(synth.images_torch(wl["seed"], n, H, W, "cuda").cpu())
    y = torch.empty(out_shape, dtype=torch.float32).pin_memory()
    g = bench.build_graph(tg, wl, x, y, False, params)
    g.set(budget=wl["budget"], torch_runtime=True, precision=prec)
    p = g.plan()
    cs = p.compute_stream(0)
    for _ in range(3):
        p.execute()
    for prof in (False, True, True, False):
        p.profiling(prof)
        K = 10
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        f0.record(cs)
        host = []
        for _ in range(K):
            t0 = time.perf_counter()
            p.execute(blocking=False)
            host.append(time.perf_counter() - t0)
        f1.record(cs)
        torch.cuda.synchronize()
        ms = f0.elapsed_time(f1) / K
        print(f"{template} {prec_name} profiling={prof}: {ms:.3f} ms/step = {n * H * W / ms / 1e3:.0f} Mpx/s; "
              f"host enqueue {1e3 * sum(host) / K:.3f} ms/step (max {1e3 * max(host):.3f})", flush=True)
        if prof:
            p.timing()
    del p, g
