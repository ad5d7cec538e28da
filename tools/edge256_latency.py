"""configs[0] latency anatomy: one 256x256 edge image, device-resident and host-to-host.
Prints host microseconds per execute call (enqueue only), device microseconds per step (CUDA
events over 2000 back-to-back steps) and the kernel's own time (profiled pass), graph on and off.

  python tools/edge256_latency.py
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch
    import bench
    from paper_conf_ipps_sundaramrc09_b200 import tg
    wl = bench.workload("edge256")
    params = bench.params_of(wl)
    dev = torch.device("cuda:0")
    x = torch.rand((1, 1, 256, 256), device=dev)
    y = torch.empty_like(x)
    out = {}
    for graph in (False, True):
        g = bench.make_graph(tg, wl, 1, x.data_ptr(), y.data_ptr(), True, params)
        p = g.plan()
        p.use_graph(graph)
        cs = torch.cuda.current_stream()
        for _ in range(20):
            p.execute(blocking=False)
        torch.cuda.synchronize()
        n = 2000
        t0 = time.perf_counter()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(cs)
        for _ in range(n):
            p.execute(blocking=False)
        e1.record(cs)
        host_us = (time.perf_counter() - t0) / n * 1e6
        torch.cuda.synchronize()
        dev_us = e0.elapsed_time(e1) / n * 1e3
        p.use_graph(False)
        p.profiling(True, copies=False)
        for _ in range(200):
            p.execute(blocking=False)
        torch.cuda.synchronize()
        tm = p.timing()
        p.profiling(False)
        k_us = sum(tm["kernel_ms"]) / 200 * 1e3
        out["graph" if graph else "direct"] = {"host_us_per_call": host_us, "device_us_per_step": dev_us,
                                               "kernel_us_profiled": k_us}
        del p, g
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
