"""Probe: bidirectional pinned copy throughput vs chunk size and number of streams per direction."""
import torch

torch.cuda.set_device(0)
TOT = 1 << 30
h = torch.empty(TOT // 4, dtype=torch.float32).pin_memory()
hd = torch.empty(TOT // 4, dtype=torch.float32).pin_memory()
d = torch.empty(TOT // 4, dtype=torch.float32, device="cuda")
dd = torch.empty(TOT // 4, dtype=torch.float32, device="cuda")


def run(chunk, nstreams, mode):
    n = chunk // 4
    k = TOT // chunk
    sh = [torch.cuda.Stream() for _ in range(nstreams)]
    sd = [torch.cuda.Stream() for _ in range(nstreams)]
    best = None
    for rep in range(3):
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e0.record()
        ends = []
        for s in sh + sd:
            s.wait_event(e0)
        for i in range(k):
            if mode in ("h2d", "bidir"):
                with torch.cuda.stream(sh[i % nstreams]):
                    d[i * n:(i + 1) * n].copy_(h[i * n:(i + 1) * n], non_blocking=True)
            if mode in ("d2h", "bidir"):
                with torch.cuda.stream(sd[i % nstreams]):
                    hd[i * n:(i + 1) * n].copy_(dd[i * n:(i + 1) * n], non_blocking=True)
        e1 = torch.cuda.Event(enable_timing=True)
        cur = torch.cuda.current_stream()
        for s in sh + sd:
            cur.wait_stream(s)
        e1.record()
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1)
        best = t if best is None else min(best, t)
    print(f"chunk {chunk/1e6:8.1f}MB streams/dir {nstreams} {mode:5s}: {TOT/best/1e6:6.1f} GB/s per direction")


for mode in ("h2d", "d2h", "bidir"):
    for chunk in (1 << 30, 1 << 26, 1 << 24, 1 << 22):
        for ns in (1, 2):
            if chunk == 1 << 30 and ns == 2:
                continue
            run(chunk, ns, mode)
