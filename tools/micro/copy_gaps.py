"""Probe: gaps between back-to-back pinned H2D copies on one stream (sizes of the edge and CNN
chunks), alone and with a concurrent D2H stream, with and without events between copies."""
import torch

torch.cuda.set_device(0)


def run(nbytes, k, with_events, concurrent_d2h):
    n = nbytes // 4
    h = torch.empty(n * k, dtype=torch.float32).pin_memory()
    d = torch.empty(n * 3, dtype=torch.float32, device="cuda")
    hd = torch.empty(n * k, dtype=torch.float32).pin_memory()
    dd = torch.empty(n, dtype=torch.float32, device="cuda")
    s0, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    evs = []
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s0)
    s2.wait_event(e0)
    for i in range(k):
        with torch.cuda.stream(s0):
            if with_events:
                a = torch.cuda.Event(enable_timing=True); a.record(s0)
            d[(i % 3) * n:(i % 3 + 1) * n].copy_(h[i * n:(i + 1) * n], non_blocking=True)
            if with_events:
                b = torch.cuda.Event(enable_timing=True); b.record(s0); evs.append((a, b))
        if concurrent_d2h:
            with torch.cuda.stream(s2):
                hd[i * n:(i + 1) * n].copy_(dd, non_blocking=True)
    e1.record(s0)
    torch.cuda.synchronize()
    tot = e0.elapsed_time(e1)
    busy = sum(a.elapsed_time(b) for a, b in evs) if evs else float("nan")
    gaps = [evs[i][1].elapsed_time(evs[i + 1][0]) for i in range(len(evs) - 1)] if evs else []
    print(f"bytes {nbytes/1e6:.1f}MB k {k} events {with_events} d2h {concurrent_d2h}: total {tot:.3f} ms "
          f"rate {nbytes*k/tot/1e6:.1f} GB/s busy {busy:.3f} mean_gap {sum(gaps)/max(1,len(gaps))*1e3:.1f} us")


for nb in (67_000_000, 13_500_000, 3_400_000):
    for ev in (False, True):
        for cc in (False, True):
            run(nb, 12, ev, cc)
