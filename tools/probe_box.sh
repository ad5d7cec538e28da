#!/bin/bash
# One-off probe of the GPU box: host RAM, cores, CPU model, GPU topology, pinned host-link bandwidth.
set -x
nproc; free -g; lscpu | head -20; nvidia-smi; nvidia-smi topo -m; numactl -H 2>/dev/null | head
python - <<'PY'
import torch, time
d = torch.device('cuda:0')
for gib in [1]:
    n = gib << 28
    h = torch.empty(n, dtype=torch.float32).pin_memory()
    g = torch.empty(n, dtype=torch.float32, device=d)
    h2 = torch.empty(n, dtype=torch.float32).pin_memory()
    s1 = torch.cuda.Stream(); s2 = torch.cuda.Stream()
    for name in ['h2d','d2h','bidir']:
        best = 1e9
        for _ in range(5):
            g2 = g if name != 'bidir' else torch.empty_like(g)
            torch.cuda.synchronize(); t = time.perf_counter()
            if name in ('h2d','bidir'):
                with torch.cuda.stream(s1): g.copy_(h, non_blocking=True)
            if name in ('d2h','bidir'):
                with torch.cuda.stream(s2): h2.copy_(g2 if name=='bidir' else g, non_blocking=True)
            torch.cuda.synchronize(); best = min(best, time.perf_counter()-t)
        b = n*4*(2 if name=='bidir' else 1)
        print(name, 'GB/s', b/best/1e9)
PY
