"""Profiling driver (run under ncu on the GPU box): the bench's device-resident edge step
(15 x 10000^2 images, one K1 launch per step), a warm-up execution and one profiled one."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_sundaramrc09_b200 import tg  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 15
H = W = 10000
x = synth.images_torch(synth.seed_for_config(2), n, H, W, "cuda:0")
y = torch.empty_like(x)
K1, _ = synth.edge_filter_np()
g, _ = tg.edge_graph(x, K1, out=y, device=True)
g.set(torch_runtime=True)
p = g.plan()
p.execute()
p.execute()
torch.cuda.synchronize()
print("done", p.launches())
