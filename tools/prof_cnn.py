"""Profiling driver (under ncu on the GPU box): the device-resident CNN step of bench.py
--template cnn3|cnn3s (64 x 480x640; fp32, bf16 = bf16_tc, fp32tc = fp32_tc): two executions."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_sundaramrc09_b200 import tg  # noqa: E402

n5 = int(sys.argv[1]) if len(sys.argv) > 1 else 120
prec = {"bf16": tg.TG_BF16_TC, "fp32tc": tg.TG_FP32_TC}.get(sys.argv[2] if len(sys.argv) > 2 else "", tg.TG_FP32)
n, H, W = 64, 480, 640
seed = synth.seed_for_config(3)
x = synth.images_torch(seed, n, H, W, "cuda:0")
prm = synth.cnn_params_np(seed, n5, H, W)
h5, w5 = synth.cnn_dims(H, W)[4]
y = torch.empty((n, 9, h5, w5), dtype=torch.float32, device="cuda:0")
g, _ = tg.cnn_graph(x, n5, prm, out=y, device=True)
g.set(torch_runtime=True, precision=prec)
p = g.plan()
p.execute()
p.execute()
torch.cuda.synchronize()
print("done", p.launches())
