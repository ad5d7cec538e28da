import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import synth
from paper_conf_ipps_sundaramrc09_b200 import tg
H, W = (int(sys.argv[1]), int(sys.argv[2])) if len(sys.argv) > 2 else (37, 41)
img = synth.images_np(1, 1, H, W)
K1, K2 = synth.random_edge_filters_np(1)
out = np.zeros_like(img)
g, _ = tg.edge_graph(img, K1, K2, out=out)
p = g.plan()
p.execute()
print("ok", H, W, float(np.abs(out).max()))
