"""Error of the fp32-accurate tensor-core CNN path (TG_FP32_TC, 3xFP16) vs the FFMA path (TG_FP32), both against the
oracle, per case: normwise per plane and absolute. Test infrastructure (loads the oracle)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))), "tests"))
import numpy as np
import torch
import synth, oracle
from paper_conf_ipps_sundaramrc09_b200 import tg

def run(img, n5, prm, prec):
    n, _, H, W = img.shape
    h5, w5 = synth.cnn_dims(H, W)[4]
    out = np.zeros((n, 9, h5, w5), np.float32)
    g, _ = tg.cnn_graph(img, n5, prm, out=out)
    g.set(torch_runtime=True, precision=prec)
    g.plan().execute()
    return out

def nw(o, r):
    o = o.astype(np.float64)
    e = np.abs(o - r).reshape(o.shape[0] * o.shape[1], -1).max(1)
    m = np.abs(r).reshape(o.shape[0] * o.shape[1], -1).max(1)
    return (e / m).max(), np.abs(o - r).max()

for (n, H, W, n5) in [(2, 32, 32, 7), (2, 32, 32, 20), (2, 36, 40, 7), (1, 120, 160, 120), (2, 92, 100, 20)]:
    seed = synth.seed_for_config(3) + 29
    img = synth.images_np(seed, n, H, W)
    prm = synth.cnn_params_np(seed, n5, H, W)
    ref = oracle.cnn(img, n5, prm)
    a = run(img, n5, prm, tg.TG_FP32)
    b = run(img, n5, prm, tg.TG_FP32_TC)
    print((n, H, W, n5), "fp32", nw(a, ref), "fp32_tc", nw(b, ref), "|ref|max", np.abs(ref).max(), flush=True)
