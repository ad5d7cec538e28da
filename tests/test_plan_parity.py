"""The library's planner (C++, tg_plan_dump_json) reproduces the planner oracle's fused
chunk rule (oracle/planner.fused_plan) bit-exactly: chunk row ranges incl. halos, slot and
arena sizes, predicted H2D/D2H bytes, I/O lower bound, Table 1 totals, shards."""
import numpy as np
import pytest

import synth
from oracle import planner as P

CASES = [
    # template, n, H, W, kwargs
    ("edge", 1, 256, 256, dict()),
    ("edge", 1, 1000, 1000, dict()),
    ("edge", 15, 10000, 10000, dict(budget=768 << 20)),
    ("edge", 15, 10000, 10000, dict()),
    ("edge", 3, 37, 41, dict(budget=20000, max_chunk_px=512)),
    ("edge", 64, 256, 256, dict(budget=8 << 20)),
    ("edge", 7, 300, 200, dict(budget=2_000_000, depth=2)),
    ("edge", 2, 100, 120, dict(ks=5, budget=60000)),
    ("edge", 4, 1000, 1000, dict(device_io=True)),
    ("edge", 15, 10000, 10000, dict(budget=768 << 20, rank=3, world=8)),
    ("cnn", 64, 480, 640, dict(n5=20)),
    ("cnn", 64, 480, 640, dict(n5=120, bias="scalar")),
    ("cnn", 1, 4800, 6400, dict(n5=120, budget=1536 << 20)),
    ("cnn", 1, 4800, 6400, dict(n5=20, budget=1536 << 20)),
    ("cnn", 1, 4800, 6400, dict(n5=120)),
    ("cnn", 26, 480, 640, dict(n5=120, budget=1536 << 20)),
    ("cnn", 3, 483, 643, dict(n5=120, budget=40 << 20, max_chunk_px=200000)),
    ("cnn", 5, 120, 100, dict(n5=20, budget=3 << 20)),
    ("cnn", 2, 480, 6400, dict(n5=20, device_io=True)),
    ("cnn", 64, 480, 640, dict(n5=120, device_io=True, budget=2 << 30)),
    ("cnn", 1, 4800, 6400, dict(n5=120, budget=1536 << 20, rank=1, world=2)),
    ("cnn", 64, 480, 640, dict(n5=120, precision="bf16_tc")),
    ("edge", 2, 500, 400, dict(orient=8, comb="max", budget=2_000_000)),
    ("edge", 1, 300, 200, dict(orient=8, comb="sum")),
    ("edge", 3, 100, 64, dict(orient=2, comb="maxabs", budget=90_000)),
    ("edge", 1, 64, 64, dict(orient=4, comb="maxabs")),
    ("cnn", 1, 4800, 6400, dict(n5=120, budget=1536 << 20, precision="bf16_tc")),
    ("cnn", 3, 200, 180, dict(n5=37, budget=2_000_000, precision="bf16_tc")),
    ("cnn", 64, 480, 640, dict(n5=120, precision="fp32_tc")),
    ("cnn", 1, 4800, 6400, dict(n5=120, budget=1536 << 20, precision="fp32_tc")),
    ("cnn", 3, 200, 180, dict(n5=37, budget=2_000_000, precision="fp32_tc")),
    ("cnn", 64, 480, 640, dict(n5=120, device_io=True, budget=2 << 30, precision="fp32_tc")),
]


def library_plan(tmpl, n, H, W, kw):
    from paper_conf_ipps_sundaramrc09_b200 import tg
    dev = kw.get("device_io", False)
    if dev:
        # device-resident I/O: planning never dereferences the pointers
        g = tg.Graph()
        x = tg.tg_input_device(g.h, n, 1, H, W, 0x1000)
    else:
        g = tg.Graph()
        img = np.zeros((1, 1, 1, 1), np.float32)          # pointer only; never read when planning
        x = tg.tg_input(g.h, n, 1, H, W, img.ctypes.data)
        g._keep.append(img)
    if tmpl == "edge":
        ks = kw.get("ks", 16)
        k1 = g.param(np.ones((1, 1, ks, ks), np.float32))
        comb = {"max": tg.TG_MAX, "sum": tg.TG_SUM, "maxabs": tg.TG_MAXABS}[kw.get("comb", "max")]
        y = g.find_edges(x, k1, kw.get("orient", 4), comb)
    else:
        n5 = kw["n5"]
        bias = kw.get("bias", "plane")
        shapes = [(8, 1, 5, 5), None, (8, 2, 2), (20, 8, 5, 5), None, (20, 2, 2), (n5, 20, 5, 5), None, (9, n5, 1, 1), None]
        (h1, w1), _, (h3, w3), _, (h5, w5) = synth.cnn_dims(H, W)
        if bias == "plane":
            bs = [(1, 8, h1, w1), (1, 20, h3, w3), (1, n5, h5, w5), (1, 9, h5, w5)]
        else:
            bs = [(8,), (20,), (n5,), (9,)]
        shapes[1], shapes[4], shapes[7], shapes[9] = bs
        dummy = np.zeros(1, np.float32)
        g._keep.append(dummy)
        ids = []
        for s in shapes:
            d = (1,) * (4 - len(s)) + tuple(s)
            ids.append(tg.tg_param(g.h, *d, dummy.ctypes.data))
        y = g.cnn(x, n5, ids, tg.TG_BIAS_PLANE if bias == "plane" else tg.TG_BIAS_SCALAR)
    if dev:
        tg.tg_output_device(g.h, y, 0x2000)
    else:
        out = np.zeros(1, np.float32)
        g._keep.append(out)
        tg.tg_output(g.h, y, out.ctypes.data)
    # chunking left unset unless the case sets it: the library's default meets the oracle's
    g.set(budget=kw.get("budget", 0), max_chunk_px=kw.get("max_chunk_px"), depth=kw.get("depth"),
          shard=(kw.get("rank", 0), kw.get("world", 1)),
          precision={"bf16_tc": tg.TG_BF16_TC, "fp32_tc": tg.TG_FP32_TC}.get(kw.get("precision"), tg.TG_FP32))
    return g.plan().json()


@pytest.mark.parametrize("case", CASES, ids=[f"{c[0]}-{c[1]}x{c[2]}x{c[3]}-{i}" for i, c in enumerate(CASES)])
def test_plan_matches_oracle(case):
    tmpl, n, H, W, kw = case
    got = library_plan(tmpl, n, H, W, kw)
    okw = {k: v for k, v in kw.items() if k not in ("orient", "comb")}
    if tmpl == "edge":
        okw["nf"] = kw.get("orient", 4) // 2
        okw["combine"] = kw.get("comb", "max")
    want = P.fused_plan(tmpl, n, H, W, **okw)
    assert set(got) == set(want)
    for k in want:
        if k == "chunks":
            assert len(got[k]) == len(want[k])
            for a, b in zip(got[k], want[k]):
                assert a == b
        else:
            assert got[k] == want[k], k
