"""The library's fused planner (C++, tg_plan_dump_json) against the planner oracle
(oracle/planner.fused_chunks): given the chunk size the library chose, every paper-derived
field is bit-exact -- chunk row ranges incl. halos, shards, H2D/D2H bytes, I/O
lower bound and Table 1 totals. The chunk size and slot layout themselves are checked by
properties only (they are the library's memory layout, not the paper's)."""
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


ECHO = ("template", "n", "H", "W", "ks", "n5", "nf", "combine", "budget", "max_chunk_px", "device_io")
PAPER = ("split", "B", "R", "bias", "n_chunks", "chunks", "shard", "h2d_param_bytes", "h2d_chunk_bytes",
         "d2h_bytes", "io_lower_bound_bytes", "io_lower_bound_data_bytes", "total_temp_bytes", "n_ops_fig7",
         "n_ds_fig7")


def oracle_for(tmpl, n, H, W, kw, got):
    """The paper-derived content of a plan, given the library's chunk size (split, B, R) and
    bias mode: row bands and halos, shards, bytes, Table 1 accounting."""
    okw = dict(rank=kw.get("rank", 0), world=kw.get("world", 1), device_io=kw.get("device_io", False))
    if tmpl == "edge":
        okw.update(ks=kw.get("ks", 16), nf=kw.get("orient", 4) // 2, combine=kw.get("comb", "max"))
    else:
        okw.update(n5=kw["n5"])
    return P.fused_chunks(tmpl, n, H, W, got["split"], got["B"], got["R"], bias=got["bias"], **okw)


@pytest.mark.parametrize("case", CASES, ids=[f"{c[0]}-{c[1]}x{c[2]}x{c[3]}-{i}" for i, c in enumerate(CASES)])
def test_plan_matches_oracle(case):
    """Bit-exact on everything the paper fixes once the chunk size is chosen."""
    tmpl, n, H, W, kw = case
    got = library_plan(tmpl, n, H, W, kw)
    want = oracle_for(tmpl, n, H, W, kw, got)
    for k in PAPER:
        assert got[k] == want[k], k
    # the echo of the plan's inputs
    exp = {"template": tmpl, "n": n, "H": H, "W": W, "budget": kw.get("budget", 0),
           "device_io": kw.get("device_io", False), "max_chunk_px": kw.get("max_chunk_px", 1 << 25)}
    for k, v in exp.items():
        assert got[k] == v, k
    if tmpl == "cnn":
        assert got["bias"] in (("resident", "streamed") if kw.get("bias", "plane") == "plane" else ("scalar",))
        assert got["precision"] == kw.get("precision", "fp32")
    else:
        assert got["bias"] == "none" and got["precision"] == "fp32"


def _min_bytes(tmpl, H, W, n5, ch, B, R):
    """The least any layout can hold per buffer: fp32 planes for the input rows, the outputs and
    the streamed bias rows (the paper's DS are fp32 'floats'); T2 / T4 at >= 2
    bytes per channel-pixel (the narrowest type any precision keeps them in)."""
    f = 4
    if tmpl == "edge":
        return {"in": B * (ch["in"][1] - ch["in"][0]) * W * f, "out": B * R * W * f}
    (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5) = synth.cnn_dims(H, W)
    sp = lambda r: r[1] - r[0]   # noqa: E731
    return {"in": B * sp(ch["in"]) * W * f, "t2": B * 8 * sp(ch["t2"]) * w2 * 2, "t4": B * 20 * sp(ch["t4"]) * w4 * 2,
            "out": B * 9 * R * w5 * f, "b1": 8 * sp(ch["c1"]) * w1 * f, "b3": 20 * sp(ch["c3"]) * w3 * f,
            "b5": n5 * R * w5 * f, "b6": 9 * R * w5 * f}


@pytest.mark.parametrize("case", CASES, ids=[f"{c[0]}-{c[1]}x{c[2]}x{c[3]}-{i}" for i, c in enumerate(CASES)])
def test_plan_layout_properties(case):
    """The chunk size and the slot layout are the library's design (not the paper's), checked by
    properties: the arena fits the budget, every buffer a chunk needs is in the
    slot, disjoint and large enough, the chunk is as large as the budget and the documented caps
    allow, and the H2D prediction adds up."""
    tmpl, n, H, W, kw = case
    got = library_plan(tmpl, n, H, W, kw)
    budget, depth = got["budget"], got["depth"]
    assert got["arena_bytes"] == got["param_bytes"] + depth * got["slot_bytes"]
    if budget:
        assert got["arena_bytes"] <= budget
    assert got["h2d_bytes"] == got["h2d_param_bytes"] + got["h2d_derived_bytes"] + got["h2d_chunk_bytes"]
    if not got["device_io"]:
        assert got["param_bytes"] >= got["h2d_param_bytes"] + got["h2d_derived_bytes"]
    assert got["h2d_derived_bytes"] == 0 or got["precision"] in ("bf16_tc", "fp32_tc")
    # buffers: disjoint, ordered inside the slot, each at least the minimum any layout needs for
    # the WIDEST chunk of the plan
    slot = got["slot"]
    spans = sorted(slot.values())
    assert all(0 <= a <= b <= got["slot_bytes"] for a, b in spans)
    assert all(a[1] <= b[0] for a, b in zip(spans, spans[1:]))
    want = {"in", "out"} if not got["device_io"] else set()
    if tmpl == "cnn":
        want |= {"t2", "t4"} | ({"b1", "b3", "b5", "b6"} if got["bias"] == "streamed" else set())
    assert set(slot) == want
    widest = max(got["chunks"], key=lambda c: (c["in"][1] - c["in"][0], c["out"][1] - c["out"][0]))
    mins = _min_bytes(tmpl, H, W, kw.get("n5", 0), widest, got["B"], got["R"])
    for k, (a, b) in slot.items():
        assert b - a >= mins[k], k
    # maximal: the next larger chunk would not fit (unless the cap binds)
    mcp = got["max_chunk_px"]
    h_out = H if tmpl == "edge" else synth.cnn_dims(H, W)[4][0]
    if got["split"] == "batch":
        n_share = -(-n // kw.get("world", 1))
        cap = n if got["device_io"] else min(n, mcp // (H * W), -(-n_share // (2 * depth)))
        assert got["chunk_cap"] == cap and 1 <= got["B"] <= cap
        at_cap = got["B"] == cap
    else:
        cap = min(h_out, max(1, mcp // (W * (1 if tmpl == "edge" else 4))))
        if not got["device_io"]:       # >= 2 x depth chunks in all
            per_img = -(-2 * depth // -(-n // kw.get("world", 1)))
            cap = min(cap, -(-h_out // per_img))
        assert got["chunk_cap"] == cap and 1 <= got["R"] <= cap
        at_cap = got["R"] == cap
    if not at_cap:
        assert budget and got["param_bytes"] + depth * got["slot_bytes_next"] > budget
    else:
        assert got["slot_bytes_next"] == 0


def test_streamed_bias_for_paper_large_cnn():
    """Large CNN at 6400x4800 under the 1.5 GB cap: the 2.6 GB bias set cannot be resident
    (SURVEY §8(c) 7b), so bias rows stream with each chunk; bytes stay within 10 % of the
    I/O bound (north_star)."""
    got = library_plan("cnn", 1, 4800, 6400, dict(n5=120, budget=1536 << 20))
    assert got["bias"] == "streamed" and got["split"] == "rows"
    assert got["h2d_bytes"] + got["d2h_bytes"] <= 1.10 * got["io_lower_bound_bytes"]


def test_edge_plan_reports_fp32_for_any_precision():
    """The edge template has no tensor-core path: its plan is fp32 whatever precision is set
    (a duplicated JSON key once reported the graph's setting instead)."""
    got = library_plan("edge", 2, 300, 200, dict(precision="bf16_tc"))
    assert got["precision"] == "fp32" and got["h2d_derived_bytes"] == 0
