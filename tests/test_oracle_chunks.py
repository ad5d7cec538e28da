"""The fused chunk rule (oracle/planner.fused_plan) and halo back-propagation, checked by
executing every chunk of a plan on the ORACLE and comparing with the unsplit oracle
bit-exactly (splitting must not change results), plus structural
properties (coverage, maximality, budget)."""
import numpy as np
import pytest

from oracle import planner as P
from synth import cnn_params_np, edge_filter_np, images_np, cnn_dims


def run_edge_chunks(orc, imgs, K1, K2, plan):
    n, _, H, W = imgs.shape
    out = np.full((n, H, W), np.nan, np.float32)
    for ch in plan["chunks"]:
        (i0, i1), (r0, r1) = ch["in"], ch["out"]
        for b in range(ch["img"], ch["img"] + ch["nimg"]):
            E = orc.edge(imgs[b, 0, i0:i1], K1, K2)
            out[b, r0:r1] = E[r0 - i0:r1 - i0]
    return out


@pytest.mark.parametrize("n,H,W,budget", [(1, 61, 47, 0), (1, 61, 47, 20000),
                                          (3, 40, 36, 30000), (2, 33, 64, 10 ** 9), (1, 20, 20, 7000)])
def test_edge_split_equals_unsplit(orc, n, H, W, budget):
    seed = 0x5EED0001
    imgs = images_np(seed, n, H, W)
    K1, K2 = edge_filter_np()
    plan = P.fused_plan("edge", n, H, W, budget=budget, max_chunk_px=4096)
    if budget:
        assert plan["arena_bytes"] <= budget
    full = np.stack([orc.edge(imgs[b, 0], K1, K2) for b in range(n)])
    got = run_edge_chunks(orc, imgs, K1, K2, plan)
    assert np.array_equal(got, full)


def run_cnn_chunks(orc, imgs, n5, prm, plan, plane):
    n, _, H, W = imgs.shape
    (h1, w1), _, (h3, w3), _, (h5, w5) = cnn_dims(H, W)
    out = np.full((n, 9, h5, w5), np.nan, np.float32)
    for ch in plan["chunks"]:
        (i0, i1), (r0, r1) = ch["in"], ch["out"]
        p = list(prm)
        if plane:   # the chunk's bias rows (the rows of each level its outputs depend on)
            p[1] = prm[1][:, :, ch["c1"][0]:ch["c1"][1]]
            p[4] = prm[4][:, :, ch["c3"][0]:ch["c3"][1]]
            p[7] = prm[7][:, :, r0:r1]
            p[9] = prm[9][:, :, r0:r1]
        for b in range(ch["img"], ch["img"] + ch["nimg"]):
            sub = np.ascontiguousarray(imgs[b, 0, i0:i1])
            o = orc.cnn(sub, n5, p, bias_plane=plane)[0]
            assert o.shape[1] == r1 - r0
            out[b, :, r0:r1] = o
    return out


@pytest.mark.parametrize("n,H,W,n5,bias,budget,mcp", [
    (1, 92, 76, 20, "plane", 0, 2000), (1, 95, 70, 120, "plane", 0, 3000),
    (3, 60, 64, 20, "plane", 0, 10 ** 6), (1, 97, 61, 20, "scalar", 0, 1500)])
def test_cnn_split_equals_unsplit(orc, n, H, W, n5, bias, budget, mcp):
    seed = 0x5EED0004
    imgs = images_np(seed, n, H, W)
    prm = cnn_params_np(seed, n5, H, W, bias)
    plan = P.fused_plan("cnn", n, H, W, n5=n5, bias=bias, budget=budget, max_chunk_px=mcp)
    full = orc.cnn(imgs, n5, prm, bias_plane=(bias == "plane"))
    got = run_cnn_chunks(orc, imgs, n5, prm, plan, bias == "plane")
    assert np.array_equal(got, full)
    if plan["split"] == "rows":
        assert len(plan["chunks"]) > n


def test_cnn_halo_closed_form():
    """Final rows [r0, r1) need input rows [4 r0, 4 r1 + 28)."""
    for r0, r1 in [(0, 1), (3, 10), (100, 199)]:
        rg = P.back_propagate_rows(P.CNN_LAYERS, r0, r1)
        assert list(rg[0]) == [4 * r0, 4 * r1 + 28]


def test_chunk_rule_properties():
    for tmpl, kw in [("edge", dict(ks=16)), ("cnn", dict(n5=120)), ("cnn", dict(n5=20, bias="scalar"))]:
        for n, H, W in [(1, 4800, 6400), (15, 1000, 1000), (64, 480, 640)]:
            for budget in [0, 768 << 20, 1536 << 20, 64 << 20]:
                try:
                    p = P.fused_plan(tmpl, n, H, W, budget=budget, **kw)
                except RuntimeError:
                    continue
                if budget:
                    assert p["arena_bytes"] <= budget
                h_out = H if tmpl == "edge" else cnn_dims(H, W)[4][0]
                cover = {}
                for ch in p["chunks"]:
                    for b in range(ch["img"], ch["img"] + ch["nimg"]):
                        cover.setdefault(b, []).append(tuple(ch["out"]))
                assert sorted(cover) == list(range(n))
                for b, rs in cover.items():
                    rs.sort()
                    assert rs[0][0] == 0 and rs[-1][1] == h_out
                    assert all(a[1] == c[0] for a, c in zip(rs, rs[1:]))
                assert p["h2d_bytes"] >= 0 and p["d2h_bytes"] >= 0


def test_sharding_partitions_chunks():
    p = P.fused_plan("edge", 15, 10000, 10000, budget=768 << 20)
    C = p["n_chunks"]
    for G in (1, 2, 4, 8):
        got = []
        for g in range(G):
            q = P.fused_plan("edge", 15, 10000, 10000, budget=768 << 20, rank=g, world=G)
            _, _, c0, c1 = q["shard"]
            got.extend(range(c0, c1))
            assert abs((c1 - c0) - C / G) < 1
        assert got == list(range(C))


def test_streamed_bias_for_paper_large_cnn():
    """Large CNN at 6400x4800 under the 1.5 GB cap: the 2.6 GB bias set cannot be resident
    (SURVEY §8(c) 7b), so bias rows stream with each chunk; bytes stay near the I/O bound."""
    p = P.fused_plan("cnn", 1, 4800, 6400, n5=120, budget=1536 << 20)
    assert p["bias"] == "streamed" and p["split"] == "rows"
    assert p["h2d_bytes"] + p["d2h_bytes"] <= 1.10 * p["io_lower_bound_bytes"]
