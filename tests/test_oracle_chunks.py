"""The fused chunking (oracle/planner.fused_chunks) and halo back-propagation, checked by
executing every chunk on the ORACLE and comparing with the unsplit oracle bit-exactly
(splitting must not change results) for many chunk sizes, plus
structural properties (coverage, shards, byte counts)."""
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


@pytest.mark.parametrize("n,H,W,split,B,R", [(1, 61, 47, "batch", 1, 61), (1, 61, 47, "rows", 1, 13),
                                              (3, 40, 36, "rows", 1, 7), (3, 40, 36, "batch", 2, 40),
                                              (2, 33, 64, "rows", 1, 1), (1, 20, 20, "rows", 1, 19)])
def test_edge_split_equals_unsplit(orc, n, H, W, split, B, R):
    seed = 0x5EED0001
    imgs = images_np(seed, n, H, W)
    K1, K2 = edge_filter_np()
    plan = P.fused_chunks("edge", n, H, W, split, B, R)
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


@pytest.mark.parametrize("n,H,W,n5,bias,split,B,R", [
    (1, 92, 76, 20, "streamed", "rows", 1, 5), (1, 95, 70, 120, "streamed", "rows", 1, 7),
    (3, 60, 64, 20, "resident", "batch", 2, 0), (1, 97, 61, 20, "scalar", "rows", 1, 3),
    (2, 70, 66, 7, "resident", "rows", 1, 1)])
def test_cnn_split_equals_unsplit(orc, n, H, W, n5, bias, split, B, R):
    seed = 0x5EED0004
    imgs = images_np(seed, n, H, W)
    pb = "scalar" if bias == "scalar" else "plane"
    prm = cnn_params_np(seed, n5, H, W, pb)
    R = R or cnn_dims(H, W)[4][0]
    plan = P.fused_chunks("cnn", n, H, W, split, B, R, n5=n5, bias=bias)
    bias = pb
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


def test_chunking_properties():
    """Every chunking covers every output row of every image exactly once, in order; the
    predicted bytes add up over the chunks."""
    for tmpl, kw in [("edge", dict(ks=16)), ("cnn", dict(n5=120, bias="streamed")), ("cnn", dict(n5=20, bias="scalar"))]:
        for n, H, W in [(1, 4800, 6400), (15, 1000, 1000), (64, 480, 640)]:
            h_out = H if tmpl == "edge" else cnn_dims(H, W)[4][0]
            for split, B, R in [("rows", 1, 199), ("rows", 1, h_out), ("batch", 7, h_out), ("rows", 1, 1)]:
                p = P.fused_chunks(tmpl, n, H, W, split, B, R, **kw)
                cover = {}
                for ch in p["chunks"]:
                    for b in range(ch["img"], ch["img"] + ch["nimg"]):
                        cover.setdefault(b, []).append(tuple(ch["out"]))
                assert sorted(cover) == list(range(n))
                for b, rs in cover.items():
                    assert rs[0][0] == 0 and rs[-1][1] == h_out
                    assert all(a[1] == c[0] for a, c in zip(rs, rs[1:]))
                planes = 1 if tmpl == "edge" else 9
                w_out = W if tmpl == "edge" else cnn_dims(H, W)[4][1]
                assert p["d2h_bytes"] == n * planes * h_out * w_out * 4
                assert p["h2d_chunk_bytes"] >= n * H * W * 4 * (1 if tmpl == "edge" or split == "batch" else 0.99)


def test_sharding_partitions_chunks():
    """Rank g of G takes chunks [floor(C g / G), floor(C (g+1) / G)): a partition of the same
    global list for every G, balanced to one chunk."""
    p = P.fused_chunks("edge", 15, 10000, 10000, "rows", 1, 3347)
    C = p["n_chunks"]
    assert C == 45
    for G in (1, 2, 4, 8):
        got, d2h = [], 0
        for g in range(G):
            q = P.fused_chunks("edge", 15, 10000, 10000, "rows", 1, 3347, rank=g, world=G)
            _, _, c0, c1 = q["shard"]
            assert q["chunks"] == p["chunks"]
            got.extend(range(c0, c1))
            d2h += q["d2h_bytes"]
            assert abs((c1 - c0) - C / G) < 1
        assert got == list(range(C))
        assert d2h == p["d2h_bytes"]
