"""GPU parity of the fused edge unit (K1) and the stream engine against the CPU oracle
(PAPER.md:629 template; tolerance 1e-5 normwise per image, R16), split ==
unsplit bit-exactly, device-resident == host-streamed bit-exactly, and sampled rows at
the bench's full size (15 x 10000^2 at the 768 MiB cap)."""
import json
import os

import numpy as np
import pytest

import synth
from conftest import GOLDEN
from gpu_util import guard_runtime, need_gpu, normwise, pinned, torch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tg():
    need_gpu()
    from paper_conf_ipps_sundaramrc09_b200 import tg as t
    torch.cuda.set_device(0)
    return t


def run_edge(tg, img, K1, K2=None, budget=0, device=False, torch_rt=True, max_chunk_px=None, depth=None):
    n, _, H, W = img.shape
    if device:
        x = torch.from_numpy(img).cuda()
        out = torch.zeros_like(x)
        g, _ = tg.edge_graph(x, K1, K2, out=out, device=True)
    else:
        out = np.zeros_like(img)
        g, _ = tg.edge_graph(img, K1, K2, out=out)
    g.set(budget=budget, torch_runtime=torch_rt, max_chunk_px=max_chunk_px, depth=depth)
    p = g.plan()
    p.execute()
    res = out.cpu().numpy() if device else out
    return res, p


def oracle_edge(orc, img, K1, K2):
    return np.stack([orc.edge(img[b, 0], K1, K2) for b in range(img.shape[0])])[:, None]


def test_hand_example_4x4(tg, orc):
    ex = json.load(open(os.path.join(GOLDEN, "hand_examples.json")))["edge_4x4"]
    img = np.asarray(ex["image"], np.float32)[None, None]
    out, _ = run_edge(tg, img, np.asarray(ex["K1"], np.float32), np.asarray(ex["K2"], np.float32))
    assert np.array_equal(out[0, 0], np.asarray(ex["E"], np.float32))


@pytest.mark.parametrize("n,H,W,ks", [(1, 37, 41, 16), (2, 256, 256, 16), (1, 130, 67, 5), (3, 64, 200, 2),
                                      (1, 1, 1, 16), (1, 1000, 1000, 16), (2, 97, 333, 9)])
def test_edge_parity(tg, orc, n, H, W, ks):
    seed = synth.seed_for_config(1)
    img = synth.images_np(seed, n, H, W)
    K1, K2 = synth.random_edge_filters_np(seed, ks)
    out, _ = run_edge(tg, img, K1, K2)
    ref = oracle_edge(orc, img, K1, K2)
    assert normwise(out, ref) <= 1e-5
    # remap + max are exact: the result is max(|E1|,|E2|) of the GPU's own convolutions
    assert np.all(out >= 0)


def test_edge_tile_geometry_invariance(tg, orc):
    """K1 picks its tile geometry from the work size (64x64 tiles of 8 warps; 32x32 when those are
    fewer than the SMs; 16x32 of 4 warps when even those are -- kernels/edge.cu): one 256x256 image
    alone (16x32 tiles), in a batch of 4 (32x32) and in a batch of 10 (64x64) gives the SAME bits,
    since every output pixel is the same FFMA sequence in the same order, and matches the oracle."""
    seed = synth.seed_for_config(1) + 5
    K1, K2 = synth.random_edge_filters_np(seed, 16)
    batch = synth.images_np(seed, 10, 256, 256)
    outs = [run_edge(tg, np.ascontiguousarray(batch[:n]), K1, K2)[0][0] for n in (1, 4, 10)]
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])
    assert normwise(outs[0][None], oracle_edge(orc, batch[:1], K1, K2)[0]) <= 1e-5


def test_find_edges_rotation(tg, orc):
    """find_edges(Image, Kernel, 4, MAX) with K2 = rot90(K1) derived in the
    library equals the oracle's template on the synthetic oriented filter."""
    img = synth.images_np(5, 2, 300, 257)
    K1, K2 = synth.edge_filter_np()
    out, _ = run_edge(tg, img, K1)
    assert normwise(out, oracle_edge(orc, img, K1, K2)) <= 1e-5


@pytest.mark.parametrize("budget,mcp,depth", [(200_000, None, None), (60_000, None, 2), (0, 4096, None),
                                              (1_000_000, 20000, 4)])
def test_split_equals_unsplit_bitexact(tg, orc, budget, mcp, depth):
    img = synth.images_np(7, 3, 211, 173)
    K1, K2 = synth.random_edge_filters_np(7)
    full, p0 = run_edge(tg, img, K1, K2)
    split, p1 = run_edge(tg, img, K1, K2, budget=budget, max_chunk_px=mcp, depth=depth)
    assert p1.stats()["n_chunks"] > p0.stats()["n_chunks"]
    if budget:
        assert p1.stats()["peak_device_bytes"][0] <= budget
    assert np.array_equal(split, full)
    assert normwise(full, oracle_edge(orc, img, K1, K2)) <= 1e-5


def test_device_io_equals_streamed(tg):
    img = synth.images_np(9, 4, 300, 320)
    K1, K2 = synth.random_edge_filters_np(9)
    a, _ = run_edge(tg, img, K1, K2, device=True)
    b, _ = run_edge(tg, img, K1, K2, budget=1_500_000)
    c, _ = run_edge(tg, img, K1, K2, torch_rt=False)
    assert np.array_equal(a, b) and np.array_equal(a, c)


def test_pinned_host_buffers_and_repeat(tg, orc):
    n, H, W = 2, 512, 640
    img_t = pinned((n, 1, H, W))
    img_t.copy_(torch.from_numpy(synth.images_np(11, n, H, W)))
    out_t = pinned((n, 1, H, W))
    K1, K2 = synth.edge_filter_np()
    g, _ = tg.edge_graph(img_t, K1, out=out_t)
    g.set(budget=2_000_000, torch_runtime=True)
    p = g.plan()
    for _ in range(3):
        out_t.zero_()
        p.execute()
    assert p.stats()["host_registered_bytes"] == 0   # already pinned: nothing registered
    ref = oracle_edge(orc, img_t.numpy(), K1, K2)
    assert normwise(out_t.numpy(), ref) <= 1e-5


def test_full_size_sampled_rows(tg, orc):
    """BASELINE configs[1] launch configuration (10000^2 images, 768 MiB cap, depth 3):
    rows at image borders and at every chunk boundary (+-8 rows) match the oracle, which
    computes each sampled row from its 16-row receptive band (exact: tests/test_oracle_chunks)."""
    n, H, W = 2, 10000, 10000
    seed = synth.seed_for_config(2)
    img_t = pinned((n, 1, H, W))
    img_t.copy_(synth.images_torch(seed, n, H, W, "cuda").cpu())
    out_t = pinned((n, 1, H, W))
    K1, K2 = synth.edge_filter_np()
    g, _ = tg.edge_graph(img_t, K1, out=out_t)
    g.set(budget=768 << 20, torch_runtime=True)
    p = g.plan()
    p.execute()
    plan = p.json()
    assert plan["arena_bytes"] <= 768 << 20 and plan["split"] == "rows"
    rows = {0, 1, 7, 8, H - 9, H - 8, H - 1}
    for ch in plan["chunks"]:
        for r in (ch["out"][0] - 1, ch["out"][0], ch["out"][1] - 1, ch["out"][1]):
            if 0 <= r < H:
                rows.add(r)
    img = img_t.numpy()
    out = out_t.numpy()
    for b in range(n):
        for r in sorted(rows):
            a0, a1 = max(0, r - 7), min(H, r + 9)
            band = orc.edge(np.ascontiguousarray(img[b, 0, a0:a1]), K1, K2)
            ref = band[r - a0]
            got = out[b, 0, r]
            err = np.abs(got.astype(np.float64) - ref).max() / np.abs(ref).max()
            assert err <= 1e-5, (b, r, err)


def test_two_host_threads_same_device(tg, orc):
    """tg_set_devices([0, 0]): the one-host-thread-per-device dispatcher with both
    shards on the one GPU of the box -- same chunk list, disjoint output rows, same bits."""
    img = synth.images_np(21, 3, 300, 260)
    K1, K2 = synth.random_edge_filters_np(21)
    ref, _ = run_edge(tg, img, K1, K2, budget=400_000)
    out = np.zeros_like(img)
    g, _ = tg.edge_graph(img, K1, K2, out=out)
    g.set(budget=400_000, devices=[0, 0], torch_runtime=True)
    p = g.plan()
    p.execute()
    assert p.stats()["n_chunks"] >= 4
    assert np.array_equal(out, ref)


def test_device_io_ordered_against_the_callers_stream(tg, orc):
    """Device-resident I/O: the execution runs after the producer of X on the caller's stream
    and before its consumer of Y (tg_execute_on), even when the producer is slow."""
    img = synth.images_np(23, 2, 512, 512)
    K1, K2 = synth.random_edge_filters_np(23)
    ref = oracle_edge(orc, img, K1, K2)
    src = torch.from_numpy(img).cuda()
    x = torch.zeros_like(src)
    y = torch.full_like(src, float("nan"))
    g, _ = tg.edge_graph(x, K1, K2, out=y, device=True)
    g.set(torch_runtime=True)
    p = g.plan()
    s = torch.cuda.Stream()
    torch.cuda.synchronize()
    for rep in range(3):
        with torch.cuda.stream(s):
            x.zero_()
            y.fill_(float("nan"))
            torch.cuda._sleep(20_000_000)       # ~10 ms of GPU time before X is written
            x.copy_(src)
            p.execute(blocking=False)            # ordered after the copy on s
            got = y.clone()                      # ordered after the execution on s
        s.synchronize()
        assert normwise(got.cpu().numpy()[:, 0], ref[:, 0]) <= 1e-5, rep
    # the legacy default stream is the default caller stream of the C calls
    x.zero_()
    torch.cuda._sleep(20_000_000)
    x.copy_(src)
    tg.tg_execute(p.h)
    torch.cuda.synchronize()
    assert normwise(y.cpu().numpy()[:, 0], ref[:, 0]) <= 1e-5


@pytest.mark.parametrize("nf", [1, 2, 3, 4])
@pytest.mark.parametrize("combine", ["max", "sum", "maxabs", "maxplain"])
def test_edge_general_combines(tg, orc, nf, combine):
    """Up to 4 convolutions (8 orientations, Fig. 1(b)) and the reductions of PAPER.md:621 in one
    fused K1 launch, split into chunks by a budget."""
    img = synth.images_np(31, 2, 150, 132)
    rs = np.random.default_rng(nf)
    K = [(rs.standard_normal((16, 16)) / 16).astype(np.float32) for _ in range(nf)]
    out = np.zeros_like(img)
    g, _ = tg.edge_graph_general(img, K, combine, out=out)
    g.set(budget=250_000, torch_runtime=True)
    p = g.plan()
    assert p.json()["nf"] == nf and p.json()["combine"] == combine and p.json()["n_chunks"] > 2
    p.execute()
    ref = np.stack([orc.edge_general(img[b, 0], K, combine) for b in range(2)])[:, None]
    assert normwise(out, ref) <= 1e-5


@pytest.mark.parametrize("ks", list(range(1, 17)))
def test_edge_every_kernel_size(tg, orc, ks):
    """Every ks in 1..16 (the kernel issues only the taps of the smallest 4/8/16 frame that
    holds the SAME-anchored ks x ks kernel): odd/even anchors and both sides of each frame edge,
    on a ragged image split into chunks."""
    img = synth.images_np(40 + ks, 1, 97, 76)
    rs = np.random.default_rng(100 + ks)
    K = [(rs.standard_normal((ks, ks)) / ks).astype(np.float32) for _ in range(3)]
    out = np.zeros_like(img)
    g, _ = tg.edge_graph_general(img, K, "max", out=out)
    g.set(budget=40_000, torch_runtime=True)
    p = g.plan()
    assert p.json()["n_chunks"] > 1
    p.execute()
    ref = orc.edge_general(img[0, 0], K, "max")[None, None]
    assert normwise(out, ref) <= 1e-5


@pytest.mark.parametrize("n_or,comb", [(8, "max"), (8, "sum"), (4, "maxabs"), (2, "max")])
def test_find_edges_orientations(tg, orc, n_or, comb):
    """find_edges(Image, Kernel, num_orientations, Combine_op) with the rotations
    of reading R18 (8 orientations: 0, 45, 90, 135 degrees + remaps), against the oracle's
    find_edges (oracle.rotate_kernel, pinned in tests/test_oracle_ops.py)."""
    img = synth.images_np(41, 1, 200, 180)
    K1, _ = synth.edge_filter_np()
    code = {"max": tg.TG_MAX, "sum": tg.TG_SUM, "maxabs": tg.TG_MAXABS}[comb]
    out = np.zeros_like(img)
    g, _ = tg.find_edges_graph(img, K1, n_or, code, out=out)
    g.set(torch_runtime=True)
    g.plan().execute()
    ref = orc.find_edges(img[0, 0], K1, n_or, comb)       # oracle: rotate_kernel (R18) + graph
    assert normwise(out[0], ref[None]) <= 1e-5


def test_pipelined_async_executions(tg):
    """Back-to-back async executions of one plan overlap across the persistent slot ring
    (depth 2, many chunks); the results equal the blocking execution bit for bit."""
    n, H, W = 3, 300, 256
    img_t = pinned((n, 1, H, W))
    img_t.copy_(torch.from_numpy(synth.images_np(12, n, H, W)))
    out_t = pinned((n, 1, H, W))
    K1, _ = synth.edge_filter_np()
    g, _ = tg.edge_graph(img_t, K1, out=out_t)
    g.set(budget=400_000, depth=2, torch_runtime=True)
    p = g.plan()
    assert p.stats()["n_chunks"] >= 8
    p.execute()
    ref = out_t.clone()
    for _ in range(3):
        out_t.zero_()
        torch.cuda.synchronize()
        for _ in range(4):
            p.execute(blocking=False)
        torch.cuda.synchronize()
        assert torch.equal(out_t, ref)


def test_trace_respects_stream_dependencies(tg):
    """tg_plan_trace_get: one record per chunk copy and launch; per chunk H2D ends before its
    kernel starts and the kernel ends before its D2H starts; a slot (depth 2) is not
    overwritten before the chunk that used it two steps earlier finished computing; copies
    of one direction never overlap each other (one stream each)."""
    n, H, W = 2, 300, 256
    img_t = pinned((n, 1, H, W))
    img_t.copy_(torch.from_numpy(synth.images_np(13, n, H, W)))
    out_t = pinned((n, 1, H, W))
    K1, _ = synth.edge_filter_np()
    g, _ = tg.edge_graph(img_t, K1, out=out_t)
    g.set(budget=400_000, depth=2, torch_runtime=True)
    p = g.plan()
    p.execute()                        # parameters resident; not profiled
    p.profiling(True)
    p.execute(blocking=False)
    p.execute(blocking=False)
    tr = p.trace()
    nc = p.stats()["n_chunks"]
    assert len(tr) == 2 * 3 * nc
    eps = 1e-3
    for e in range(2):
        recs = tr[e * 3 * nc:(e + 1) * 3 * nc]
        by = {(r["kind"], r["chunk"]): r for r in recs}
        assert len(by) == 3 * nc
        for c in range(nc):
            h, k, d = by[("h2d", c)], by[("edge", c)], by[("d2h", c)]
            assert h["t0_ms"] <= h["t1_ms"] <= k["t0_ms"] + eps
            assert k["t1_ms"] <= d["t0_ms"] + eps
            if c >= 2:
                assert by[("edge", c - 2)]["t1_ms"] <= h["t0_ms"] + eps
    for kind in ("h2d", "d2h", "edge"):
        iv = sorted((r["t0_ms"], r["t1_ms"]) for r in tr if r["kind"] == kind)
        assert all(a[1] <= b[0] + eps for a, b in zip(iv, iv[1:])), kind


@pytest.mark.parametrize("budget,nf", [(0, 2), (300_000, 2), (120_000, 4), (90_000, 1)])
def test_edge_slot_layout_covers_every_buffer(tg, orc, budget, nf):
    """Slot-layout property on the GPU (see the CNN test of the same name): guard bands around a
    NaN-filled arena stay intact and the output matches the oracle."""
    img = synth.images_np(71, 2, 170, 236)
    rs = np.random.default_rng(nf)
    K = [(rs.standard_normal((16, 16)) / 16).astype(np.float32) for _ in range(nf)]
    out = np.zeros_like(img)
    g, _ = tg.edge_graph_general(img, K, "max", out=out)
    rt = guard_runtime(tg)
    g.runtime = rt
    tg.tg_set_runtime(g.h, rt.struct)
    g.set(budget=budget)
    p = g.plan()
    p.execute()
    assert rt.guards_intact()
    ref = np.stack([orc.edge_general(img[b, 0], K, "max") for b in range(2)])[:, None]
    assert np.isfinite(out).all() and normwise(out, ref) <= 1e-5


def test_graph_replay_equals_direct_execution(tg, orc):
    """tg_plan_set_graph: executions replayed as one captured CUDA graph give the same bits as
    direct executions, follow new input values in the bound buffers, and count their launches;
    device-resident (configs[0]-sized) and host-streamed multi-chunk plans."""
    img = synth.images_np(29, 2, 256, 256)
    K1, K2 = synth.random_edge_filters_np(29)
    ref = oracle_edge(orc, img, K1, K2)
    x = torch.from_numpy(img).cuda()
    y = torch.zeros_like(x)
    g, _ = tg.edge_graph(x, K1, K2, out=y, device=True)
    g.set(torch_runtime=True)
    p = g.plan()
    p.execute()
    direct = y.clone()
    p.use_graph(True)
    for rep in range(3):
        y.zero_()
        l0 = p.launches()
        p.execute()
        assert p.launches() == l0 + 1
        assert torch.equal(y, direct), rep
    x.mul_(0.5)                                     # new values in the bound input buffer
    p.execute()
    assert normwise(y.cpu().numpy()[:, 0], oracle_edge(orc, img * np.float32(0.5), K1, K2)[:, 0]) <= 1e-5
    assert normwise(direct.cpu().numpy()[:, 0], ref[:, 0]) <= 1e-5
    # host-streamed, several chunks over a depth-2 ring
    out = pinned((2, 1, 256, 256))
    gh, _ = tg.edge_graph(pinned((2, 1, 256, 256)).copy_(torch.from_numpy(img)), K1, K2, out=out)
    gh.set(torch_runtime=True, budget=300_000, depth=2)
    ph = gh.plan()
    assert ph.stats()["n_chunks"] >= 4
    ph.execute()
    want = out.clone()
    ph.use_graph(True)
    for rep in range(3):
        out.zero_()
        ph.execute()
        assert torch.equal(out, want), rep


def test_shard_holds_only_its_images(tg, orc):
    """Multi-process sharding (tg_set_shard) as bench.py and tools/config5.py run it: each rank
    pins host buffers for ITS images only and passes base pointers offset by the images before
    them -- the library touches (and registers) nothing else. Every rank's rows equal the
    one-process run bit for bit (the same global chunk list)."""
    n, H, W = 6, 200, 256
    img = synth.images_np(33, n, H, W)
    K1, K2 = synth.random_edge_filters_np(33)
    full = np.zeros_like(img)
    g, _ = tg.edge_graph(img, K1, K2, out=full)
    g.set(torch_runtime=True, budget=500_000)
    g.plan().execute()
    world = 3
    for rank in range(world):
        probe, _ = tg.edge_graph(img, K1, K2, out=np.zeros_like(img))
        probe.set(budget=500_000, shard=(rank, world))
        j = probe.plan().json()
        mine = j["chunks"][j["shard"][2]:j["shard"][3]]
        i0 = min(c["img"] for c in mine)
        i1 = max(c["img"] + c["nimg"] for c in mine)
        xs = pinned((i1 - i0, 1, H, W))
        xs.copy_(torch.from_numpy(img[i0:i1]))
        ys = pinned((i1 - i0, 1, H, W))
        gs = tg.Graph()
        x = tg.tg_input(gs.h, n, 1, H, W, xs.data_ptr() - i0 * H * W * 4)
        k1 = gs.param(K1.reshape(1, 1, 16, 16))
        k2 = gs.param(K2.reshape(1, 1, 16, 16))
        e1 = gs.conv2d(x, k1, -1, tg.TG_SAME)
        e2 = gs.conv2d(x, k2, -1, tg.TG_SAME)
        tg.tg_output(gs.h, gs.max_combine([e1, e2, gs.neg(e1), gs.neg(e2)]), ys.data_ptr() - i0 * H * W * 4)
        gs._keep += [xs, ys]
        gs.set(torch_runtime=True, budget=500_000, shard=(rank, world))
        p = gs.plan()
        assert p.json()["chunks"] == j["chunks"]
        p.execute()
        for c in mine:
            for b in range(c["img"], c["img"] + c["nimg"]):
                r0, r1 = c["out"]
                assert np.array_equal(ys[b - i0, 0, r0:r1].numpy(), full[b, 0, r0:r1]), (rank, b)
