"""Multi-process sharding on CPU (gloo, world_size 2): the host-side logic of the multi-GPU
path. Each rank plans its shard through the C ABI (planning needs no GPU);
the shards partition the global chunk list with no overlap, chunk boundaries do not depend
on the world size, every rank's chunks executed on the oracle and assembled into disjoint
output slices reproduce the unsplit template exactly (no collective on the data path), and
bench.py's max-over-ranks timing and min-over-ranks host-link reductions work over gloo."""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import bench
        import oracle
        import synth
        from paper_conf_ipps_sundaramrc09_b200 import tg
        res = {}
        # ---- edge: 3 images of 70x90, a budget that forces row chunks
        n, H, W = 3, 70, 90
        img = synth.images_np(5, n, H, W)
        K1, K2 = synth.random_edge_filters_np(5)
        out = np.zeros_like(img)
        g, _ = tg.edge_graph(img, K1, K2, out=out)
        g.set(budget=60_000, shard=(rank, world))
        plan = g.plan().json()
        c0, c1 = plan["shard"][2:]
        mine = np.full((n, H, W), np.nan, np.float32)
        for ch in plan["chunks"][c0:c1]:
            (i0, i1), (r0, r1) = ch["in"], ch["out"]
            for b in range(ch["img"], ch["img"] + ch["nimg"]):
                mine[b, r0:r1] = oracle.edge(img[b, 0, i0:i1], K1, K2)[r0 - i0:r1 - i0]
        ranges = [None] * world
        dist.all_gather_object(ranges, (c0, c1, len(plan["chunks"])))
        parts = [None] * world
        dist.all_gather_object(parts, mine)
        res["edge_ranges"] = ranges
        assembled = np.where(np.isnan(parts[0]), parts[1], parts[0]) if world == 2 else parts[0]
        full = np.stack([oracle.edge(img[b, 0], K1, K2) for b in range(n)])
        res["edge_exact"] = bool(np.array_equal(assembled, full))
        res["edge_disjoint"] = bool(not np.any(~np.isnan(parts[0]) & ~np.isnan(parts[1]))) if world == 2 else True
        # chunk boundaries are independent of the world size
        g1, _ = tg.edge_graph(img, K1, K2, out=out)
        g1.set(budget=60_000)
        res["same_chunks"] = g1.plan().json()["chunks"] == plan["chunks"]
        # ---- timing reduction used by bench.py
        res["max"] = bench.max_over_ranks(float(rank + 1), world)
        res["min"] = bench.min_over_ranks(float(rank + 1), world)  # the host-link denominator
        res["gather"] = bench.gather_objects({rank: rank * 10}, world)
        # a rank may hold ONLY its share of the global input/output: the plan's shard touches a
        # contiguous image span, and a base pointer offset into a smaller buffer plans the same
        span = sorted({b for ch in plan["chunks"][c0:c1] for b in range(ch["img"], ch["img"] + ch["nimg"])})
        part_in = np.ascontiguousarray(img[span[0]:span[-1] + 1])
        gs = tg.Graph()
        xs = tg.tg_input(gs.h, n, 1, H, W, part_in.ctypes.data - span[0] * H * W * 4)
        k1 = gs.param(K1.reshape(1, 1, 16, 16))
        k2 = gs.param(K2.reshape(1, 1, 16, 16))
        e1 = gs.conv2d(xs, k1, -1, tg.TG_SAME)
        e2 = gs.conv2d(xs, k2, -1, tg.TG_SAME)
        e = gs.max_combine([e1, e2, gs.neg(e1), gs.neg(e2)])
        part_out = np.zeros((span[-1] + 1 - span[0], 1, H, W), np.float32)
        tg.tg_output(gs.h, e, part_out.ctypes.data - span[0] * H * W * 4)
        gs.set(budget=60_000, shard=(rank, world))
        res["span_plan_same"] = gs.plan().json()["chunks"] == plan["chunks"]
        q.put((rank, res))
        dist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, {"error": traceback.format_exc()}))


def test_two_rank_sharding_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    results = dict(q.get(timeout=240) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    for r in range(world):
        assert "error" not in results[r], results[r].get("error")
    ranges = results[0]["edge_ranges"]
    C = ranges[0][2]
    assert ranges[0][0] == 0 and ranges[0][1] == ranges[1][0] and ranges[1][1] == C and C >= 4
    for r in range(world):
        assert results[r]["edge_exact"] and results[r]["edge_disjoint"] and results[r]["same_chunks"]
        assert results[r]["max"] == 2.0 and results[r]["min"] == 1.0
        assert results[r]["gather"] == [{0: 0}, {1: 10}] and results[r]["span_plan_same"]
