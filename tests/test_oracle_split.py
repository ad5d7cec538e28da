"""Pins of the splitting oracle (oracle/planner.py::split_plan, reading R19)
and of the matmul oracle (oracle.c orc_matmul), against what the paper and the
mathematics fix:
  * the paper's own example: a 100x100 image and a 5x5 kernel split in two give
    two 52-row input pieces (not 50) and two 48-row output pieces;
  * step 3's fixpoint: every piece operator fits, the search is tight (re-planning at the
    largest piece requirement gives the same k) and more memory never needs more pieces;
  * the sinks' pieces tile the output exactly; each input piece is what its consumer needs;
  * executing the pieces in the plan's DFS order, each reading only its pieces, reproduces
    the unsplit graph bit for bit (PAPER.md:357 splitting does not change the computation)
    -- a wrong halo, offset or stride anywhere makes this fail;
  * uncapped / fitting graphs are not split (k = 1, whole data structures);
  * matmul: hand example, identity, brute force against numpy in fp64."""
import numpy as np
import pytest

import synth
from oracle import planner as P
from split_graphs import cnn_spec, edge_spec, mixed_spec, run_split, run_unsplit


def test_paper_example_367():
    shapes = [(1, 1, 100, 100), (1, 1, 5, 5), (1, 1, 96, 96)]
    nodes = [P.SNode("conv_valid", [0, 1], 2, kh=5)]
    r = P.split_plan(shapes, ["input", "param", "output"], nodes, 2, capacity=40000)
    assert r["k"] == {0: 2}
    ins = [(a, b) for d, a, b in r["pieces"] if d == 0]
    outs = [(a, b) for d, a, b in r["pieces"] if d == 2]
    assert [b - a for a, b in ins] == [52, 52]          # "two 100x52 input matrices (not 100x50)"
    assert [b - a for a, b in outs] == [48, 48]         # "two 96x48 output matrices"
    assert ins == [(0, 52), (48, 100)] and outs == [(0, 48), (48, 96)]
    # the kernel is never split
    assert [(a, b) for d, a, b in r["pieces"] if d == 1] == [(0, 5)]


def _check_fixpoint(spec, r, capacity):
    g = r["graph"]
    for o in g.ops:
        ds = set(o.ins) | set(o.outs)
        assert sum(g.ds[j].size for j in ds) <= capacity
    # sinks (the output) tiled exactly by its pieces
    outs = sorted((a, b) for d, a, b in r["pieces"] if d == spec.output)
    h = spec.shapes[spec.output][2]
    assert outs[0][0] == 0 and outs[-1][1] == h
    assert all(outs[i][1] == outs[i + 1][0] for i in range(len(outs) - 1))
    # step 3 stops at the first k that fits: k - 1 pieces (when above the paper's start
    # ceil(req / M)) leave some piece operator over the capacity
    k = max(r["k"].values())
    if k > 1:
        k0 = max(-(-sum(4 * int(np.prod(spec.shapes[d])) for d in set(nd.ins) | {nd.out}) // capacity)
                 for nd in spec.nodes)
        if k - 1 >= max(k0, 2):
            gk = spec_plan_forced(spec, capacity, k - 1)["graph"]
            assert max(sum(gk.ds[j].size for j in set(o.ins) | set(o.outs)) for o in gk.ops) > capacity
    # more memory never needs more pieces
    assert all(spec.plan(int(capacity * f))["k"][i] <= r["k"][i] for f in (1.5, 3.0) for i in r["k"])


def spec_plan_forced(spec, capacity, k):
    return P.split_plan(spec.shapes, spec.kinds, spec.nodes, spec.output, capacity, force_k=k)


@pytest.mark.parametrize("capacity_frac", [1.0, 0.5, 0.2, 0.08])
def test_edge_split_equals_unsplit(capacity_frac):
    K1, K2 = synth.random_edge_filters_np(7)
    spec = edge_spec(61, 37, K1, K2, n=2, rng=3)
    full = spec.total_bytes()
    cap = int(full * capacity_frac)
    r = spec.plan(cap)
    if capacity_frac == 1.0:
        assert set(r["k"].values()) == {1}
        assert len(r["pieces"]) == len(spec.shapes)
    else:
        assert max(r["k"].values()) > 1
    _check_fixpoint(spec, r, cap)
    ref = run_unsplit(spec)
    out = run_split(spec, r)
    assert np.array_equal(out, ref)
    # the unsplit executor is the oracle's edge template
    import oracle
    want = np.stack([oracle.edge(spec.data[0][i, 0], K1, K2) for i in range(2)])
    assert np.abs(ref[:, 0] - want).max() <= 1e-5 * np.abs(want).max()


def test_edge_halo_pieces_overlap():
    K1, K2 = synth.random_edge_filters_np(7)
    spec = edge_spec(200, 40, K1, K2)
    r = spec.plan(int(spec.total_bytes() * 0.1))
    k = r["k"][0]
    img = [(a, b) for d, a, b in r["pieces"] if d == 0]
    out = [(a, b) for d, a, b in r["pieces"] if d == spec.output]
    assert len(img) == len(out) == k
    for (ia, ib), (oa, ob) in zip(img, out):  # SAME 16x16: rows [a-7, b+8) clipped
        assert ia == max(0, oa - 7) and ib == min(200, ob + 8)


@pytest.mark.parametrize("frac", [1.0, 0.3, 0.2, 0.17])
def test_cnn_split_equals_unsplit(frac):
    H, W, n5 = 77, 41, 4
    prm = synth.cnn_params_np(11, n5, H, W)
    spec = cnn_spec(1, H, W, n5, prm)
    cap = int(spec.total_bytes() * frac)
    r = spec.plan(cap)
    _check_fixpoint(spec, r, cap)
    ref = run_unsplit(spec)
    assert np.array_equal(run_split(spec, r), ref)
    import oracle
    want = oracle.cnn(spec.data[0], n5, prm)
    assert np.abs(ref - want).max() <= 1e-5 * np.abs(want).max()


@pytest.mark.parametrize("frac", [1.0, 0.4, 0.15])
def test_mixed_split_equals_unsplit(frac):
    spec = mixed_spec(83, 30, 7)
    cap = int(spec.total_bytes() * frac)
    r = spec.plan(cap)
    _check_fixpoint(spec, r, cap)
    assert np.array_equal(run_split(spec, r), run_unsplit(spec))
    # the matmul's second matrix is read whole by every piece
    mm = [i for i, nd in enumerate(spec.nodes) if nd.kind == "matmul"][0]
    B = spec.nodes[mm].ins[1]
    assert [(a, b) for d, a, b in r["pieces"] if d == B] == [(0, spec.shapes[B][2])]


def test_infeasible_when_kernel_alone_exceeds():
    shapes = [(1, 1, 64, 64), (1, 1, 32, 32), (1, 1, 33, 33)]
    with pytest.raises(ValueError):
        P.split_plan(shapes, ["input", "param", "output"], [P.SNode("conv_valid", [0, 1], 2, kh=32)], 2, 4 * 1000)


def test_matmul_oracle_pins():
    import oracle
    A = np.array([[1, 2, 3], [4, 5, 6]], np.float32)
    B = np.array([[7, 8], [9, 10], [11, 12]], np.float32)
    assert np.array_equal(oracle.matmul(A, B), np.array([[58, 64], [139, 154]], np.float32))
    rng = np.random.default_rng(0)
    X = rng.standard_normal((37, 29)).astype(np.float32)
    assert np.array_equal(oracle.matmul(np.eye(37, dtype=np.float32), X), X)
    assert np.array_equal(oracle.matmul(X, np.eye(29, dtype=np.float32)), X)
    A = rng.standard_normal((45, 300)).astype(np.float32)
    B = rng.standard_normal((300, 23)).astype(np.float32)
    ref = (A.astype(np.float64) @ B.astype(np.float64))
    got = oracle.matmul(A, B)
    assert np.abs(got - ref).max() <= np.abs(ref).max() * 2 ** -23   # one rounding of an fp64 sum
    assert np.allclose(oracle.matmul(B.T.copy(), A.T.copy()), got.T, rtol=0, atol=1e-4)
