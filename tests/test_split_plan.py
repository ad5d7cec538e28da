"""The library's operator splitting (TG_PER_OP, reading R19) built through
the C ABI on a CPU-only box, bit-exact against the splitting oracle (oracle/planner.py::
split_plan): the same pieces (DS, row band), the same piece operators, the same DFS order
(PAPER.md:381), the same next-use transfer trace and byte counts, for the
edge template, the CNN and a conv/tanh/subsample/matmul/affine chain at several budgets."""
import numpy as np
import pytest

import synth
from split_graphs import cnn_spec, edge_spec, lib_graph, mixed_spec

KIND = {"input": 0, "param": 1, "temp": 2, "output": 3}


def check_layout(j):
    """The static arena layout (the library's design, not the paper's; checked by properties):
    every residency interval of a piece lies inside the arena and no two pieces resident at the
    same step of the trace overlap."""
    a256 = lambda v: (max(v, 1) + 255) // 256 * 256   # noqa: E731
    res = {}
    for (kind, i), off in zip(j["trace_full"], j["trace_off"]):
        if kind == 0 or kind == 1:
            d = i if kind == 0 else j["ops"][i][1][0]
            if d not in res:
                res[d] = (off, off + a256(j["ds"][d][0]))
                assert res[d][1] <= j["arena_bytes"]
            assert off == res[d][0]
            iv = sorted(res.values())
            assert all(iv[t][1] <= iv[t + 1][0] for t in range(len(iv) - 1))
        elif kind == 3:
            res.pop(i, None)


def compare(spec, budget):
    """The library's TG_PER_OP plan against the splitting oracle AT THE LIBRARY'S CAPACITY M:
    pieces, piece operators, k, DFS order, next-use trace and bytes bit for bit. M itself
    follows the fragmentation margin: the budget less 1/8, less further 1/16
    steps while the static layout does not fit (uncapped: every DS once)."""
    from paper_conf_ipps_sundaramrc09_b200 import tg
    out = np.zeros(spec.shapes[spec.output], np.float32)
    g = lib_graph(spec, out, budget=budget)
    j = g.plan(tg.TG_PER_OP).json()
    from oracle import planner as P
    M = j["capacity"]
    if budget:
        steps = (budget - budget // 8 - M) / (budget // 16)
        assert steps == int(steps) and steps >= 0
    else:       # uncapped: room for every DS the output depends on, once
        used = {d for nd in spec.nodes for d in nd.ins + [nd.out]} | {spec.output}
        assert M == 4 * sum(int(np.prod(spec.shapes[d])) for d in used)
    r = P.per_op_plan(spec.shapes, spec.kinds, spec.nodes, spec.output, M)
    og = r["graph"]
    assert j["pieces"] == r["pieces"]
    assert j["ds"] == [[d.size, KIND[d.kind]] for d in og.ds]
    assert j["ops"] == [[o.ins, o.outs] for o in og.ops]
    assert j["op_piece"] == r["op_piece"]
    assert {int(k): v for k, v in j["k"].items()} == r["k"]
    assert j["order"] == r["order"]
    kind = {"h2d": 0, "run": 1, "d2h": 2}
    names_ds = {d.name: i for i, d in enumerate(og.ds)}
    names_op = {o.name: i for i, o in enumerate(og.ops)}
    assert j["trace"] == [[kind[k], names_op[n] if k == "run" else names_ds[n]] for k, n in r["trace"]]
    assert j["h2d_bytes"] + j["d2h_bytes"] == r["moved"]
    if budget:
        kf = {"h2d": 0, "run": 1, "d2h": 2, "free": 3}
        assert j["trace_full"] == [[kf[k], names_op[n] if k == "run" else names_ds[n]] for k, n in r["trace_full"]]
        check_layout(j)
    return j, r


@pytest.mark.parametrize("frac", [0, 0.5, 0.2, 0.08])
def test_edge_split_plan_matches_oracle(frac):
    K1, K2 = synth.random_edge_filters_np(7)
    spec = edge_spec(301, 64, K1, K2, n=2, rng=3)
    budget = int(spec.total_bytes() * frac) // 256 * 256
    j, r = compare(spec, budget)
    if frac and frac < 0.5:
        assert max(r["k"].values()) > 1


@pytest.mark.parametrize("frac", [0, 0.3, 0.25, 0.2])
def test_cnn_split_plan_matches_oracle(frac):
    H, W, n5 = 77, 41, 4
    spec = cnn_spec(1, H, W, n5, synth.cnn_params_np(11, n5, H, W))
    compare(spec, int(spec.total_bytes() * frac) // 256 * 256)


@pytest.mark.parametrize("frac", [0, 0.4, 0.15])
def test_mixed_split_plan_matches_oracle(frac):
    spec = mixed_spec(83, 30, 7)
    compare(spec, int(spec.total_bytes() * frac) // 256 * 256)


def test_paper_example_367_through_the_library():
    from paper_conf_ipps_sundaramrc09_b200 import tg
    x = np.zeros((1, 1, 100, 100), np.float32)
    g = tg.Graph()
    xi = g.input(x)
    k = g.param(np.zeros((1, 1, 5, 5), np.float32))
    y = g.conv2d(xi, k)
    g.output(y, np.zeros((1, 1, 96, 96), np.float32))
    g.set(budget=45568)                   # capacity 39,872 B: two pieces
    j = g.plan(tg.TG_PER_OP).json()
    assert [p[1:] for p in j["pieces"] if p[0] == xi] == [[0, 52], [48, 100]]
    assert [p[1:] for p in j["pieces"] if p[0] == y] == [[0, 48], [48, 96]]
    with pytest.raises(tg.TGError) as e:   # the baseline never splits
        g.plan(tg.TG_BASELINE)
    assert e.value.code == tg.TG_E_INFEASIBLE


def test_infeasible_when_nothing_fits():
    from paper_conf_ipps_sundaramrc09_b200 import tg
    g = tg.Graph()
    xi = g.input(np.zeros((1, 1, 64, 64), np.float32))
    k = g.param(np.zeros((1, 1, 32, 32), np.float32))
    g.output(g.conv2d(xi, k), np.zeros((1, 1, 33, 33), np.float32))
    g.set(budget=4608)
    with pytest.raises(tg.TGError) as e:
        g.plan(tg.TG_PER_OP)
    assert e.value.code == tg.TG_E_INFEASIBLE


@pytest.mark.parametrize("S_over_M,regime", [(0.09, "all_fit"), (0.107, "max_separate"), (0.133, "max_split"),
                                             (0.533, "conv_remap_split"), (1.07, "input_chunked")])
def test_fig1c_regimes_on_real_plans(S_over_M, regime):
    """Fig. 1(c) on real TG_PER_OP plans of the 8-orientation edge graph
    (tg_find_edges, 4 convolutions + 4 remaps + one 8-input max): with the image S bytes and the
    scheduling capacity M,
      all_fit           (10 S <= M)       nothing split, only the I/O lower bound moves;
      max_separate      (9 S <= M < 10 S) nothing split although the whole graph does not fit at
                        once (the DFS order with eager deletion keeps it to the I/O bound here);
      max_split / conv_remap_split / input_chunked (9 S > M) the graph is split, into at least
                        ceil(9 S / M) pieces (the paper's k for max; R19 splits the connected
                        operators together).
    The oracle's closed-form regime (fig1c_regime) names the case at the same S / M."""
    from oracle import planner as P
    from paper_conf_ipps_sundaramrc09_b200 import tg
    assert P.fig1c_regime(S_over_M * 1500.0, 1500.0) == regime
    H = W = 384
    S = 4 * H * W
    M = int(S / S_over_M)
    budget = (M * 8 + 6) // 7 + 16 * 1024          # capacity = budget - budget/8 >= M (kernels: 8 x 1 KB)
    img = np.zeros((1, 1, H, W), np.float32)
    g = tg.Graph()
    x = g.input(img)
    k = g.param(synth.edge_filter_np()[0].reshape(1, 1, 16, 16))
    e = g.find_edges(x, k, 8, tg.TG_MAX)
    g.output(e, np.zeros_like(img))
    g.set(budget=budget)
    j = g.plan(tg.TG_PER_OP).json()
    assert len(j["ops"]) >= 9
    kmax = max(j["k"].values())
    moved = j["h2d_bytes"] + j["d2h_bytes"]
    if regime == "all_fit":
        assert kmax == 1 and moved == j["io_lower_bound_bytes"]
    elif regime == "max_separate":
        assert kmax == 1 and j["total_temp_bytes"] > j["capacity"] and moved >= j["io_lower_bound_bytes"]
    else:
        assert kmax >= -(-9 * S // j["capacity"])
