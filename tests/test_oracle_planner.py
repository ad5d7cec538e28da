"""Pins for the planner oracle (oracle/planner.py) against the numbers the paper prints:
Table 1 accounting, operator/DS counts, Fig. 3 and
Fig. 6 transfer volumes, the PAPER.md:367 split example and the
Fig. 1(c) regimes."""
import json
import os

import pytest

from conftest import GOLDEN
from oracle import planner as P


def golden(name):
    with open(os.path.join(GOLDEN, name)) as fh:
        return json.load(fh)


def test_table1_edge():
    for row in golden("table1.json")["edge"]:
        g = P.edge_graph(row["H"], row["W"], 16)
        assert len(g.ops) == 5 and len(g.ds) == 8
        assert g.total_temp() == row["total"]
        assert g.io_lower_bound() == row["io"]
        if row["baseline"] is not None:
            assert g.baseline() == row["baseline"]


@pytest.mark.parametrize("idx", range(6))
def test_table1_cnn_total_and_io(idx):
    row = golden("table1.json")["cnn"][idx]
    g = P.cnn_graph_fig7(row["H"], row["W"], row["n5"])
    counts = golden("table1.json")["cnn_counts"][row["net"]]
    assert len(g.ops) == counts["ops"]
    assert len(g.ds) == counts["ds"]
    assert g.total_temp() == row["total"]
    assert g.io_lower_bound() == row["io"]


def test_table1_cnn_baseline_large_minus_small():
    """Only the large - small differences of the baseline column are reproduced (the
    absolute values are parity-unpinned)."""
    rows = golden("table1.json")["cnn"]
    for s, l in zip(rows[:3], rows[3:]):
        assert (s["H"], s["W"]) == (l["H"], l["W"])
        d_model = (P.cnn_conv_accumulate_baseline(l["H"], l["W"], 120)
                   - P.cnn_conv_accumulate_baseline(s["H"], s["W"], 20))
        assert d_model == l["baseline"] - s["baseline"]


def _order(ops, names):
    return [ops[n] for n in names]


def test_fig3_schedules():
    gold = golden("schedules.json")["fig3"]
    g, ops = P.fig3_graph()
    assert P.simulate_transfers(g, _order(ops, gold["a"]["order"]), gold["capacity"]) == gold["a"]["units"]
    assert P.simulate_transfers(g, _order(ops, gold["b"]["order"]), gold["capacity"]) == gold["b"]["units"]


def test_fig6_optimum_and_timeline():
    gold = golden("schedules.json")
    g, ops = P.fig3_graph()
    best, n_orders, n_best = P.brute_force_min_transfers(g, gold["fig3"]["capacity"])
    assert best == gold["fig6"]["optimal_units"]
    assert n_orders == 264 and n_best >= 1
    trace = []
    P.simulate_transfers(g, _order(ops, gold["fig3"]["b"]["order"]), 5, trace)
    assert [list(t) for t in trace[:4]] == gold["fig6"]["first_steps"]


def test_dfs_order_hand_examples():
    """DFS orders worked by hand from PAPER.md:381 / R11 (tests/golden/schedules.json "dfs")."""
    gold = golden("schedules.json")["dfs"]
    g, ops = P.fig3_graph()
    assert [g.ops[i].name for i in P.dfs_order(g)] == gold["fig3"]["order"]
    ex = gold["backtrack"]
    g2 = P.Graph()
    ids = {nm: g2.add_ds(nm, 1, kind) for nm, kind in ex["ds"]}
    for nm, ins, outs in ex["ops"]:
        g2.add_op(nm, [ids[a] for a in ins], [ids[b] for b in outs])
    assert [g2.ops[i].name for i in P.dfs_order(g2)] == ex["order"]


def test_dfs_order_is_a_topological_order():
    g, ops = P.fig3_graph()
    order = P.dfs_order(g)
    assert order in list(P.topological_orders(g))
    # depth first: C1's sub-tree (R1', R1'') before its sibling C2
    names = [g.ops[i].name for i in order]
    assert names.index("R1'") < names.index("C2")


def test_p367_split_example():
    gold = golden("schedules.json")["p367"]
    out_h = gold["H"] - gold["k"] + 1
    step = out_h // gold["parts"]
    for (o0, o1), (i0, i1) in zip(gold["out_rows"], gold["in_rows"]):
        assert o1 - o0 == step
        rg = P.back_propagate_rows([("valid", gold["k"])], o0, o1)
        assert list(rg[0]) == [i0, i1] and i1 - i0 == 52


def test_fig1c_regimes():
    gold = golden("schedules.json")["fig1c"]
    th = gold["thresholds"]
    probes = [th[0] * 0.99, (th[0] + th[1]) / 2, (th[1] + th[2]) / 2, (th[2] + th[3]) / 2, th[3] * 1.01]
    got = [P.fig1c_regime(s, gold["M"]) for s in probes]
    assert got == gold["regimes"]
    # the boundaries themselves: max = 9S, C/R = 2S, total = 10S
    assert P.fig1c_regime(th[0] * 1.0001, gold["M"]) == "max_separate"
    assert P.fig1c_regime(th[1] * 1.0001, gold["M"]) == "max_split"
    assert P.fig1c_regime(th[2] * 1.0001, gold["M"]) == "conv_remap_split"


def test_split_factors_8_orientations():
    g = P.edge_graph(1, 1, orientations=8, kernel_floats=False)
    for S, k_max, k_cr in [(160, 1, 1), (200, 2, 1), (800, 5, 2), (1600, 10, 3)]:
        g2 = P.edge_graph(1, S, orientations=8, kernel_floats=False)
        k = P.split_factors(g2, 1500)
        assert k["max"] == k_max and k["C1"] == k_cr and k["R1"] == k_cr


def test_edge_graph_general_counts_by_hand():
    """Operator / DS counts of the edge graph variants, counted by hand from PAPER.md:621-629:
    max over nf responses and their remaps = nf convs + nf remaps + 1 max (Fig. 3 at nf = 2:
    5 ops, 8 DS); sum = nf convs + 1 add, DS Im + nf kernels + nf responses + E; maxabs adds
    one abs op and DS per response."""
    for nf in (1, 2, 3, 4):
        g = P.edge_graph_general(10, 12, 16, nf, "max")
        assert (len(g.ops), len(g.ds)) == (2 * nf + 1, 1 + nf + 2 * nf + 1)
        g = P.edge_graph_general(10, 12, 16, nf, "sum")
        assert (len(g.ops), len(g.ds)) == (nf + 1, 1 + nf + nf + 1)
        g = P.edge_graph_general(10, 12, 16, nf, "maxabs")
        assert (len(g.ops), len(g.ds)) == (2 * nf + 1, 1 + nf + 2 * nf + 1)
        assert g.io_lower_bound() == 2 * 10 * 12 + nf * 256
    g = P.edge_graph_general(1000, 1000, 16, 2, "max")
    assert (g.total_temp(), g.io_lower_bound(), g.baseline()) == (6_000_512, 2_000_512, 13_000_512)
