"""The paper-faithful plans of the library (TG_PER_OP: per-operator offload units, DFS order,
latest-time-of-use transfers; TG_BASELINE: PAPER.md:613) built through the
C ABI on a CPU-only box: Table 1 edge counts on a real plan and the schedule
bit-exact against the planner oracle for several budgets (edge and CNN graphs)."""
import numpy as np
import pytest

import synth
from oracle import planner as P

KIND = {0: "input", 1: "param", 2: "temp", 3: "output"}


def edge_plan(mode, H=1000, W=1000, budget=0):
    from paper_conf_ipps_sundaramrc09_b200 import tg
    img = np.zeros((1, 1, H, W), np.float32)
    K1, K2 = synth.random_edge_filters_np(3)
    g, _ = tg.edge_graph(img, K1, K2, out=np.zeros_like(img))
    g.set(budget=budget)
    return g.plan(mode)


def oracle_of(js):
    g = P.Graph()
    for i, (size, kind) in enumerate(js["ds"]):
        g.add_ds(f"d{i}", size, KIND[kind])
    for i, (ins, outs) in enumerate(js["ops"]):
        g.add_op(f"o{i}", ins, outs)
    return g


def check_against_oracle(js):
    g = oracle_of(js)
    order = P.dfs_order(g)
    assert js["order"] == order
    if js["mode"] == "per_op":
        tr = []
        moved = P.simulate_transfers(g, order, js["capacity"], tr)
        kind = {"h2d": 0, "run": 1, "d2h": 2}
        names_ds = {d.name: i for i, d in enumerate(g.ds)}
        names_op = {o.name: i for i, o in enumerate(g.ops)}
        want = [[kind[k], names_op[n] if k == "run" else names_ds[n]] for k, n in tr]
        assert js["trace"] == want
        assert js["h2d_bytes"] + js["d2h_bytes"] == moved


def test_table1_edge_counts_on_real_plans():
    from paper_conf_ipps_sundaramrc09_b200 import tg
    base = edge_plan(tg.TG_BASELINE)
    s = base.stats()
    assert (s["h2d_bytes"] + s["d2h_bytes"]) // 4 == 13000512      # Table 1 baseline
    assert s["total_temp_bytes"] // 4 == 6000512 and s["io_lower_bound_bytes"] // 4 == 2000512
    per = edge_plan(tg.TG_PER_OP)
    s = per.stats()
    assert (s["h2d_bytes"] + s["d2h_bytes"]) // 4 == 2000512       # all fits: I/O only
    j = per.json()
    assert j["mode"] == "per_op" and len(j["ops"]) == 5 and len(j["ds"]) == 8


@pytest.mark.parametrize("budget", [0, 40 << 20, 28 << 20, 24 << 20])
def test_edge_per_op_schedule_matches_oracle(budget):
    from paper_conf_ipps_sundaramrc09_b200 import tg
    p = edge_plan(tg.TG_PER_OP, budget=budget)
    j = p.json()
    check_against_oracle(j)
    if budget:
        assert j["arena_bytes"] == budget and j["capacity"] == budget - budget // 8
    check_against_oracle(edge_plan(tg.TG_BASELINE, budget=budget).json())


def test_baseline_infeasible_per_op_splits():
    """The max operator needs 5 x 4 MB: the baseline (operators whole) cannot
    run it in 16 MB, the paper's method splits it (tests/test_split_plan.py)."""
    from paper_conf_ipps_sundaramrc09_b200 import tg
    with pytest.raises(tg.TGError) as e:
        edge_plan(tg.TG_BASELINE, budget=16 << 20)
    assert e.value.code == tg.TG_E_INFEASIBLE
    j = edge_plan(tg.TG_PER_OP, budget=16 << 20).json()
    assert max(j["k"].values()) > 1 and len(j["ops"]) > 5


@pytest.mark.parametrize("budget", [0, 12 << 20, 6 << 20])
def test_cnn_per_op_schedule_matches_oracle(budget):
    from paper_conf_ipps_sundaramrc09_b200 import tg
    H, W, n5 = 120, 160, 20
    img = np.zeros((2, 1, H, W), np.float32)
    prm = synth.cnn_params_np(1, n5, H, W)
    h5, w5 = synth.cnn_dims(H, W)[4]
    g, _ = tg.cnn_graph(img, n5, prm, out=np.zeros((2, 9, h5, w5), np.float32))
    g.set(budget=budget)
    j = g.plan(tg.TG_PER_OP).json()
    assert len(j["ops"]) == 11
    check_against_oracle(j)
