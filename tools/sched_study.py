"""Heuristic gap of the paper's operator schedule: on the Fig. 3 / Fig. 6
instance and on random DAGs, the transfer volume of several operator orders -- the paper's DFS
(tg_sched_dfs_order), DFS with reversed child order, Kahn (breadth-first)
order, insertion order -- each with the next-use transfer rule (tg_sched_transfers), against
the exact optimum over all orders (tg_sched_optimal). CPU only; library calls only.

  python tools/sched_study.py [--dags 300] [--max-ops 9] > profiles/r01/sched_study.json
"""
import argparse
import json
import os
import random
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_sundaramrc09_b200 import tg  # noqa: E402


class G:
    def __init__(self):
        self.ds, self.ops = [], []  # ds: [size, kind]; ops: (ins, outs)


def random_dag(rng, n_ops):
    g = G()
    avail = []
    for _ in range(rng.randint(1, 3)):
        g.ds.append([rng.randint(1, 4), tg.TG_DS_INPUT])
        avail.append(len(g.ds) - 1)
    for _ in range(n_ops):
        ins = rng.sample(avail, min(len(avail), rng.randint(1, 3)))
        outs = []
        for _ in range(rng.randint(1, 2)):
            g.ds.append([rng.randint(1, 4), tg.TG_DS_TEMP])
            outs.append(len(g.ds) - 1)
        g.ops.append((ins, outs))
        avail.extend(outs)
    read = {j for ins, _ in g.ops for j in ins}
    for j, d in enumerate(g.ds):
        if d[1] == tg.TG_DS_TEMP and j not in read:
            d[1] = tg.TG_DS_OUTPUT
    return g


def fig3():
    """Fig. 3 / Fig. 6: Im 2 units, the others 1, memory 5 units."""
    g = G()
    names = ["Im", "E1'", "E1''", "E2'", "E2''", "E5'", "E5''", "E6'", "E6''", "E'", "E''"]
    ix = {n: i for i, n in enumerate(names)}
    for n in names:
        g.ds.append([2 if n == "Im" else 1, tg.TG_DS_INPUT if n == "Im" else
                     tg.TG_DS_OUTPUT if n in ("E'", "E''") else tg.TG_DS_TEMP])
    for ins, outs in [(["Im"], ["E1'", "E1''"]), (["Im"], ["E2'", "E2''"]), (["E1'"], ["E5'"]),
                      (["E1''"], ["E5''"]), (["E2'"], ["E6'"]), (["E2''"], ["E6''"]),
                      (["E1'", "E2'", "E5'", "E6'"], ["E'"]), (["E1''", "E2''", "E5''", "E6''"], ["E''"])]:
        g.ops.append(([ix[n] for n in ins], [ix[n] for n in outs]))
    return g


def to_sched(g):
    s = tg.Sched()
    for size, kind in g.ds:
        s.add_ds(size, kind)
    for ins, outs in g.ops:
        s.add_op(ins, outs)
    return s


def deps(g):
    prod = {j: i for i, (_, outs) in enumerate(g.ops) for j in outs}
    preds = [{prod[j] for j in ins if j in prod} for ins, _ in g.ops]
    cons = [sorted({c for c in range(len(g.ops)) if i in preds[c]}) for i in range(len(g.ops))]
    return preds, cons


def dfs(g, reverse=False):
    preds, cons = deps(g)
    seen, order = set(), []

    def visit(i):
        seen.add(i)
        order.append(i)
        for c in (reversed(cons[i]) if reverse else cons[i]):
            if c not in seen and preds[c] <= seen:
                visit(c)

    for r in range(len(g.ops)):
        if r not in seen and preds[r] <= seen:
            visit(r)
    return order


def kahn(g):
    preds, _ = deps(g)
    placed, order = set(), []
    while len(order) < len(g.ops):
        layer = [i for i in range(len(g.ops)) if i not in placed and preds[i] <= placed]
        order.extend(layer)
        placed.update(layer)
    return order


def study(g, cap):
    s = to_sched(g)
    opt, _, n_orders, n_best = s.optimal(cap)
    r = {"optimum": opt, "orders": n_orders, "optimal_orders": n_best}
    for name, order in [("dfs_paper", s.dfs_order()), ("dfs_reversed", dfs(g, True)), ("kahn", kahn(g)),
                        ("insertion", list(range(len(g.ops))))]:
        r[name] = s.transfers(order, cap)
    assert s.dfs_order() == dfs(g)  # the library's DFS is the one restated here
    return r


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dags", type=int, default=300)
    ap.add_argument("--max-ops", type=int, default=9)
    ap.add_argument("--seed", type=int, default=2009)
    args = ap.parse_args()
    out = {"what": "transfer volume of operator orders under the next-use rule vs the exact optimum over all "
                   "orders (tg_sched_optimal)", "fig3_fig6": study(fig3(), 5)}
    rng = random.Random(args.seed)
    rows = []
    for _ in range(args.dags):
        g = random_dag(rng, rng.randint(4, args.max_ops))
        need = max(sum(g.ds[j][0] for j in set(ins) | set(outs)) for ins, outs in g.ops)
        for slack in (0, 2):
            rows.append(study(g, need + slack))
    agg = {}
    for h in ("dfs_paper", "dfs_reversed", "kahn", "insertion"):
        ratios = [r[h] / r["optimum"] for r in rows if r["optimum"] > 0]
        agg[h] = {"mean_ratio_to_optimum": statistics.mean(ratios), "max_ratio": max(ratios),
                  "optimal_fraction": sum(1 for r in rows if r[h] == r["optimum"]) / len(rows)}
    out["random_dags"] = {"instances": len(rows), "ops": f"4..{args.max_ops}", "seed": args.seed,
                          "capacity": "largest single-operator footprint (+0 and +2 units)", "heuristics": agg}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
