"""Test helper (not the oracle, not the product): small operator graphs described once and
turned into (a) the splitting oracle's input (oracle.planner.SNode lists), (b) a library
graph through the C ABI binding, and (c) a plain numpy executor that evaluates the graph
unsplit or piece by piece following the oracle's split plan -- the CPU check of the paper's
claim that splitting does not change the result.

Every node writes fp32; convolutions accumulate in fp64 over (ci, i, j) and round once, so
a row's value does not depend on which piece computes it (bit-exact split == unsplit)."""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from oracle import planner as P


@dataclass
class Spec:
    shapes: list = field(default_factory=list)   # (n, c, h, w) per DS
    kinds: list = field(default_factory=list)    # input | param | temp | output
    data: dict = field(default_factory=dict)     # DS id -> np.float32 array (inputs, params)
    nodes: list = field(default_factory=list)    # P.SNode
    ops: list = field(default_factory=list)      # per node: dict(op=..., pad/elem/a/b/s)
    output: int = -1

    def ds(self, shape, kind="temp", data=None) -> int:
        shape = (1,) * (4 - len(shape)) + tuple(int(v) for v in shape)   # the binding's _dims4
        self.shapes.append(shape)
        self.kinds.append(kind)
        if data is not None:
            self.data[len(self.shapes) - 1] = np.ascontiguousarray(data, np.float32).reshape(shape)
        return len(self.shapes) - 1

    # ---- operators (shapes as the library infers them)
    def conv(self, x, k, bias=-1, pad="valid"):
        n, ci, h, w = self.shapes[x]
        co, _, kh, kw = self.shapes[k]
        ho, wo = (h, w) if pad == "same" else (h - kh + 1, w - kw + 1)
        y = self.ds((n, co, ho, wo))
        ins = [x, k] + ([bias] if bias >= 0 else [])
        plane = bias >= 0 and int(np.prod(self.shapes[bias])) != co
        self.nodes.append(P.SNode("conv_same" if pad == "same" else "conv_valid", ins, y, kh=kh, bias_plane=plane))
        self.ops.append(dict(op="conv", pad=pad, kh=kh, kw=kw))
        return y

    def elem(self, op, xs, a=1.0, b=0.0):
        y = self.ds(self.shapes[xs[0]])
        self.nodes.append(P.SNode("elem", list(xs), y))
        self.ops.append(dict(op=op, a=a, b=b))
        return y

    def sub(self, x, p, s=2):
        n, c, h, w = self.shapes[x]
        y = self.ds((n, c, (h - s) // s + 1, (w - s) // s + 1))
        self.nodes.append(P.SNode("sub", [x, p], y, s=s))
        self.ops.append(dict(op="sub", s=s))
        return y

    def matmul(self, a, b):
        m, k = self.shapes[a][2:]
        n = self.shapes[b][3]
        y = self.ds((1, 1, m, n))
        self.nodes.append(P.SNode("matmul", [a, b], y))
        self.ops.append(dict(op="matmul"))
        return y

    def set_output(self, y):
        self.kinds[y] = "output"
        self.output = y

    def plan(self, capacity):
        return P.split_plan(self.shapes, self.kinds, self.nodes, self.output, capacity)

    def total_bytes(self):
        return sum(4 * int(np.prod(s)) for s in self.shapes)


# ------------------------------------------------------------------------------ graphs
def edge_spec(H, W, K1, K2, n=1, rng=None, img=None):
    s = Spec()
    if img is None:
        img = (np.random.default_rng(rng).integers(0, 256, (n, 1, H, W)) / 255).astype(np.float32)
    x = s.ds((n, 1, H, W), "input", img)
    k1 = s.ds((1, 1) + K1.shape, "param", K1)
    k2 = s.ds((1, 1) + K2.shape, "param", K2)
    e1 = s.conv(x, k1, pad="same")
    e2 = s.conv(x, k2, pad="same")
    e = s.elem("max", [e1, e2, s.elem("neg", [e1]), s.elem("neg", [e2])])
    s.set_output(e)
    return s


def cnn_spec(n, H, W, n5, prm, bias_plane=True, img=None, seed=0):
    """The F2 CNN at layer granularity from primitives (C1 T S2 T C3 T S4 T C5 T C6)."""
    s = Spec()
    if img is None:
        img = (np.random.default_rng(seed).integers(0, 256, (n, 1, H, W)) / 255).astype(np.float32)
    x = s.ds((n, 1, H, W), "input", img)
    K1, B1, P2, K3, B3, P4, K5, B5, K6, B6 = prm
    ids = [s.ds(p.shape, "param", p) for p in prm]
    k1, b1, p2, k3, b3, p4, k5, b5, k6, b6 = ids
    t = s.elem("tanh", [s.conv(x, k1, b1)])
    t = s.elem("tanh", [s.sub(t, p2)])
    t = s.elem("tanh", [s.conv(t, k3, b3)])
    t = s.elem("tanh", [s.sub(t, p4)])
    t = s.elem("tanh", [s.conv(t, k5, b5)])
    y = s.conv(t, k6, b6)
    s.set_output(y)
    return s


def mixed_spec(H, W, M, seed=0):
    """conv VALID 3x3 + bias plane -> tanh -> subsample -> matmul (the second matrix whole,
    PAPER.md:369) -> affine: every splitting rule in one chain."""
    rng = np.random.default_rng(seed)
    s = Spec()
    x = s.ds((1, 1, H, W), "input", rng.random((1, 1, H, W)))
    k = s.ds((1, 1, 3, 3), "param", rng.uniform(-0.5, 0.5, (1, 1, 3, 3)))
    b = s.ds((1, 1, H - 2, W - 2), "param", rng.uniform(-0.1, 0.1, (1, 1, H - 2, W - 2)))
    p = s.ds((1, 2, 2), "param", rng.uniform(-0.5, 0.5, (1, 2, 2)))
    t = s.elem("tanh", [s.conv(x, k, b)])
    u = s.sub(t, p)
    wq = s.shapes[u][3]
    B = s.ds((1, 1, wq, M), "param", rng.uniform(-1, 1, (1, 1, wq, M)))
    y = s.elem("affine", [s.matmul(u, B)], a=0.5, b=0.25)
    s.set_output(y)
    return s


# ------------------------------------------------------------------------------ numpy executor
def _conv_rows(x, xa, K, pad, a, b, H):
    """Output rows [a, b) of a conv whose input band x holds rows [xa, xa + rows)."""
    n, ci, _, W = x.shape
    co, _, kh, kw = K.shape
    pt, pl = ((kh - 1) // 2, (kw - 1) // 2) if pad == "same" else (0, 0)
    wo = W if pad == "same" else W - kw + 1
    r0, r1 = a - pt, b - pt + kh - 1          # input rows needed (before clipping)
    ext = np.zeros((n, ci, r1 - r0, W + (kw - 1 if pad == "same" else 0)), np.float64)
    lo, hi = max(r0, 0), min(r1, H)
    ext[:, :, lo - r0:hi - r0, pl:pl + W] = x[:, :, lo - xa:hi - xa, :]
    acc = np.zeros((n, co, b - a, wo), np.float64)
    for o in range(co):
        for c in range(ci):
            for i in range(kh):
                for j in range(kw):
                    acc[:, o] += ext[:, c, i:i + b - a, j:j + wo] * np.float64(K[o, c, i, j])
    return acc


def eval_node(spec, i, bands, a, b):
    """Rows [a, b) of node i's output; bands[d] = (array, first row) of every input."""
    nd, op = spec.nodes[i], spec.ops[i]
    if op["op"] == "conv":
        x, xa = bands[nd.ins[0]]
        K = bands[nd.ins[1]][0]
        acc = _conv_rows(x, xa, K, op["pad"], a, b, spec.shapes[nd.ins[0]][2])
        if len(nd.ins) > 2:
            bb, ba = bands[nd.ins[2]]
            if nd.bias_plane:
                acc = acc.astype(np.float32).astype(np.float64) + bb[:, :, a - ba:b - ba]
            else:
                acc = acc.astype(np.float32).astype(np.float64) + bb.reshape(1, -1, 1, 1)
        return acc.astype(np.float32)
    if op["op"] == "sub":
        x, xa = bands[nd.ins[0]]
        Pw = bands[nd.ins[1]][0].reshape(-1, op["s"], op["s"])
        s_ = op["s"]
        n, c = x.shape[:2]
        wo = spec.shapes[nd.out][3]
        acc = np.zeros((n, c, b - a, wo), np.float64)
        for u in range(s_):
            for v in range(s_):
                rows = x[:, :, s_ * a + u - xa:s_ * (b - 1) + u + 1 - xa:s_, v:v + s_ * (wo - 1) + 1:s_]
                acc += rows.astype(np.float64) * Pw[:, u, v].reshape(1, -1, 1, 1)
        return acc.astype(np.float32)
    if op["op"] == "matmul":
        A, aa = bands[nd.ins[0]]
        Bm = bands[nd.ins[1]][0]
        return (A[0, 0, a - aa:b - aa].astype(np.float64) @ Bm[0, 0].astype(np.float64)).astype(np.float32)[None, None]
    xs = [bands[d][0][:, :, a - bands[d][1]:b - bands[d][1]] for d in nd.ins]
    if op["op"] == "tanh":
        return np.tanh(xs[0].astype(np.float64)).astype(np.float32)
    if op["op"] == "neg":
        return -xs[0]
    if op["op"] == "abs":
        return np.abs(xs[0])
    if op["op"] == "affine":
        return (np.float32(op["a"]) * xs[0] + np.float32(op["b"])).astype(np.float32)
    if op["op"] == "add":
        v = xs[0]
        for t in xs[1:]:
            v = (v + t).astype(np.float32)
        return v
    if op["op"] == "max":
        v = xs[0]
        for t in xs[1:]:
            v = np.where(t > v, t, v)
        return v
    raise ValueError(op)


def run_unsplit(spec):
    vals = {d: (a, 0) for d, a in spec.data.items()}
    for i, nd in enumerate(spec.nodes):
        vals[nd.out] = (eval_node(spec, i, vals, 0, spec.shapes[nd.out][2]), 0)
    return vals[spec.output][0]


def run_split(spec, plan):
    """Execute the piece operators of an oracle split plan in its DFS order, each reading
    only the DS pieces the plan gives it (a piece is the rows [r0, r1) of its DS)."""
    g = plan["graph"]
    store = {}
    for pid, (d, r0, r1) in enumerate(plan["pieces"]):
        if d in spec.data:
            store[pid] = spec.data[d][:, :, r0:r1]
    out = np.full(tuple(spec.shapes[spec.output]), np.nan, np.float32)
    for o in plan["order"]:
        i, _ = plan["op_piece"][o]
        nd = spec.nodes[i]
        bands = {}
        for pid in g.ops[o].ins:
            d, r0, r1 = plan["pieces"][pid]
            if d in bands and bands[d][1] <= r0:    # whole reads of a split DS: stitch pieces
                prev, pa = bands[d]
                bands[d] = (np.concatenate([prev[:, :, :r0 - pa], store[pid]], axis=2), pa)
            else:
                bands[d] = (store[pid], r0)
        (opid,) = g.ops[o].outs
        d, a, b = plan["pieces"][opid]
        store[opid] = eval_node(spec, i, bands, a, b)
        if d == spec.output:
            out[:, :, a:b] = store[opid]
    return out


# ------------------------------------------------------------------------------ library graph
def lib_graph(spec, out, budget=0, torch_runtime=False):
    """The same graph through the C ABI (DS ids in the same creation order as the spec)."""
    from paper_conf_ipps_sundaramrc09_b200 import tg
    g = tg.Graph()
    made = {}
    node_of = {nd.out: i for i, nd in enumerate(spec.nodes)}
    codes = {"add": tg.TG_ADD, "neg": tg.TG_NEG, "affine": tg.TG_AFFINE, "abs": tg.TG_ABS}
    for d in range(len(spec.shapes)):
        if d in spec.data:
            a = spec.data[d]
            made[d] = g.input(a) if spec.kinds[d] == "input" else g.param(a)
            continue
        i = node_of[d]
        nd, op = spec.nodes[i], spec.ops[i]
        xs = [made[x] for x in nd.ins]
        if op["op"] == "conv":
            y = g.conv2d(xs[0], xs[1], xs[2] if len(xs) > 2 else -1, tg.TG_SAME if op["pad"] == "same" else tg.TG_VALID)
        elif op["op"] == "sub":
            y = g.subsample(xs[0], xs[1], op["s"])
        elif op["op"] == "matmul":
            y = g.matmul(xs[0], xs[1])
        elif op["op"] == "tanh":
            y = g.tanh(xs[0])
        elif op["op"] == "max":
            y = g.max_combine(xs)
        else:
            y = g.elementwise(codes[op["op"]], xs, op["a"], op["b"])
        assert y == d, (y, d)
        assert tuple(g.shape(y)) == tuple(spec.shapes[d])
        made[d] = y
    g.output(made[spec.output], out)
    g.set(budget=budget, torch_runtime=torch_runtime)
    return g


# ------------------------------------------------------------------------------ random graphs
def random_spec(seed: int) -> Spec:
    """A random operator graph for fuzzing the splitting rule: a chain of 3-8 operators over a
    small image with side branches (elementwise ops of two same-shape data structures), VALID
    and SAME convolutions (1/3/5-tap kernels, 1-3 maps, bias plane / scalar / none), tanh,
    remap, abs, affine, subsample and -- on single-plane data -- matmul."""
    rng = np.random.default_rng(seed)
    s = Spec()
    n, c = int(rng.integers(1, 3)), int(rng.integers(1, 3))
    if rng.random() < 0.3:
        n = c = 1
    h, w = int(rng.integers(24, 90)), int(rng.integers(12, 40))
    x = s.ds((n, c, h, w), "input", rng.random((n, c, h, w)))
    cur = x
    pool = [x]
    for _ in range(int(rng.integers(3, 9))):
        N, C, H, W = s.shapes[cur]
        r = rng.random()
        if r < 0.3 and H >= 6 and W >= 6:
            kh = int(rng.choice([1, 3, 5]))
            co = int(rng.integers(1, 4))
            pad = "same" if rng.random() < 0.5 else "valid"
            k = s.ds((co, C, kh, kh), "param", rng.uniform(-0.5, 0.5, (co, C, kh, kh)))
            ho, wo = (H, W) if pad == "same" else (H - kh + 1, W - kh + 1)
            bk = rng.random()
            if bk < 0.4:
                b = s.ds((1, co, ho, wo), "param", rng.uniform(-0.1, 0.1, (1, co, ho, wo)))
            elif bk < 0.7:
                b = s.ds((co,), "param", rng.uniform(-0.1, 0.1, (co,)))
            else:
                b = -1
            cur = s.conv(cur, k, b, pad)
        elif r < 0.45:
            cur = s.elem("tanh", [cur])
        elif r < 0.55:
            cur = s.elem(str(rng.choice(["neg", "abs"])), [cur])
        elif r < 0.62:
            cur = s.elem("affine", [cur], a=float(rng.uniform(-2, 2)), b=float(rng.uniform(-1, 1)))
        elif r < 0.77:
            same = [d for d in pool if s.shapes[d] == s.shapes[cur] and d != cur]
            if same:
                other = int(rng.choice(same))
                cur = s.elem(str(rng.choice(["add", "max"])), [cur, other] if rng.random() < 0.5 else [other, cur])
            else:
                cur = s.elem("tanh", [cur])
        elif r < 0.9 and H >= 4 and W >= 4:
            p = s.ds((C, 2, 2), "param", rng.uniform(-0.5, 0.5, (C, 2, 2)))
            cur = s.sub(cur, p)
        elif N == 1 and C == 1:
            m = int(rng.integers(3, 30))
            B = s.ds((1, 1, W, m), "param", rng.uniform(-1, 1, (1, 1, W, m)))
            cur = s.matmul(cur, B)
        else:
            cur = s.elem("tanh", [cur])
        pool.append(cur)
    s.set_output(cur)
    return s
