"""Planner oracle -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Plain Python restatement of the paper's planning steps, written for checking by eye:

  * operator graphs with static footprints (PAPER.md:345, :349 fn. 1): `Graph`
  * the edge template graph of Fig. 1(b)/Fig. 3 and the CNN layers expanded as Fig. 7
  * Table 1 accounting: total temporary data, I/O lower bound, per-operator baseline
    
  * operator splitting: per-operator memory requirement and split factors
    (PAPER.md:359-365), Fig. 1(c) regimes
  * halo back-propagation "from the leaves to the root"
  * depth-first operator schedule and the "latest time of use" transfer
    schedule with eager deletion (read as NEXT use, R10)
  * brute force over all operator orders for tiny graphs (stands in for the PB model of
    Fig. 5)
  * what a fused plan's chunks read, write and move, given its chunk size (row bands,
    halos, shards, bytes; tests/test_plan_parity.py compares the library bit-exactly).
"""
from __future__ import annotations

import itertools
import math
from dataclasses import dataclass, field


# ============================================================================ graphs
@dataclass
class DS:
    name: str
    size: int               # floats (PAPER.md:741 counts floats)
    kind: str = "temp"      # "input" | "param" | "temp" | "output"


@dataclass
class Op:
    name: str
    ins: list[int]
    outs: list[int]


@dataclass
class Graph:
    ds: list[DS] = field(default_factory=list)
    ops: list[Op] = field(default_factory=list)

    def add_ds(self, name, size, kind="temp") -> int:
        self.ds.append(DS(name, int(size), kind))
        return len(self.ds) - 1

    def add_op(self, name, ins, outs) -> int:
        self.ops.append(Op(name, list(ins), list(outs)))
        return len(self.ops) - 1

    # ---- accounting (Table 1)
    def total_temp(self) -> int:
        """'Total temporary data needed': sum of the sizes of all data structures."""
        return sum(d.size for d in self.ds)

    def io_lower_bound(self) -> int:
        """'I/O transfers only (lower bound)': template inputs (data and parameters) plus
        template outputs, each moved once."""
        return sum(d.size for d in self.ds if d.kind in ("input", "param", "output"))

    def baseline(self) -> int:
        """Baseline of PAPER.md:613: 'For each operator, transfer input data to the GPU,
        perform the operation and copy the results back to the CPU immediately.'"""
        return sum(sum(self.ds[j].size for j in op.ins) + sum(self.ds[j].size for j in op.outs)
                   for op in self.ops)

    def req(self, op: Op) -> int:
        """Memory requirement of an operator: 'sum of sizes of data structures associated
        with each operator'."""
        return sum(self.ds[j].size for j in set(op.ins) | set(op.outs))


def edge_graph(H: int, W: int, ks: int = 16, orientations: int = 4, kernel_floats=True) -> Graph:
    """Edge template: `orientations`/2 convolutions with precomputed rotated kernels, as many
    remaps (negations), one max over all responses (Fig. 1(b), Fig. 3).
    4 orientations: C1 C2 R1 R2 max; 8 orientations: C1-C4 R1-R4 max (Fig. 1(b))."""
    g = Graph()
    S = H * W
    im = g.add_ds("Im", S, "input")
    nconv = orientations // 2
    ks_ = [g.add_ds(f"K{i+1}", ks * ks if kernel_floats else 0, "param") for i in range(nconv)]
    conv_out, remap_out = [], []
    for i in range(nconv):
        e = g.add_ds(f"E{i+1}", S)
        g.add_op(f"C{i+1}", [im, ks_[i]], [e])
        conv_out.append(e)
    for i in range(nconv):
        e = g.add_ds(f"E{i+1+nconv}", S)
        g.add_op(f"R{i+1}", [conv_out[i]], [e])
        remap_out.append(e)
    E = g.add_ds("E", S, "output")
    g.add_op("max", conv_out + remap_out, [E])
    return g


def edge_graph_general(H: int, W: int, ks: int, nf: int, combine: str) -> Graph:
    """Edge graph with nf convolutions combined by 'max' (responses and their remaps,
    PAPER.md:627-629), 'sum' (addition), 'maxabs' (max absolute value) or 'maxplain' (max of
    the responses) -- the reductions PAPER.md:621 lists."""
    if combine == "max":
        return edge_graph(H, W, ks, orientations=2 * nf)
    g = Graph()
    S = H * W
    im = g.add_ds("Im", S, "input")
    resp = []
    for i in range(nf):
        k = g.add_ds(f"K{i+1}", ks * ks, "param")
        e = g.add_ds(f"E{i+1}", S)
        g.add_op(f"C{i+1}", [im, k], [e])
        resp.append(e)
    if combine == "maxabs":
        absd = []
        for i, e in enumerate(resp):
            a = g.add_ds(f"A{i+1}", S)
            g.add_op(f"abs{i+1}", [e], [a])
            absd.append(a)
        resp = absd
    E = g.add_ds("E", S, "output")
    g.add_op("sum" if combine == "sum" else "max", resp, [E])
    return g


def cnn_dims(H: int, W: int):
    """Per-level plane sizes: VALID 5x5 convs and 2x2/2 subsampling
    with floor((D-2)/2)+1."""
    h1, w1 = H - 4, W - 4
    h2, w2 = (h1 - 2) // 2 + 1, (w1 - 2) // 2 + 1
    h3, w3 = h2 - 4, w2 - 4
    h4, w4 = (h3 - 2) // 2 + 1, (w3 - 2) // 2 + 1
    h5, w5 = h4 - 4, w4 - 4
    return [(h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5)]


def cnn_graph_fig7(H: int, W: int, n5: int) -> Graph:
    """CNN template expanded operator by operator as Fig. 7: per layer
    and output plane j, convolutions L_ij = In_i * K_ij, a chain of adds S_j1 = L_1j + L_2j,
    S_jk = S_j(k-1) + L_(k+1)j, and O_j = S_last + B_j with a full-size bias plane B_j;
    tanh: one op and one DS per plane; subsample: one op, a 4-float kernel and one output
    per plane."""
    g = Graph()
    (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5) = cnn_dims(H, W)
    planes = [g.add_ds("In1", H * W, "input")]

    def conv(planes_in, n_out, k, ho, wo, tag, last=False):
        outs = []
        for j in range(n_out):
            Ls = []
            for i, p in enumerate(planes_in):
                K = g.add_ds(f"{tag}.K{i+1}{j+1}", k * k, "param")
                L = g.add_ds(f"{tag}.L{i+1}{j+1}", ho * wo)
                g.add_op(f"{tag}.C{i+1}{j+1}", [p, K], [L])
                Ls.append(L)
            acc = Ls[0]
            for i in range(1, len(Ls)):
                S = g.add_ds(f"{tag}.S{j+1}{i}", ho * wo)
                g.add_op(f"{tag}.A{j+1}{i}", [acc, Ls[i]], [S])
                acc = S
            B = g.add_ds(f"{tag}.B{j+1}", ho * wo, "param")
            O = g.add_ds(f"{tag}.O{j+1}", ho * wo, "output" if last else "temp")
            g.add_op(f"{tag}.AB{j+1}", [acc, B], [O])
            outs.append(O)
        return outs

    def tanh(planes_in, size, tag):
        outs = []
        for i, p in enumerate(planes_in):
            o = g.add_ds(f"{tag}.T{i+1}", size)
            g.add_op(f"{tag}.tanh{i+1}", [p], [o])
            outs.append(o)
        return outs

    def sub(planes_in, size, tag):
        outs = []
        for i, p in enumerate(planes_in):
            P = g.add_ds(f"{tag}.P{i+1}", 4, "param")
            o = g.add_ds(f"{tag}.O{i+1}", size)
            g.add_op(f"{tag}.sub{i+1}", [p, P], [o])
            outs.append(o)
        return outs

    x = conv(planes, 8, 5, h1, w1, "C1")
    x = tanh(x, h1 * w1, "T1")
    x = sub(x, h2 * w2, "S2")
    x = tanh(x, h2 * w2, "T2")
    x = conv(x, 20, 5, h3, w3, "C3")
    x = tanh(x, h3 * w3, "T3")
    x = sub(x, h4 * w4, "S4")
    x = tanh(x, h4 * w4, "T4")
    x = conv(x, n5, 5, h5, w5, "C5")
    x = tanh(x, h5 * w5, "T5")
    conv(x, 9, 1, h5, w5, "C6", last=True)
    return g


def cnn_conv_accumulate_baseline(H: int, W: int, n5: int) -> int:
    """Layer-level baseline variant: every conv pair moves In_i + K_ij + the
    accumulator in and the accumulator out; tanh moves in + out; subsample in + P + out.
    Only the large-minus-small differences are pinned by Table 1."""
    (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5) = cnn_dims(H, W)
    A0, A1, A2, A3, A4, A5 = H * W, h1 * w1, h2 * w2, h3 * w3, h4 * w4, h5 * w5
    t = 0
    for n_in, n_out, k, a_in, a_out in [(1, 8, 5, A0, A1), (8, 20, 5, A2, A3),
                                         (20, n5, 5, A4, A5), (n5, 9, 1, A5, A5)]:
        t += n_in * n_out * (a_in + k * k + 2 * a_out)
    t += 8 * 2 * A1 + 8 * (A1 + 4 + A2) + 8 * 2 * A2          # T1, S2, T2
    t += 20 * 2 * A3 + 20 * (A3 + 4 + A4) + 20 * 2 * A4       # T3, S4, T4
    t += n5 * 2 * A5                                          # T5
    return t


# ============================================================================ splitting
def split_factors(g: Graph, M: int) -> dict[str, int]:
    """Paper-mode operator splitting: an operator whose requirement
    exceeds the GPU memory M is split into k = ceil(req/M) equal pieces."""
    return {op.name: max(1, math.ceil(g.req(op) / M)) for op in g.ops}


def fig1c_regime(S: float, M: float = 1500.0) -> str:
    """Fig. 1(c) strategy for the 8-orientation edge graph at image size S on a GPU of
    memory M, from req(C)=req(R)=2S, req(max)=9S, total=10S."""
    g = edge_graph(1, 1, orientations=8, kernel_floats=False)
    req = {op.name: g.req(op) * S for op in g.ops}
    total = g.total_temp() * S
    if S > M:
        return "input_chunked"
    if total <= M:
        return "all_fit"
    if req["max"] <= M:
        return "max_separate"
    if max(req[o] for o in req if o != "max") <= M:
        return "max_split"
    return "conv_remap_split"


def back_propagate_rows(layers, r0: int, r1: int, H_in: int | None = None):
    """Walk a chain of row-local operators from the output back to the input ('traversing
    the split graph from the leaves to the root and inferring the sizes and offsets from
    the kernel and output sizes'). layers: list of (kind, param) from input
    to output, kind in {"valid", "same", "sub", "elem"}. Returns the row range needed at
    every level, input first. SAME ranges are clipped to [0, H_in) (zeros outside)."""
    ranges = [(r0, r1)]
    a, b = r0, r1
    for kind, p in reversed(layers):
        if kind == "valid":
            a, b = a, b + p - 1
        elif kind == "same":
            a, b = a - (p - 1) // 2, b + p // 2
            if H_in is not None:
                a, b = max(0, a), min(H_in, b)
        elif kind == "sub":
            a, b = p * a, p * b
        elif kind == "elem":
            pass
        else:
            raise ValueError(kind)
        ranges.append((a, b))
    return list(reversed(ranges))


CNN_LAYERS = [("valid", 5), ("elem", 0), ("sub", 2), ("elem", 0), ("valid", 5), ("elem", 0),
              ("sub", 2), ("elem", 0), ("valid", 5), ("elem", 0), ("valid", 1)]


# ============================================================================ scheduling
def dfs_order(g: Graph) -> list[int]:
    """Depth-first operator schedule: schedule the entire sub-tree of a
    child before its siblings; a node whose inputs are not ready is skipped (backtrack to
    the parent and explore its other children). Children = consumers of an op's outputs in
    graph-insertion order; start nodes in id order (R11)."""
    producer = {}
    for i, op in enumerate(g.ops):
        for j in op.outs:
            producer[j] = i
    preds = [{producer[j] for j in op.ins if j in producer} for op in g.ops]
    consumers = [[] for _ in g.ops]
    for c, op in enumerate(g.ops):
        for j in op.ins:
            if j in producer and c not in consumers[producer[j]]:
                consumers[producer[j]].append(c)
    for lst in consumers:
        lst.sort()
    done: list[int] = []
    seen = set()

    def visit(i):
        done.append(i)
        seen.add(i)
        for c in consumers[i]:
            if c not in seen and preds[c] <= seen:
                visit(c)

    for i in range(len(g.ops)):
        if i not in seen and preds[i] <= seen:
            visit(i)
    assert len(done) == len(g.ops)
    return done


def simulate_transfers(g: Graph, order: list[int], capacity: int, trace=None, frees: bool = False) -> int:
    """Transfer volume of an operator order under the 'latest time of use' policy
    (read as next use -- DESIGN.md R10):
      * the inputs and outputs of the running operator must be resident; a missing input is
        copied to the GPU; outputs are allocated on the GPU;
      * on shortage, move to the CPU the resident DS whose next use is furthest in the
        future (no further use = infinitely far); ties: host-valid (clean) data first, then
        lowest DS id; clean data is dropped for free, dirty data costs a copy to the CPU;
      * data is deleted eagerly once no later operator uses it (template outputs are
        instead copied to the CPU when evicted or at the end);
      * initially everything is on the CPU, nothing on the GPU (PB constraints (11),(12)).
    Returns the number of floats moved (H2D + D2H). With frees=True the trace also records
    ("free", name) whenever a DS leaves the GPU (evicted, or deleted eagerly in id order)."""
    uses = {j: [] for j in range(len(g.ds))}
    for t, i in enumerate(order):
        for j in set(g.ops[i].ins) | set(g.ops[i].outs):
            uses[j].append(t)
    outputs = {j for j, d in enumerate(g.ds) if d.kind == "output"}
    on_gpu: dict[int, bool] = {}          # DS -> dirty (GPU copy newer than host)
    host_valid = {j for j, d in enumerate(g.ds) if d.kind in ("input", "param")}
    moved = 0

    def next_use(j, t):
        for u in uses[j]:
            if u > t:
                return u
        return math.inf

    def used(t):
        return sum(g.ds[j].size for j in on_gpu)

    for t, i in enumerate(order):
        op = g.ops[i]
        need = list(dict.fromkeys(list(op.ins) + list(op.outs)))
        pinned = set(need)
        for j in need:
            if j in on_gpu:
                continue
            sz = g.ds[j].size
            while used(t) + sz > capacity:
                cands = [k for k in on_gpu if k not in pinned]
                if not cands:
                    raise RuntimeError("operator does not fit")
                cands.sort(key=lambda k: (-next_use(k, t), 0 if not on_gpu[k] else 1, k))
                v = cands[0]
                if on_gpu[v] and (next_use(v, t) != math.inf or v in outputs):
                    moved += g.ds[v].size          # write back dirty data still needed
                    host_valid.add(v)
                    if trace is not None:
                        trace.append(("d2h", g.ds[v].name))
                del on_gpu[v]
                if trace is not None and frees:
                    trace.append(("free", g.ds[v].name))
            if j in op.ins:
                assert j in host_valid, g.ds[j].name
                moved += sz
                on_gpu[j] = False
                if trace is not None:
                    trace.append(("h2d", g.ds[j].name))
            else:
                on_gpu[j] = True
                host_valid.discard(j)
        if trace is not None:
            trace.append(("run", op.name))
        # eager deletion of data no later operator needs (outputs stay until copied back)
        for j in sorted(on_gpu):
            if next_use(j, t) == math.inf and j not in outputs:
                del on_gpu[j]
                if trace is not None and frees:
                    trace.append(("free", g.ds[j].name))
    for j in sorted(on_gpu):          # outputs still on the GPU go to the host, in id order
        if j in outputs and on_gpu[j]:
            moved += g.ds[j].size
            if trace is not None:
                trace.append(("d2h", g.ds[j].name))
    return moved


def topological_orders(g: Graph):
    """All operator orders that respect the data dependences (PB constraints (1)-(3))."""
    producer = {}
    for i, op in enumerate(g.ops):
        for j in op.outs:
            producer[j] = i
    preds = [{producer[j] for j in op.ins if j in producer} for op in g.ops]
    n = len(g.ops)

    def rec(prefix, placed):
        if len(prefix) == n:
            yield list(prefix)
            return
        for i in range(n):
            if i not in placed and preds[i] <= placed:
                prefix.append(i)
                placed.add(i)
                yield from rec(prefix, placed)
                placed.discard(i)
                prefix.pop()

    yield from rec([], set())


def brute_force_min_transfers(g: Graph, capacity: int):
    """Exhaustive minimum over all operator orders of the next-use transfer volume (a
    tiny-graph stand-in for the PB optimum of Fig. 5/Fig. 6). Returns (min, n_orders,
    n_optimal_orders)."""
    best, n, nbest = math.inf, 0, 0
    for order in topological_orders(g):
        n += 1
        v = simulate_transfers(g, order, capacity)
        if v < best:
            best, nbest = v, 1
        elif v == best:
            nbest += 1
    return best, n, nbest


def fig3_graph() -> tuple[Graph, dict[str, int]]:
    """The split edge graph of Fig. 3 / Fig. 6: Im is 2 units, every
    other DS 1 unit, convolution/remap/max split in two (kernels not drawn, size 0)."""
    g = Graph()
    im = g.add_ds("Im", 2, "input")
    e = {}
    for nm in ["E1'", "E1''", "E2'", "E2''", "E5'", "E5''", "E6'", "E6''"]:
        e[nm] = g.add_ds(nm, 1)
    e["E'"] = g.add_ds("E'", 1, "output")
    e["E''"] = g.add_ds("E''", 1, "output")
    ops = {}
    ops["C1"] = g.add_op("C1", [im], [e["E1'"], e["E1''"]])
    ops["C2"] = g.add_op("C2", [im], [e["E2'"], e["E2''"]])
    ops["R1'"] = g.add_op("R1'", [e["E1'"]], [e["E5'"]])
    ops["R1''"] = g.add_op("R1''", [e["E1''"]], [e["E5''"]])
    ops["R2'"] = g.add_op("R2'", [e["E2'"]], [e["E6'"]])
    ops["R2''"] = g.add_op("R2''", [e["E2''"]], [e["E6''"]])
    ops["max1"] = g.add_op("max1", [e["E1'"], e["E2'"], e["E5'"], e["E6'"]], [e["E'"]])
    ops["max2"] = g.add_op("max2", [e["E1''"], e["E2''"], e["E5''"], e["E6''"]], [e["E''"]])
    return g, ops


# ============================================================================ operator splitting
# The paper's splitting algorithm (steps 1-3) on an operator graph with
# static shapes, in the reading DESIGN.md R19:
#   * the split axis is the output rows (R12); an operator's inputs are "row-linked" when an
#     output row band needs only a row band of them (convolution image, bias plane,
#     subsample input, elementwise inputs, the first matrix of a matmul -- PAPER.md:369
#     "breaking up one of the input matrices and the output matrix") and "whole" otherwise
#     (convolution kernels, "should not be split"; subsample weights; the
#     second matrix of a matmul; scalar biases);
#   * "When an operator is split, other operators that produce/receive data from the split
#     operator also need to be modified": the operators joined by row-linked
#     data form a component that is split into the same number k of pieces;
#   * the pieces of every data structure are found "by traversing the split graph from the
#     leaves to the root and inferring the sizes and offsets from the kernel and output
#     sizes": the component's sinks are cut into k equal row bands
#     [i*h//k, (i+1)*h//k), and each input band is the band its consumers' piece i needs
#     (the hull over consumers), halos included -- so input pieces overlap (the paper's
#     "two 100x52 input matrices (not 100x50)");
#   * k starts at max ceil(req(op) / M) over the component's operators (step 2) and grows by
#     one until every piece operator fits (step 3); a component whose operators all fit
#     stays whole (k = 1, every data structure one piece).


@dataclass
class SNode:
    """A graph operator with its row semantics (for splitting only)."""
    kind: str                  # "conv_valid" | "conv_same" | "sub" | "elem" | "matmul"
    ins: list[int]             # graph DS ids in the library's order (conv: x, k[, bias])
    out: int
    kh: int = 1                # convolution kernel rows
    s: int = 1                 # subsample window = stride
    bias_plane: bool = False   # conv: the third input is a bias plane (row-linked)


def in_rows(node: SNode, slot: int, a: int, b: int, h_in: int):
    """Rows of input `slot` that output rows [a, b) of `node` need, or None if the input is
    read whole. (the 5x5 VALID conv's output rows [0, 48) need input rows
    [0, 52).)"""
    if node.kind == "conv_valid":
        if slot == 0:
            return (a, b + node.kh - 1)
        return (a, b) if slot == 2 and node.bias_plane else None
    if node.kind == "conv_same":
        if slot == 0:
            return (max(0, a - (node.kh - 1) // 2), min(h_in, b + node.kh // 2))
        return (a, b) if slot == 2 and node.bias_plane else None
    if node.kind == "sub":
        return (node.s * a, node.s * b) if slot == 0 else None
    if node.kind == "matmul":
        return (a, b) if slot == 0 else None
    return (a, b)              # elementwise / tanh / max: row for row


def split_plan(shapes, kinds, nodes: list[SNode], output: int, capacity: int, force_k: int | None = None):
    """Split the operators feeding `output` (reading R19) and schedule the
    pieces with the DFS order and the next-use transfer policy.
    shapes[d] = (n, c, h, w), kinds[d] in {"input", "param", "temp", "output"}; sizes are
    bytes of fp32. Returns a dict with the pieces, piece operators, k per node, order and
    trace; raises ValueError when some operator cannot be made to fit. force_k (tests only):
    cut every component that needs splitting into exactly force_k pieces, fitting or not."""
    def nbytes(d, rows):
        return 4 * shapes[d][0] * shapes[d][1] * rows * shapes[d][3]

    # step 0: the operators the output depends on (graph order is topological)
    need_ds = {output}
    live = []
    for i in reversed(range(len(nodes))):
        if nodes[i].out in need_ds:
            live.append(i)
            need_ds.update(nodes[i].ins)
    live.reverse()

    def linked(nd, slot):
        return in_rows(nd, slot, 0, 1, shapes[nd.ins[slot]][2]) is not None

    # components of row-linked data (union-find over DS ids, smallest id is the root)
    parent = list(range(len(shapes)))

    def find(x):
        while parent[x] != x:
            x = parent[x]
        return x

    for i in live:
        nd = nodes[i]
        for slot, d in enumerate(nd.ins):
            if linked(nd, slot):
                ra, rb = find(d), find(nd.out)
                if ra != rb:
                    parent[max(ra, rb)] = min(ra, rb)
    comps = []                     # in order of their first operator
    comp_nodes = {}
    for i in live:
        c = find(nodes[i].out)
        if c not in comp_nodes:
            comps.append(c)
            comp_nodes[c] = []
        comp_nodes[c].append(i)

    def sinks(c):
        consumed = {d for i in comp_nodes[c] for slot, d in enumerate(nodes[i].ins) if linked(nodes[i], slot)}
        outs = [nodes[i].out for i in comp_nodes[c]]
        return [d for d in dict.fromkeys(outs) if d not in consumed or d == output]

    def bands_for(c, k):
        """Piece i of every DS of component c: sinks cut into k equal row bands, every other
        DS the hull of what its consumers' piece i needs (leaves to root)."""
        band = {d: [(i * shapes[d][2] // k, (i + 1) * shapes[d][2] // k) for i in range(k)] for d in sinks(c)}
        for i in reversed(comp_nodes[c]):
            nd = nodes[i]
            for slot, d in enumerate(nd.ins):
                if not linked(nd, slot):
                    continue
                h = shapes[d][2]
                want = []
                for a, b in band[nd.out]:
                    ra, rb = in_rows(nd, slot, a, b, h)
                    want.append((max(0, ra), min(h, rb)))
                if d in band:
                    band[d] = [(min(p[0], q[0]), max(p[1], q[1])) for p, q in zip(band[d], want)]
                else:
                    band[d] = want
        return band

    k_of = {}
    band_of = {}

    def bands(d, cur=None, cur_k=1, cur_band=None):
        c = find(d)
        if c == cur and cur_k > 1:
            return cur_band[d]
        if k_of.get(c, 1) > 1:
            return band_of[c][d]
        return [(0, shapes[d][2])]

    def op_pieces(nd, p, k, c, band):
        """DS pieces (d, r0, r1) that piece p of operator nd reads and writes."""
        keys = []
        for slot, d in enumerate(nd.ins):
            if linked(nd, slot) and k > 1:
                keys.append((d, *band[d][p]))
            else:
                keys.extend((d, *r) for r in bands(d, c, k, band))
        keys.append((nd.out, *(band[nd.out][p] if k > 1 else (0, shapes[nd.out][2]))))
        return keys

    def req(keys):
        return sum(nbytes(d, b - a) for d, a, b in dict.fromkeys(keys))

    for c in comps:
        cn = comp_nodes[c]
        k0 = max(-(-req(op_pieces(nodes[i], 0, 1, c, None)) // capacity) for i in cn)   # step 1-2
        if k0 <= 1:
            k_of[c] = 1
            continue
        kmax = min(shapes[d][2] for d in sinks(c))
        k = k0 if force_k is None else force_k
        while force_k is None:                                                             # step 3
            if k > kmax:
                raise ValueError("infeasible: an operator does not fit even split into single rows")
            band = bands_for(c, k)
            if all(req(op_pieces(nodes[i], p, k, c, band)) <= capacity for i in cn for p in range(k)):
                break
            k += 1
        k_of[c] = k
        band_of[c] = bands_for(c, k)
    # the split graph for the scheduler: DS pieces by first appearance, piece operators in
    # (node, piece) order
    g = Graph()
    pieces = []
    pid = {}
    op_piece = []
    for i in live:
        nd = nodes[i]
        c = find(nd.out)
        k = k_of[c]
        for p in range(k):
            ids = []
            for d, a, b in op_pieces(nd, p, k, c, band_of.get(c)):
                if (d, a, b) not in pid:
                    pid[(d, a, b)] = g.add_ds(f"d{d}[{a}:{b}]", nbytes(d, b - a), kinds[d])
                    pieces.append([d, a, b])
                ids.append(pid[(d, a, b)])
            g.add_op(f"n{i}.{p}", ids[:-1], ids[-1:])
            op_piece.append([i, p])
    if force_k is not None:
        return {"graph": g, "pieces": pieces, "op_piece": op_piece}
    order = dfs_order(g)
    tr = []
    moved = simulate_transfers(g, order, capacity, tr)
    return {"graph": g, "pieces": pieces, "op_piece": op_piece, "order": order, "trace": tr,
            "moved": moved, "k": {i: k_of[find(nodes[i].out)] for i in live}}


def per_op_plan(shapes, kinds, nodes: list[SNode], output: int, capacity: int):
    """TG_PER_OP at a scheduling capacity M: split (R19) and schedule within
    M, plus the transfer trace with frees. How M is derived from the budget (PAPER.md:409:
    "set to a value less than the actual amount of GPU memory ... to account for
    fragmentation") and where buffers sit in the arena are the library's static-layout design:
    M is an INPUT here; tests/test_split_plan.py checks the layout by properties."""
    r = split_plan(shapes, kinds, nodes, output, capacity)
    tr = []
    simulate_transfers(r["graph"], r["order"], capacity, tr, frees=True)
    r["capacity"] = capacity
    r["trace_full"] = tr
    return r


# ============================================================================ chunk rule
F32 = 4


def _edge_rows(H: int, ks: int, r0: int, r1: int) -> dict:
    rg = back_propagate_rows([("same", ks)], r0, r1, H_in=H)
    return {"in": list(rg[0]), "out": list(rg[1])}


def _cnn_rows(r0: int, r1: int) -> dict:
    rg = back_propagate_rows(CNN_LAYERS, r0, r1)
    # levels: 0 in, 1 C1, 2 T1, 3 S2, 4 T2, 5 C3, 6 T3, 7 S4, 8 T4, 9 C5, 10 T5, 11 C6
    return {"in": list(rg[0]), "c1": list(rg[1]), "t2": list(rg[4]), "c3": list(rg[5]),
            "t4": list(rg[8]), "out": list(rg[11])}


def _span(r) -> int:
    return r[1] - r[0]


def template_params(template: str, H: int, W: int, *, ks: int = 16, n5: int = 20, bias: str = "plane",
                    nf: int = 2):
    """Parameter floats of a template instance and which of them are bias planes: the edge
    template's nf kernels of ks x ks (the 2 x 256 kernel floats of Table 1 at nf = 2,
    PAPER.md:743); the CNN's K1 B1 P2 K3 B3 P4 K5 B5 K6 B6, biases one plane per
    output map (Fig. 7) or one scalar per map."""
    if template == "edge":
        return [ks * ks] * nf, [False] * nf
    (h1, w1), _, (h3, w3), _, (h5, w5) = cnn_dims(H, W)
    bs = [8 * h1 * w1, 20 * h3 * w3, n5 * h5 * w5, 9 * h5 * w5] if bias == "plane" else [8, 20, n5, 9]
    params = [8 * 25, bs[0], 8 * 4, 20 * 8 * 25, bs[1], 20 * 4, n5 * 20 * 25, bs[2], 9 * n5, bs[3]]
    return params, [False, True, False, False, True, False, False, True, False, True]


def fused_chunks(template: str, n: int, H: int, W: int, split: str, B: int, R: int, *, ks: int = 16,
                 n5: int = 20, bias: str = "none", rank: int = 0, world: int = 1, device_io: bool = False,
                 nf: int = 2, combine: str = "max") -> dict:
    """What a fused plan moves and computes, given its chunk size -- restated from the paper:

      * chunks (R12): whole images, B per chunk (split 'batch'), or per image output
        row bands [i*R, min((i+1)*R, h_out)) (split 'rows': split the image, never the kernel,
        PAPER.md:367, :371), image-major;
      * the rows every chunk needs at every level, by back-propagation from its output rows
        "from the leaves to the root" (back_propagate_rows);
      * the shard of rank g of G: chunks [floor(C g / G), floor(C (g+1) / G));
      * host->device bytes: the parameter floats (never split; bias planes that
        travel with the chunks -- bias 'streamed' -- excluded) and per chunk its input rows, plus
        in 'streamed' mode the bias rows of C1, C3, C5 and C6 it needs; device->host bytes: its
        output rows (the template output);
      * Table 1 accounting at Fig. 7 granularity.

    How large B or R is -- the device-memory layout of a chunk slot -- is the library's design
    decision, not the paper's: it is an INPUT here, and tests/test_plan_parity.py checks it by
    properties (fits the budget, maximal, every buffer present)."""
    f = F32
    if n <= 0 or H <= 0 or W <= 0:
        raise ValueError("empty input")
    if template == "edge":
        h_out, w_out, planes_out = H, W, 1
        rows = lambda r0, r1: _edge_rows(H, ks, r0, r1)          # noqa: E731
        pbias = "plane"
    elif template == "cnn":
        (h1, w1), (h2, w2), (h3, w3), (h4, w4), (h5, w5) = cnn_dims(H, W)
        if h5 <= 0 or w5 <= 0:
            raise ValueError("image too small for the CNN")
        h_out, w_out, planes_out = h5, w5, 9
        rows = _cnn_rows
        pbias = "scalar" if bias == "scalar" else "plane"
    else:
        raise ValueError(template)
    params, is_bias = template_params(template, H, W, ks=ks, n5=n5, bias=pbias, nf=nf)
    streamed = bias == "streamed"

    chunks = []
    if split == "batch":
        for b0 in range(0, n, B):
            chunks.append({"img": b0, "nimg": min(B, n - b0), **rows(0, h_out)})
    elif split == "rows":
        for b0 in range(n):
            for r0 in range(0, h_out, R):
                chunks.append({"img": b0, "nimg": 1, **rows(r0, min(h_out, r0 + R))})
    else:
        raise ValueError(split)
    C = len(chunks)
    c0, c1 = (C * rank) // world, (C * (rank + 1)) // world
    mine = chunks[c0:c1]

    h2d_param = h2d_chunk = d2h = 0
    if not device_io:
        h2d_param = sum(p * f for p, b in zip(params, is_bias) if not (streamed and b))
        for ch in mine:
            h2d_chunk += ch["nimg"] * _span(ch["in"]) * W * f
            if streamed:
                h2d_chunk += 8 * _span(ch["c1"]) * w1 * f + 20 * _span(ch["c3"]) * w3 * f
                h2d_chunk += (n5 + 9) * _span(ch["out"]) * w5 * f
            d2h += ch["nimg"] * planes_out * _span(ch["out"]) * w_out * f

    if template == "edge":
        g = edge_graph_general(H, W, ks, nf, combine)
    else:
        g = cnn_graph_fig7(H, W, n5)
    param_floats = sum(params)
    per_img_floats = sum(d.size for d in g.ds if d.kind != "param")
    out_floats = sum(d.size for d in g.ds if d.kind == "output")
    return {
        "split": split, "B": B, "R": R, "bias": bias, "n_chunks": C, "chunks": chunks,
        "shard": [rank, world, c0, c1],
        "h2d_param_bytes": h2d_param, "h2d_chunk_bytes": h2d_chunk, "d2h_bytes": d2h,
        "io_lower_bound_bytes": (n * (H * W + out_floats) + param_floats) * f,
        "io_lower_bound_data_bytes": n * (H * W + out_floats) * f,
        "total_temp_bytes": (n * per_img_floats + param_floats) * f,
        "n_ops_fig7": len(g.ops), "n_ds_fig7": len(g.ds),
    }
