// planner_perop.cpp -- the paper-faithful plans (pure host code):
//   TG_PER_OP   the paper's method on any operator graph: operators whose memory requirement
//               exceeds the GPU memory are split into row pieces (DESIGN.md
//               R19), every operator piece is its own offload unit ("In our
//               implementation, the individual operators are taken to be the offload units"),
//               pieces in depth-first order, transfers by "latest time of use"
//               with eager deletion, within "Total GPU Memory" set below the
//               arena to leave room for fragmentation (7/8 of the budget here);
//   TG_BASELINE "For each operator, transfer input data to the GPU, perform the operation and
//               copy the results back to the CPU immediately. There is no persistent storage in
//               GPU memory." -- operators run whole (the paper's baseline failed
//               once an operator no longer fit): TG_E_INFEASIBLE.
// The splitting rule is restated in oracle/planner.py::split_plan; the two agree bit-exactly
// (tests/test_split_plan.py). Arena offsets are assigned statically (largest buffer first, lowest free offset) over the
// trace, so the executor and the generated code (codegen.cpp) replay the same layout.
#include <algorithm>
#include <map>
#include <sstream>
#include <tuple>

#include "kernels/kernels.h"
#include "tg_internal.h"

namespace tg {

static uint64_t a256(uint64_t x) { return (x + 255) / 256 * 256; }

namespace {

// ---------------------------------------------------------------------------- splitting
struct Band {
    int64_t a, b;
};

// Rows of input `slot` of node nd that its output rows [a, b) need; false = read whole.
// (a 5x5 VALID convolution's output rows [0, 48) need input rows [0, 52).)
bool in_rows(const Graph& g, const Node& nd, int slot, int64_t a, int64_t b, int64_t h_in, Band& r) {
    switch (nd.op) {
        case OpKind::Conv: {
            const int64_t kh = g.ds[nd.ins[1]].d[2];
            if (slot == 0) {
                if (nd.pad == TG_VALID) {
                    r = {a, b + kh - 1};
                } else {
                    r = {std::max<int64_t>(0, a - (kh - 1) / 2), std::min(h_in, b + kh / 2)};
                }
                return true;
            }
            if (slot == 2) {  // bias: a plane is row-linked, a scalar is read whole
                const Ds& B = g.ds[nd.bias];
                if (B.numel() != g.ds[nd.ins[1]].d[0]) {
                    r = {a, b};
                    return true;
                }
            }
            return false;  // the kernel is never split
        }
        case OpKind::Sub:
            if (slot != 0) return false;
            r = {(int64_t)nd.s * a, (int64_t)nd.s * b};
            return true;
        case OpKind::Matmul:  // rows of A and C; B whole
            if (slot != 0) return false;
            r = {a, b};
            return true;
        default:  // elementwise / tanh / max: row for row
            r = {a, b};
            return true;
    }
}

// the operator's inputs in the library's order: conv x, k[, bias]; others as built
std::vector<int> slots_of(const Node& nd) {
    std::vector<int> v = nd.ins;
    if (nd.op == OpKind::Conv && nd.bias >= 0) v.push_back(nd.bias);
    return v;
}

struct Splitter {
    const Graph& g;
    int output;
    uint64_t capacity;
    std::vector<int> live;              // needed nodes, graph order
    std::vector<int> parent;            // union-find over DS ids
    std::vector<int> comps;             // component roots in order of their first node
    std::map<int, std::vector<int>> comp_nodes;
    std::map<int, int> k_of;
    std::map<int, std::map<int, std::vector<Band>>> band_of;

    Splitter(const Graph& g_, int out, uint64_t cap) : g(g_), output(out), capacity(cap) {}

    uint64_t nbytes(int d, int64_t rows) const {
        const Ds& D = g.ds[d];
        return 4ull * (uint64_t)(D.d[0] * D.d[1] * rows * D.d[3]);
    }
    int find(int x) const {
        while (parent[x] != x) x = parent[x];
        return x;
    }
    bool linked(const Node& nd, int slot) const {
        Band r;
        const std::vector<int> sl = slots_of(nd);
        return in_rows(g, nd, slot, 0, 1, g.ds[sl[slot]].d[2], r);
    }

    void components() {
        std::vector<char> need_ds(g.ds.size(), 0);
        need_ds[output] = 1;
        for (int n = (int)g.nodes.size() - 1; n >= 0; --n) {
            if (!need_ds[g.nodes[n].out]) continue;
            live.push_back(n);
            for (int x : slots_of(g.nodes[n])) need_ds[x] = 1;
        }
        std::reverse(live.begin(), live.end());
        parent.resize(g.ds.size());
        for (size_t i = 0; i < parent.size(); ++i) parent[i] = (int)i;
        for (int n : live) {
            const Node& nd = g.nodes[n];
            const std::vector<int> sl = slots_of(nd);
            for (int s = 0; s < (int)sl.size(); ++s)
                if (linked(nd, s)) {
                    const int ra = find(sl[s]), rb = find(nd.out);
                    if (ra != rb) parent[std::max(ra, rb)] = std::min(ra, rb);
                }
        }
        for (int n : live) {
            const int c = find(g.nodes[n].out);
            if (!comp_nodes.count(c)) comps.push_back(c);
            comp_nodes[c].push_back(n);
        }
    }

    std::vector<int> sinks(int c) const {
        std::vector<char> consumed(g.ds.size(), 0);
        for (int n : comp_nodes.at(c)) {
            const Node& nd = g.nodes[n];
            const std::vector<int> sl = slots_of(nd);
            for (int s = 0; s < (int)sl.size(); ++s)
                if (linked(nd, s)) consumed[sl[s]] = 1;
        }
        std::vector<int> out;
        for (int n : comp_nodes.at(c)) {
            const int d = g.nodes[n].out;
            if ((!consumed[d] || d == output) && std::find(out.begin(), out.end(), d) == out.end()) out.push_back(d);
        }
        return out;
    }

    // piece i of every DS of component c: sinks in k equal bands, the rest back-propagated
    // from their consumers' piece i (hull), leaves to root
    std::map<int, std::vector<Band>> bands_for(int c, int k) const {
        std::map<int, std::vector<Band>> band;
        for (int d : sinks(c)) {
            const int64_t h = g.ds[d].d[2];
            std::vector<Band> v;
            for (int i = 0; i < k; ++i) v.push_back({i * h / k, (i + 1) * h / k});
            band[d] = v;
        }
        const std::vector<int>& cn = comp_nodes.at(c);
        for (auto it = cn.rbegin(); it != cn.rend(); ++it) {
            const Node& nd = g.nodes[*it];
            const std::vector<int> sl = slots_of(nd);
            for (int s = 0; s < (int)sl.size(); ++s) {
                if (!linked(nd, s)) continue;
                const int d = sl[s];
                const int64_t h = g.ds[d].d[2];
                std::vector<Band> want;
                for (const Band& ob : band.at(nd.out)) {
                    Band r;
                    in_rows(g, nd, s, ob.a, ob.b, h, r);
                    want.push_back({std::max<int64_t>(0, r.a), std::min(h, r.b)});
                }
                auto f = band.find(d);
                if (f == band.end()) {
                    band[d] = want;
                } else {
                    for (int i = 0; i < k; ++i) {
                        f->second[i].a = std::min(f->second[i].a, want[i].a);
                        f->second[i].b = std::max(f->second[i].b, want[i].b);
                    }
                }
            }
        }
        return band;
    }

    std::vector<Band> bands(int d, int cur, int cur_k, const std::map<int, std::vector<Band>>* cur_band) const {
        const int c = find(d);
        if (c == cur && cur_k > 1) return cur_band->at(d);
        auto k = k_of.find(c);
        if (k != k_of.end() && k->second > 1) return band_of.at(c).at(d);
        return {Band{0, g.ds[d].d[2]}};
    }

    struct Key {
        int d;
        int64_t a, b;
        bool operator==(const Key& o) const { return d == o.d && a == o.a && b == o.b; }
    };

    // DS pieces that piece p of node n reads (in slot order) and writes (last)
    std::vector<Key> op_pieces(int n, int p, int k, int c, const std::map<int, std::vector<Band>>* band) const {
        const Node& nd = g.nodes[n];
        const std::vector<int> sl = slots_of(nd);
        std::vector<Key> keys;
        for (int s = 0; s < (int)sl.size(); ++s) {
            const int d = sl[s];
            if (linked(nd, s) && k > 1) {
                const Band& b = band->at(d)[p];
                keys.push_back({d, b.a, b.b});
            } else {
                for (const Band& b : bands(d, c, k, band)) keys.push_back({d, b.a, b.b});
            }
        }
        if (k > 1) {
            const Band& b = band->at(nd.out)[p];
            keys.push_back({nd.out, b.a, b.b});
        } else {
            keys.push_back({nd.out, 0, g.ds[nd.out].d[2]});
        }
        return keys;
    }

    uint64_t req(const std::vector<Key>& keys) const {
        uint64_t t = 0;
        for (size_t i = 0; i < keys.size(); ++i) {
            bool dup = false;
            for (size_t j = 0; j < i; ++j) dup = dup || keys[j] == keys[i];
            if (!dup) t += nbytes(keys[i].d, keys[i].b - keys[i].a);
        }
        return t;
    }

    tg_status run(bool allow_split) {
        components();
        for (int c : comps) {
            const std::vector<int>& cn = comp_nodes[c];
            uint64_t k0 = 1;  // step 1-2: k = ceil(req / M)
            for (int n : cn) k0 = std::max(k0, (req(op_pieces(n, 0, 1, c, nullptr)) + capacity - 1) / capacity);
            if (k0 <= 1) {
                k_of[c] = 1;
                continue;
            }
            if (!allow_split) {
                std::ostringstream m;
                m << "plan: an operator needs more than the " << capacity
                  << " B the budget allows (7/8 of the budget, PAPER.md:409); TG_BASELINE runs operators whole";
                return fail(TG_E_INFEASIBLE, m.str());
            }
            int64_t kmax = INT64_MAX;
            for (int d : sinks(c)) kmax = std::min(kmax, g.ds[d].d[2]);
            int64_t k = (int64_t)k0;
            std::map<int, std::vector<Band>> band;
            for (;; ++k) {  // step 3: split further until every piece fits
                if (k > kmax) {
                    std::ostringstream m;
                    m << "plan: an operator does not fit within " << capacity
                      << " B even when split into single output rows (PAPER.md:371)";
                    return fail(TG_E_INFEASIBLE, m.str());
                }
                band = bands_for(c, (int)k);
                bool ok = true;
                for (int n : cn)
                    for (int p = 0; p < k && ok; ++p) ok = req(op_pieces(n, p, (int)k, c, &band)) <= capacity;
                if (ok) break;
            }
            k_of[c] = (int)k;
            band_of[c] = band;
        }
        return TG_OK;
    }
};

}  // namespace

constexpr tg_status kLayoutFailed = 1;  // internal: retry with a lower capacity
static tg_status plan_at(const Graph& g, int32_t mode, int out, const std::vector<char>& need_ds, uint64_t cap,
                         PlanCore& p);

tg_status make_plan_per_op(const Graph& g, int32_t mode, PlanCore& p) {
    int out = -1, nout = 0;
    for (int i = 0; i < (int)g.ds.size(); ++i)
        if (g.ds[i].dst) {
            out = i;
            ++nout;
        }
    if (nout != 1) return fail(TG_E_STATE, "plan: bind exactly one template output with tg_output");
    if (g.ds[out].dst_loc != Loc::Host)
        return fail(TG_E_UNSUPPORTED, "plan: TG_PER_OP / TG_BASELINE execute host-resident graphs (use tg_output)");
    // nodes the output depends on (graph order is a topological order by construction)
    std::vector<char> need_ds(g.ds.size(), 0);
    need_ds[out] = 1;
    for (int n = (int)g.nodes.size() - 1; n >= 0; --n) {
        if (!need_ds[g.nodes[n].out]) continue;
        for (int x : slots_of(g.nodes[n])) need_ds[x] = 1;
        const Node& nd = g.nodes[n];
        if ((nd.op == OpKind::Elem || nd.op == OpKind::Max) && (int)nd.ins.size() > kGenMaxInputs)
            return fail(TG_E_UNSUPPORTED, "plan: elementwise/max nodes take at most 16 inputs");
    }
    uint64_t whole_total = 0;
    for (size_t i = 0; i < g.ds.size(); ++i) {
        if (!need_ds[i]) continue;
        if (g.ds[i].kind == DsKind::Input && g.ds[i].src_loc != Loc::Host)
            return fail(TG_E_UNSUPPORTED, "plan: TG_PER_OP / TG_BASELINE execute host-resident graphs (use tg_input)");
        whole_total += (uint64_t)g.ds[i].numel() * 4;
    }
    if (g.world != 1) return fail(TG_E_UNSUPPORTED, "plan: TG_PER_OP / TG_BASELINE run on one device");
    // "Total GPU Memory" below the arena to account for fragmentation: the
    // budget less 1/8, lowered by another 1/16 of the budget while the static
    // layout of the schedule does not fit the arena (restated in oracle per_op_plan)
    uint64_t cap = g.budget ? g.budget - g.budget / 8 : std::max<uint64_t>(whole_total, 1);
    for (;;) {
        PlanCore q = p;
        const tg_status st = plan_at(g, mode, out, need_ds, cap, q);
        if (st == TG_OK) {
            p = std::move(q);
            return TG_OK;
        }
        if (st != kLayoutFailed) return st;
        if (!g.budget || cap <= g.budget / 16) return fail(TG_E_INFEASIBLE, "plan: the arena is too fragmented for any schedule");
        cap -= g.budget / 16;
    }
}

static tg_status plan_at(const Graph& g, int32_t mode, int out, const std::vector<char>& need_ds, uint64_t cap,
                         PlanCore& p) {
    p.po_capacity = cap;
    // operator splitting (R19); TG_BASELINE never splits
    Splitter sp(g, out, p.po_capacity);
    if (tg_status st = sp.run(mode == TG_PER_OP); st != TG_OK) return st;
    // abstract schedule graph: DS pieces in order of first appearance, piece operators in
    // (node, piece) order
    tg_sched s;
    std::map<std::tuple<int, int64_t, int64_t>, int32_t> keys;  // (DS, r0, r1) -> sched DS id
    auto piece_id = [&](const Splitter::Key& kk) {
        const auto key = std::make_tuple(kk.d, kk.a, kk.b);
        auto it = keys.find(key);
        if (it != keys.end()) return it->second;
        const int32_t id = (int32_t)keys.size();
        keys.emplace(key, id);
        const Ds& d = g.ds[kk.d];
        int32_t kind = d.kind == DsKind::Input ? TG_DS_INPUT : d.kind == DsKind::Param ? TG_DS_PARAM : TG_DS_TEMP;
        if (kk.d == out) kind = TG_DS_OUTPUT;
        s.ds.push_back({sp.nbytes(kk.d, kk.b - kk.a), kind});
        p.po_ds.push_back(kk.d);
        p.po_r0.push_back(kk.a);
        p.po_r1.push_back(kk.b);
        return id;
    };
    p.po_k.assign(g.nodes.size(), 0);
    for (int n : sp.live) {
        const int c = sp.find(g.nodes[n].out);
        const int k = sp.k_of[c];
        p.po_k[n] = k;
        const auto* band = k > 1 ? &sp.band_of[c] : nullptr;
        for (int q = 0; q < k; ++q) {
            const std::vector<Splitter::Key> pk = sp.op_pieces(n, q, k, c, band);
            tg_sched::O o;
            for (size_t i = 0; i + 1 < pk.size(); ++i) o.ins.push_back(piece_id(pk[i]));
            o.outs.push_back(piece_id(pk.back()));
            s.ops.push_back(o);
            p.po_ops.push_back(n);
            p.po_piece.push_back(q);
        }
    }
    // a whole-read operand is looked up through at most kGenMaxSeg pieces
    for (size_t j = 0; j < s.ops.size(); ++j) {
        std::map<int, int> per_ds;
        for (int32_t i : s.ops[j].ins) ++per_ds[p.po_ds[i]];
        for (auto& kv : per_ds)
            if (kv.second > kGenMaxSeg)
                return fail(TG_E_UNSUPPORTED, "plan: an operand read whole spans more than 8 pieces of a split operator");
    }
    for (auto& d : s.ds) {
        p.po_size.push_back(d.size);
        p.po_kind.push_back(d.kind);
    }
    for (auto& o : s.ops) {
        p.po_ins.push_back(o.ins);
        p.po_outs.push_back(o.outs);
    }
    p.mode = mode;
    p.precision = TG_FP32;
    p.budget = g.budget;
    p.depth = 1;
    p.device_io = false;
    p.po_order = sched_dfs(s);
    uint64_t total = 0, io = 0;  // Table 1 accounting over the unsplit graph
    for (size_t i = 0; i < g.ds.size(); ++i) {
        if (!need_ds[i]) continue;
        const uint64_t b = (uint64_t)g.ds[i].numel() * 4;
        total += b;
        if (g.ds[i].kind != DsKind::Temp || (int)i == out) io += b;
    }
    p.total = total;
    p.io_lb = io;
    p.nops = (int64_t)s.ops.size();
    p.nds = (int64_t)s.ds.size();
    p.n_units = (int64_t)s.ops.size();
    p.po_trace.clear();
    uint64_t h2d = 0, d2h = 0;
    if (mode == TG_PER_OP) {
        if (sched_transfers(s, p.po_order, p.po_capacity, &p.po_trace, true) == UINT64_MAX)
            return fail(TG_E_INFEASIBLE, "plan: transfer scheduling failed");
    } else {  // TG_BASELINE: everything in, run, everything out, nothing kept
        for (int32_t op : p.po_order) {
            std::vector<int32_t> in = s.ops[op].ins;
            std::sort(in.begin(), in.end());
            in.erase(std::unique(in.begin(), in.end()), in.end());
            for (int32_t j : in) p.po_trace.push_back({0, j});
            p.po_trace.push_back({1, op});
            for (int32_t j : s.ops[op].outs) p.po_trace.push_back({2, j});
            for (int32_t j : in) p.po_trace.push_back({3, j});
            for (int32_t j : s.ops[op].outs) p.po_trace.push_back({3, j});
        }
    }
    for (auto& e : p.po_trace) {
        if (e.first == 0) h2d += s.ds[e.second].size;
        if (e.first == 2) d2h += s.ds[e.second].size;
    }
    p.h2d = h2d;
    p.d2h = d2h;
    p.param_bytes = 0;
    p.slot_bytes = 0;
    // static arena layout (restated in oracle arena_layout): every residency interval of a
    // piece (copy-in or production .. free or end) is a buffer of a256(size) bytes; buffers
    // are placed largest first (ties: earlier start, lower id), each at the lowest offset
    // clear of every placed buffer live at the same time. Capped: the arena is the budget and
    // the margin between the scheduling capacity and the arena absorbs fragmentation
    // (PAPER.md:409); uncapped: room for every DS piece.
    uint64_t all = 0;
    for (auto& d : s.ds) all += a256(std::max<uint64_t>(d.size, 1));
    p.arena_bytes = g.budget ? g.budget / 256 * 256 : all;
    struct Iv {
        size_t t0, t1;
        int32_t j;
        uint64_t off;
    };
    std::vector<Iv> iv;
    {
        std::map<int32_t, size_t> opened;
        for (size_t t = 0; t < p.po_trace.size(); ++t) {
            const auto& e = p.po_trace[t];
            if (e.first == 0 || e.first == 1) {
                const int32_t j = e.first == 0 ? e.second : s.ops[e.second].outs[0];
                if (!opened.count(j)) opened[j] = t;
            } else if (e.first == 3) {
                auto it = opened.find(e.second);
                if (it != opened.end()) {
                    iv.push_back({it->second, t, e.second, 0});
                    opened.erase(it);
                }
            }
        }
        // still resident at the end, in order of first opening (the oracle's dict order)
        std::vector<std::pair<size_t, int32_t>> rest;
        for (auto& kv : opened) rest.push_back({kv.second, kv.first});
        std::sort(rest.begin(), rest.end());
        for (auto& r : rest) iv.push_back({r.first, p.po_trace.size(), r.second, 0});
    }
    auto isz = [&](const Iv& v) { return a256(std::max<uint64_t>(s.ds[v.j].size, 1)); };
    std::vector<size_t> ord(iv.size());
    for (size_t i = 0; i < ord.size(); ++i) ord[i] = i;
    std::stable_sort(ord.begin(), ord.end(), [&](size_t x, size_t y) {
        if (isz(iv[x]) != isz(iv[y])) return isz(iv[x]) > isz(iv[y]);
        if (iv[x].t0 != iv[y].t0) return iv[x].t0 < iv[y].t0;
        return iv[x].j < iv[y].j;
    });
    std::vector<size_t> placed;
    for (size_t i : ord) {
        const uint64_t sz = isz(iv[i]);
        std::vector<std::pair<uint64_t, uint64_t>> conf;
        for (size_t q : placed)
            if (iv[q].t0 < iv[i].t1 && iv[i].t0 < iv[q].t1) conf.push_back({iv[q].off, iv[q].off + isz(iv[q])});
        std::sort(conf.begin(), conf.end());
        uint64_t cur = 0;
        for (auto& c : conf) {
            if (c.first >= cur + sz) break;
            cur = std::max(cur, c.second);
        }
        if (cur + sz > p.arena_bytes) return kLayoutFailed;
        iv[i].off = cur;
        placed.push_back(i);
    }
    {
        std::map<std::pair<int32_t, size_t>, uint64_t> off;
        for (auto& v : iv) off[{v.j, v.t0}] = v.off;
        std::map<int32_t, size_t> start;
        p.po_trace_off.clear();
        for (size_t t = 0; t < p.po_trace.size(); ++t) {
            const auto& e = p.po_trace[t];
            const int32_t j = e.first == 1 ? s.ops[e.second].outs[0] : e.second;
            if ((e.first == 0 || e.first == 1) && !start.count(j)) start[j] = t;
            p.po_trace_off.push_back(off.at({j, start.at(j)}));
            if (e.first == 3) start.erase(j);
        }
    }
    p.split = "none";
    for (int n : sp.live)
        if (p.po_k[n] > 1) p.split = "rows";
    p.bias = "none";
    p.c0 = 0;
    p.c1 = 0;
    p.rank = g.rank;
    p.world = g.world;
    return TG_OK;
}

std::string plan_json_per_op(const PlanCore& p) {
    std::ostringstream o;
    o << "{\"template\": \"graph\", \"mode\": \"" << (p.mode == TG_PER_OP ? "per_op" : "baseline") << "\", ";
    o << "\"budget\": " << p.budget << ", \"capacity\": " << p.po_capacity << ", ";
    o << "\"ds\": [";
    for (size_t i = 0; i < p.po_size.size(); ++i) o << (i ? ", " : "") << "[" << p.po_size[i] << ", " << p.po_kind[i] << "]";
    o << "], \"ops\": [";
    for (size_t i = 0; i < p.po_ins.size(); ++i) {
        o << (i ? ", " : "") << "[[";
        for (size_t k = 0; k < p.po_ins[i].size(); ++k) o << (k ? ", " : "") << p.po_ins[i][k];
        o << "], [";
        for (size_t k = 0; k < p.po_outs[i].size(); ++k) o << (k ? ", " : "") << p.po_outs[i][k];
        o << "]]";
    }
    o << "], \"order\": [";
    for (size_t i = 0; i < p.po_order.size(); ++i) o << (i ? ", " : "") << p.po_order[i];
    o << "], \"trace\": [";
    bool first = true;
    for (auto& e : p.po_trace) {
        if (e.first == 3) continue;  // frees are an executor detail
        o << (first ? "" : ", ") << "[" << e.first << ", " << e.second << "]";
        first = false;
    }
    o << "], \"trace_full\": [";
    for (size_t i = 0; i < p.po_trace.size(); ++i)
        o << (i ? ", " : "") << "[" << p.po_trace[i].first << ", " << p.po_trace[i].second << "]";
    o << "], \"trace_off\": [";
    for (size_t i = 0; i < p.po_trace_off.size(); ++i) o << (i ? ", " : "") << p.po_trace_off[i];
    o << "], \"pieces\": [";
    for (size_t i = 0; i < p.po_ds.size(); ++i)
        o << (i ? ", " : "") << "[" << p.po_ds[i] << ", " << p.po_r0[i] << ", " << p.po_r1[i] << "]";
    o << "], \"op_piece\": [";
    for (size_t i = 0; i < p.po_ops.size(); ++i) o << (i ? ", " : "") << "[" << p.po_ops[i] << ", " << p.po_piece[i] << "]";
    o << "], \"k\": {";
    bool fk = true;
    for (size_t n = 0; n < p.po_k.size(); ++n)
        if (p.po_k[n] > 0) {
            o << (fk ? "" : ", ") << "\"" << n << "\": " << p.po_k[n];
            fk = false;
        }
    o << "}, \"h2d_bytes\": " << p.h2d << ", \"d2h_bytes\": " << p.d2h << ", \"arena_bytes\": " << p.arena_bytes
      << ", \"io_lower_bound_bytes\": " << p.io_lb << ", \"total_temp_bytes\": " << p.total << ", \"n_ops\": " << p.nops
      << ", \"n_ds\": " << p.nds << "}";
    return o.str();
}

}  // namespace tg
