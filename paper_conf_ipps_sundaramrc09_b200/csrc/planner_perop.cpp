// planner_perop.cpp -- the paper-faithful plans (pure host code):
//   TG_PER_OP   every operator is its own offload unit ("In our implementation,
//               the individual operators are taken to be the offload units"), operators in
//               depth-first order, transfers by "latest time of use" with eager
//               deletion, within "Total GPU Memory" set below the arena to
//               leave room for fragmentation (7/8 of the budget here);
//   TG_BASELINE "For each operator, transfer input data to the GPU, perform the operation and
//               copy the results back to the CPU immediately. There is no persistent storage in
//               GPU memory."
// Operators run whole (no splitting in these modes: an operator that does not fit is
// TG_E_INFEASIBLE); the fused mode (planner.cpp) is the one that splits.
#include <algorithm>
#include <sstream>

#include "kernels/kernels.h"
#include "tg_internal.h"

namespace tg {

static uint64_t a256(uint64_t x) { return (x + 255) / 256 * 256; }

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
    std::vector<char> need_node(g.nodes.size(), 0), need_ds(g.ds.size(), 0);
    need_ds[out] = 1;
    for (int n = (int)g.nodes.size() - 1; n >= 0; --n) {
        if (!need_ds[g.nodes[n].out]) continue;
        need_node[n] = 1;
        for (int x : g.nodes[n].ins) need_ds[x] = 1;
        if (g.nodes[n].bias >= 0) need_ds[g.nodes[n].bias] = 1;
    }
    for (size_t i = 0; i < g.ds.size(); ++i)
        if (need_ds[i] && g.ds[i].kind == DsKind::Input && g.ds[i].src_loc != Loc::Host)
            return fail(TG_E_UNSUPPORTED, "plan: TG_PER_OP / TG_BASELINE execute host-resident graphs (use tg_input)");
    // abstract schedule graph: DS in order of first appearance, nodes in graph order
    tg_sched s;
    std::vector<int> sid(g.ds.size(), -1);
    auto ds_id = [&](int gid) {
        if (sid[gid] < 0) {
            sid[gid] = (int)s.ds.size();
            const Ds& d = g.ds[gid];
            int32_t kind = d.kind == DsKind::Input ? TG_DS_INPUT : d.kind == DsKind::Param ? TG_DS_PARAM : TG_DS_TEMP;
            if (gid == out) kind = TG_DS_OUTPUT;
            s.ds.push_back({(uint64_t)d.numel() * 4, kind});
            p.po_ds.push_back(gid);
        }
        return sid[gid];
    };
    for (int n = 0; n < (int)g.nodes.size(); ++n) {
        if (!need_node[n]) continue;
        const Node& nd = g.nodes[n];
        tg_sched::O o;
        for (int x : nd.ins) o.ins.push_back(ds_id(x));
        if (nd.bias >= 0) o.ins.push_back(ds_id(nd.bias));
        o.outs.push_back(ds_id(nd.out));
        if (nd.op == OpKind::Elem || nd.op == OpKind::Max)
            if ((int)nd.ins.size() > kGenMaxInputs)
                return fail(TG_E_UNSUPPORTED, "plan: elementwise/max nodes take at most 16 inputs");
        s.ops.push_back(o);
        p.po_ops.push_back(n);
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
    uint64_t total = 0, io = 0;
    for (auto& d : s.ds) {
        total += d.size;
        if (d.kind != TG_DS_TEMP) io += d.size;
    }
    p.total = total;
    p.io_lb = io;
    p.nops = (int64_t)s.ops.size();
    p.nds = (int64_t)s.ds.size();
    p.n_units = (int64_t)s.ops.size();
    uint64_t req_max = 0;
    for (auto& o : s.ops) {
        std::vector<int32_t> t = o.ins;
        t.insert(t.end(), o.outs.begin(), o.outs.end());
        std::sort(t.begin(), t.end());
        t.erase(std::unique(t.begin(), t.end()), t.end());
        uint64_t r = 0;
        for (int32_t j : t) r += s.ds[j].size;
        req_max = std::max(req_max, r);
    }
    p.po_capacity = g.budget ? g.budget - g.budget / 8 : total;
    if (req_max > p.po_capacity) {
        std::ostringstream m;
        m << "plan: an operator needs " << req_max << " B at once but the budget allows " << p.po_capacity
          << " B (7/8 of the budget, PAPER.md:409); TG_PER_OP does not split operators -- use TG_FUSED";
        return fail(TG_E_INFEASIBLE, m.str());
    }
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
    // byte counts and the peak residency (arena) from the trace
    uint64_t cur = 0, peak = 0;
    std::vector<char> on(s.ds.size(), 0);
    for (auto& e : p.po_trace) {
        if (e.first == 0) {
            h2d += s.ds[e.second].size;
            if (!on[e.second]) {
                on[e.second] = 1;
                cur += a256(s.ds[e.second].size);
            }
        } else if (e.first == 1) {
            for (int32_t j : s.ops[e.second].outs)
                if (!on[j]) {
                    on[j] = 1;
                    cur += a256(s.ds[j].size);
                }
        } else if (e.first == 2) {
            d2h += s.ds[e.second].size;
        } else if (on[e.second]) {
            on[e.second] = 0;
            cur -= a256(s.ds[e.second].size);
        }
        peak = std::max(peak, cur);
    }
    p.h2d = h2d;
    p.d2h = d2h;
    p.param_bytes = 0;
    p.slot_bytes = 0;
    // first-fit allocation inside the arena; capped: the 1/8 margin between the scheduling
    // capacity and the arena absorbs fragmentation; uncapped: room for every DS
    uint64_t all = 0;
    for (auto& d : s.ds) all += a256(d.size);
    (void)peak;
    p.arena_bytes = g.budget ? g.budget : all;
    p.split = "none";
    p.bias = "none";
    p.c0 = 0;
    p.c1 = 0;
    p.rank = g.rank;
    p.world = g.world;
    if (g.world != 1) return fail(TG_E_UNSUPPORTED, "plan: TG_PER_OP / TG_BASELINE run on one device");
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
    o << "], \"h2d_bytes\": " << p.h2d << ", \"d2h_bytes\": " << p.d2h << ", \"arena_bytes\": " << p.arena_bytes
      << ", \"io_lower_bound_bytes\": " << p.io_lb << ", \"total_temp_bytes\": " << p.total << ", \"n_ops\": " << p.nops
      << ", \"n_ds\": " << p.nds << "}";
    return o.str();
}

}  // namespace tg
