// sched.cpp -- offload and data-transfer scheduling of the paper's heuristic solution
// (Section 3.3.1) over an abstract operator graph:
//   1. a depth-first operator schedule: schedule the entire sub-tree of a
//      child before its siblings; a node whose inputs are not ready is skipped and reached
//      again from its last producer (children = consumers in insertion order, sources in
//      id order: DESIGN.md R11);
//   2. the "latest time of use" transfer schedule, read as NEXT use
//      (Belady; R10): inputs and outputs of the running operator must be on the
//      GPU; on shortage, the resident data structure used furthest in the future goes back
//      to the host (clean data is dropped for free; ties: clean first, then lowest id);
//      dead data is deleted eagerly; template outputs go to the host when evicted or at the
//      end. Initially everything is on the host (PB constraints (11), (12)).
// Used by the per-operator plans of the library and pinned against oracle/planner.py
// (tests/test_sched_parity.py: Fig. 3's 15 and 8 units, random DAGs bit-exact).
#include <algorithm>
#include <cstdint>
#include <limits>
#include <map>
#include <new>
#include <vector>

#include "tg_internal.h"

namespace tg {

std::vector<int32_t> sched_dfs(const tg_sched& s) {
    const int n = (int)s.ops.size();
    std::map<int32_t, int32_t> producer;
    for (int i = 0; i < n; ++i)
        for (int32_t j : s.ops[i].outs) producer[j] = i;
    std::vector<std::vector<int32_t>> preds(n), consumers(n);
    for (int c = 0; c < n; ++c)
        for (int32_t j : s.ops[c].ins) {
            auto it = producer.find(j);
            if (it == producer.end()) continue;
            const int p = it->second;
            if (std::find(preds[c].begin(), preds[c].end(), p) == preds[c].end()) preds[c].push_back(p);
            if (std::find(consumers[p].begin(), consumers[p].end(), c) == consumers[p].end()) consumers[p].push_back(c);
        }
    for (auto& v : consumers) std::sort(v.begin(), v.end());
    std::vector<char> seen(n, 0);
    std::vector<int32_t> order;
    auto ready = [&](int c) {
        for (int p : preds[c])
            if (!seen[p]) return false;
        return true;
    };
    // iterative DFS with an explicit stack of (node, next child index)
    for (int root = 0; root < n; ++root) {
        if (seen[root] || !ready(root)) continue;
        std::vector<std::pair<int, size_t>> st;
        seen[root] = 1;
        order.push_back(root);
        st.push_back({root, 0});
        while (!st.empty()) {
            auto& top = st.back();
            if (top.second >= consumers[top.first].size()) {
                st.pop_back();
                continue;
            }
            const int c = consumers[top.first][top.second++];
            if (!seen[c] && ready(c)) {
                seen[c] = 1;
                order.push_back(c);
                st.push_back({c, 0});
            }
        }
    }
    return order;
}

// Returns the transfer volume; trace entries are (kind, id): 0 = H2D of DS id, 1 = run op id,
// 2 = D2H of DS id. Returns UINT64_MAX if an operator does not fit at all.
uint64_t sched_transfers(const tg_sched& s, const std::vector<int32_t>& order, uint64_t capacity,
                         std::vector<std::pair<int32_t, int32_t>>* trace, bool frees) {
    const size_t nds = s.ds.size();
    std::vector<std::vector<size_t>> uses(nds);
    for (size_t t = 0; t < order.size(); ++t) {
        const auto& op = s.ops[order[t]];
        std::vector<int32_t> touched = op.ins;
        touched.insert(touched.end(), op.outs.begin(), op.outs.end());
        std::sort(touched.begin(), touched.end());
        touched.erase(std::unique(touched.begin(), touched.end()), touched.end());
        for (int32_t j : touched) uses[j].push_back(t);
    }
    const size_t INF = std::numeric_limits<size_t>::max();
    auto next_use = [&](int32_t j, size_t t) {
        for (size_t u : uses[j])
            if (u > t) return u;
        return INF;
    };
    auto is_output = [&](int32_t j) { return s.ds[j].kind == TG_DS_OUTPUT; };
    std::vector<int8_t> on_gpu(nds, -1);  // -1 absent, 0 clean, 1 dirty
    std::vector<char> host_valid(nds, 0);
    for (size_t j = 0; j < nds; ++j) host_valid[j] = s.ds[j].kind == TG_DS_INPUT || s.ds[j].kind == TG_DS_PARAM;
    uint64_t used = 0, moved = 0;
    for (size_t t = 0; t < order.size(); ++t) {
        const auto& op = s.ops[order[t]];
        std::vector<int32_t> need;  // inputs then outputs, first occurrence order
        for (int32_t j : op.ins)
            if (std::find(need.begin(), need.end(), j) == need.end()) need.push_back(j);
        for (int32_t j : op.outs)
            if (std::find(need.begin(), need.end(), j) == need.end()) need.push_back(j);
        for (int32_t j : need) {
            if (on_gpu[j] >= 0) continue;
            const uint64_t sz = s.ds[j].size;
            while (used + sz > capacity) {
                int32_t victim = -1;
                size_t vnext = 0;
                int vdirty = 0;
                for (size_t k = 0; k < nds; ++k) {
                    if (on_gpu[k] < 0 || std::find(need.begin(), need.end(), (int32_t)k) != need.end()) continue;
                    const size_t nu = next_use((int32_t)k, t);
                    const int dirty = on_gpu[k];
                    // furthest next use; ties: clean before dirty, then lowest id
                    if (victim < 0 || nu > vnext || (nu == vnext && dirty < vdirty)) {
                        victim = (int32_t)k;
                        vnext = nu;
                        vdirty = dirty;
                    }
                }
                if (victim < 0) return UINT64_MAX;
                if (on_gpu[victim] == 1 && (vnext != INF || is_output(victim))) {
                    moved += s.ds[victim].size;  // write back dirty data that is still needed
                    host_valid[victim] = 1;
                    if (trace) trace->push_back({2, victim});
                }
                on_gpu[victim] = -1;
                used -= s.ds[victim].size;
                if (trace && frees) trace->push_back({3, victim});
            }
            const bool is_in = std::find(op.ins.begin(), op.ins.end(), j) != op.ins.end();
            if (is_in) {
                if (!host_valid[j]) return UINT64_MAX;  // reading data nobody produced
                moved += sz;
                on_gpu[j] = 0;
                if (trace) trace->push_back({0, j});
            } else {
                on_gpu[j] = 1;
                host_valid[j] = 0;
            }
            used += sz;
        }
        if (trace) trace->push_back({1, order[t]});
        for (size_t k = 0; k < nds; ++k)  // eager deletion of dead data
            if (on_gpu[k] >= 0 && next_use((int32_t)k, t) == INF && !is_output((int32_t)k)) {
                on_gpu[k] = -1;
                used -= s.ds[k].size;
                if (trace && frees) trace->push_back({3, (int32_t)k});
            }
    }
    for (size_t k = 0; k < nds; ++k)
        if (on_gpu[k] == 1 && is_output((int32_t)k)) {
            moved += s.ds[k].size;
            if (trace) trace->push_back({2, (int32_t)k});
        }
    return moved;
}

// Exhaustive minimum of the next-use transfer volume over every operator order that respects
// the data dependences (PB constraints (1)-(3) of Fig. 5): the exact
// counterpart of the DFS heuristic for small graphs (the paper solved the PB model
// with MiniSAT+, which is out of scope). Orders are enumerated depth-first with
// operators tried in id order, so the order returned is the lexicographically smallest optimal
// one. Returns false if more than max_orders orders exist.
bool sched_optimal(const tg_sched& s, uint64_t capacity, uint64_t max_orders, std::vector<int32_t>& best_order,
                   uint64_t& best, uint64_t& n_orders, uint64_t& n_best) {
    const int n = (int)s.ops.size();
    std::map<int32_t, int32_t> producer;
    for (int i = 0; i < n; ++i)
        for (int32_t j : s.ops[i].outs) producer[j] = i;
    std::vector<std::vector<int32_t>> preds(n);
    for (int c = 0; c < n; ++c)
        for (int32_t j : s.ops[c].ins) {
            auto it = producer.find(j);
            if (it != producer.end()) preds[c].push_back(it->second);
        }
    best = UINT64_MAX;
    n_orders = n_best = 0;
    std::vector<int32_t> prefix;
    std::vector<char> placed(n, 0);
    bool ok = true;
    // explicit-stack DFS over the choices at each depth
    std::vector<int> next(n + 1, 0);
    int depth = 0;
    while (depth >= 0 && ok) {
        if (depth == n) {
            if (++n_orders > max_orders) {
                ok = false;
                break;
            }
            const uint64_t v = sched_transfers(s, prefix, capacity, nullptr, false);
            if (v < best) {
                best = v;
                n_best = 1;
                best_order = prefix;
            } else if (v == best && v != UINT64_MAX) {
                ++n_best;
            }
            --depth;
            if (depth >= 0) {
                placed[prefix.back()] = 0;
                prefix.pop_back();
            }
            continue;
        }
        int i = next[depth];
        for (; i < n; ++i) {
            if (placed[i]) continue;
            bool ready = true;
            for (int p : preds[i])
                if (!placed[p]) {
                    ready = false;
                    break;
                }
            if (ready) break;
        }
        if (i >= n) {  // no more choices at this depth: backtrack
            next[depth] = 0;
            --depth;
            if (depth >= 0) {
                placed[prefix.back()] = 0;
                prefix.pop_back();
            }
            continue;
        }
        next[depth] = i + 1;
        placed[i] = 1;
        prefix.push_back(i);
        ++depth;
        next[depth] = 0;
    }
    return ok;
}

}  // namespace tg

using namespace tg;

extern "C" {

tg_status tg_sched_create(tg_sched** s) {
    if (!s) return fail(TG_E_ARG, "tg_sched_create: NULL out pointer");
    try {
        *s = new tg_sched();
    } catch (const std::bad_alloc&) {
        return fail(TG_E_OOM, "tg_sched_create: out of memory");
    }
    return TG_OK;
}

void tg_sched_destroy(tg_sched* s) { delete s; }

tg_status tg_sched_add_ds(tg_sched* s, uint64_t size, int32_t kind, int32_t* id) {
    if (!s || !id) return fail(TG_E_ARG, "tg_sched_add_ds: NULL argument");
    if (kind < TG_DS_INPUT || kind > TG_DS_OUTPUT) return fail(TG_E_ARG, "tg_sched_add_ds: bad kind");
    s->ds.push_back({size, kind});
    *id = (int32_t)s->ds.size() - 1;
    return TG_OK;
}

tg_status tg_sched_add_op(tg_sched* s, const int32_t* ins, int32_t nin, const int32_t* outs, int32_t nout,
                          int32_t* id) {
    if (!s || !id || (nin && !ins) || (nout && !outs) || nin < 0 || nout < 0)
        return fail(TG_E_ARG, "tg_sched_add_op: bad argument");
    tg_sched::O o;
    for (int i = 0; i < nin; ++i) {
        if (ins[i] < 0 || ins[i] >= (int32_t)s->ds.size()) return fail(TG_E_ARG, "tg_sched_add_op: unknown input");
        o.ins.push_back(ins[i]);
    }
    for (int i = 0; i < nout; ++i) {
        if (outs[i] < 0 || outs[i] >= (int32_t)s->ds.size()) return fail(TG_E_ARG, "tg_sched_add_op: unknown output");
        o.outs.push_back(outs[i]);
    }
    s->ops.push_back(std::move(o));
    *id = (int32_t)s->ops.size() - 1;
    return TG_OK;
}

tg_status tg_sched_dfs_order(const tg_sched* s, int32_t* order) {
    if (!s || (!order && !s->ops.empty())) return fail(TG_E_ARG, "tg_sched_dfs_order: NULL argument");
    std::vector<int32_t> o = sched_dfs(*s);
    if (o.size() != s->ops.size()) return fail(TG_E_ARG, "tg_sched_dfs_order: the graph has a cycle");
    std::copy(o.begin(), o.end(), order);
    return TG_OK;
}

tg_status tg_sched_transfers(const tg_sched* s, const int32_t* order, uint64_t capacity, uint64_t* moved,
                             int32_t* trace, int64_t trace_cap, int64_t* trace_len) {
    if (!s || !order || !moved) return fail(TG_E_ARG, "tg_sched_transfers: NULL argument");
    std::vector<int32_t> ord(order, order + s->ops.size());
    std::vector<char> placed(s->ops.size(), 0);
    for (int32_t i : ord) {
        if (i < 0 || i >= (int32_t)s->ops.size() || placed[i]) return fail(TG_E_ARG, "tg_sched_transfers: order is not a permutation");
        placed[i] = 1;
    }
    std::vector<std::pair<int32_t, int32_t>> tr;
    const uint64_t m = sched_transfers(*s, ord, capacity, &tr, false);
    if (m == UINT64_MAX)
        return fail(TG_E_INFEASIBLE, "tg_sched_transfers: an operator does not fit, or reads data not yet produced");
    *moved = m;
    if (trace_len) *trace_len = (int64_t)tr.size();
    if (trace) {
        if (trace_cap < (int64_t)tr.size()) return fail(TG_E_ARG, "tg_sched_transfers: trace buffer too small");
        for (size_t i = 0; i < tr.size(); ++i) {
            trace[2 * i] = tr[i].first;
            trace[2 * i + 1] = tr[i].second;
        }
    }
    return TG_OK;
}

tg_status tg_sched_optimal(const tg_sched* s, uint64_t capacity, uint64_t max_orders, int32_t* order,
                           uint64_t* moved, uint64_t* n_orders, uint64_t* n_optimal) {
    if (!s || !moved || (!order && !s->ops.empty())) return fail(TG_E_ARG, "tg_sched_optimal: NULL argument");
    std::vector<int32_t> best_order;
    uint64_t best = 0, no = 0, nb = 0;
    if (!sched_optimal(*s, capacity, max_orders, best_order, best, no, nb))
        return fail(TG_E_UNSUPPORTED, "tg_sched_optimal: more operator orders than max_orders");
    if (no == 0 && !s->ops.empty()) return fail(TG_E_ARG, "tg_sched_optimal: the graph has a cycle");
    if (best == UINT64_MAX)
        return fail(TG_E_INFEASIBLE, "tg_sched_optimal: no order fits the capacity");
    std::copy(best_order.begin(), best_order.end(), order);
    *moved = best;
    if (n_orders) *n_orders = no;
    if (n_optimal) *n_optimal = nb;
    return TG_OK;
}

}  // extern "C"
