// engine_perop.cu -- executor of the paper-faithful plans (TG_PER_OP, TG_BASELINE).
//
// Replays the plan's schedule (planner_perop.cpp) literally on one stream, the way the paper
// ran its plans (no copy/compute overlap): H2D copies of data-structure pieces
// (row bands of the host arrays), one generic kernel per operator piece (the
// "operator library", Fig. 4), D2H copies of evicted or final pieces, and eager frees. Device
// memory is one arena of plan.arena_bytes laid out statically by the planner (largest buffer first over
// the trace); pieces evicted to the host live in staging buffers owned by the plan.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <map>
#include <string>
#include <vector>

#include "kernels/kernels.h"
#include "tg_internal.h"

struct tg_perop_exec {
    int dev = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    char* arena = nullptr;
    bool own_arena = false;
    std::vector<std::vector<float>> staging;  // per sched DS: host copy of evicted temporaries
    std::vector<int64_t> off;                 // per sched DS: arena offset or -1
    bool profiling = false;
    bool ready = false;
    tg_timing timing{};
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> prof;
};

namespace tg {
namespace {

#define CK(call)                                                                                   \
    do {                                                                                           \
        cudaError_t e_ = (call);                                                                   \
        if (e_ != cudaSuccess) {                                                                   \
            char m_[384];                                                                          \
            std::snprintf(m_, sizeof m_, "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_),   \
                          __FILE__, __LINE__);                                                     \
            return fail(TG_E_CUDA, m_);                                                            \
        }                                                                                          \
    } while (0)

// The tg_oplib_op descriptor of sched op `op` (graph node piece) with the arena offsets
// `off` of its resident pieces (-1: not resident). Shared with the code generator.
}  // namespace

bool oplib_desc(const Graph& g, const PlanCore& c, int op, const std::vector<int64_t>& off, const char* arena,
                tg_oplib_op& d) {
    const Node& nd = g.nodes[c.po_ops[op]];
    d = tg_oplib_op{};
    // the operator's input slots in order (conv x, k[, bias]); each slot's pieces are the
    // consecutive entries of po_ins that belong to its DS
    std::vector<int> slots = nd.ins;
    if (nd.op == OpKind::Conv && nd.bias >= 0) slots.push_back(nd.bias);
    if (slots.size() > (size_t)TG_OPLIB_MAX_IN) return false;
    std::vector<std::vector<int32_t>> pieces(slots.size());
    const std::vector<int32_t>& ins = c.po_ins[op];
    size_t i = 0;
    for (size_t s = 0; s < slots.size(); ++s) {
        while (i < ins.size() && c.po_ds[ins[i]] == slots[s]) pieces[s].push_back(ins[i++]);
        if (pieces[s].empty())  // repeated operand (e.g. add(x, x)): same pieces again
            for (size_t t = 0; t < s; ++t)
                if (slots[t] == slots[s]) pieces[s] = pieces[t];
    }
    d.nin = (int32_t)slots.size();
    for (size_t s = 0; s < slots.size(); ++s) {
        if (pieces[s].empty() || pieces[s].size() > (size_t)TG_OPLIB_MAX_SEG) return false;
        for (int32_t id : pieces[s]) {
            if (off[id] < 0) return false;
            d.in[s].seg[d.in[s].nseg++] = tg_oplib_seg{(const float*)((uintptr_t)arena + (uint64_t)off[id]), c.po_r0[id], c.po_r1[id]};
        }
        for (int q = 0; q < 4; ++q) d.in_dims[s][q] = g.ds[slots[s]].d[q];
    }
    const int32_t yo = c.po_outs[op][0];
    if (off[yo] < 0) return false;
    d.y = (float*)((uintptr_t)arena + (uint64_t)off[yo]);
    for (int q = 0; q < 4; ++q) d.y_dims[q] = g.ds[nd.out].d[q];
    d.r0 = c.po_r0[yo];
    d.r1 = c.po_r1[yo];
    d.pad = nd.pad;
    d.s = nd.s;
    d.a = nd.a;
    d.b = nd.b;
    switch (nd.op) {
        case OpKind::Conv: d.kind = TG_OPLIB_CONV; break;
        case OpKind::Sub: d.kind = TG_OPLIB_SUB; break;
        case OpKind::Matmul: d.kind = TG_OPLIB_MATMUL; break;
        default:
            d.kind = TG_OPLIB_ELEM;
            d.elem = nd.op == OpKind::Tanh ? 4 : nd.op == OpKind::Max ? 5 : nd.elem;
    }
    return true;
}

namespace {

tg_status launch_node(const Graph& g, const PlanCore& c, tg_perop_exec& x, int op) {
    tg_oplib_op d;
    if (!oplib_desc(g, c, op, x.off, x.arena, d)) return fail(TG_E_STATE, "per-op executor: operand not resident");
    return oplib_run(d, x.stream);
}

// copy rows [r0, r1) of every [n][c] plane between a whole host DS and a piece buffer
cudaError_t copy_rows(void* dst, const void* src, const Ds& d, int64_t r0, int64_t r1, bool h2d, cudaStream_t s) {
    const size_t row = (size_t)d.d[3] * 4, planes = (size_t)(d.d[0] * d.d[1]);
    const size_t piece = (size_t)(r1 - r0) * row, whole = (size_t)d.d[2] * row;
    if (r0 == 0 && r1 == d.d[2])
        return cudaMemcpyAsync(dst, src, planes * whole, h2d ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToHost, s);
    if (h2d)
        return cudaMemcpy2DAsync(dst, piece, (const char*)src + r0 * row, whole, piece, planes, cudaMemcpyHostToDevice, s);
    return cudaMemcpy2DAsync((char*)dst + r0 * row, whole, src, piece, piece, planes, cudaMemcpyDeviceToHost, s);
}

}  // namespace

tg_status exec_run_per_op(tg_plan* p, bool blocking) {
    const Graph& g = p->graph->g;
    const PlanCore& c = p->core;
    if (!p->perop) p->perop = new tg_perop_exec();
    if (!p->perop->ready) {
        tg_perop_exec& x = *p->perop;
        CK(cudaGetDevice(&x.dev));
        if (!g.devices.empty()) x.dev = g.devices[0];
        CK(cudaSetDevice(x.dev));
        void* s = (g.has_rt && g.rt.stream) ? g.rt.stream(x.dev, 1, g.rt.ctx) : nullptr;
        if (s) {
            x.stream = (cudaStream_t)s;
        } else {
            CK(cudaStreamCreateWithFlags(&x.stream, cudaStreamNonBlocking));
            x.own_stream = true;
        }
        const size_t bytes = std::max<uint64_t>(c.arena_bytes, 256);
        if (g.has_rt && g.rt.alloc) {
            x.arena = (char*)g.rt.alloc(bytes, x.dev, g.rt.ctx);
            if (!x.arena) return fail(TG_E_OOM, "runtime alloc of the device arena failed");
        } else {
            if (cudaMalloc((void**)&x.arena, bytes) != cudaSuccess) {
                cudaGetLastError();
                return fail(TG_E_OOM, "cudaMalloc of the device arena failed");
            }
            x.own_arena = true;
        }
        x.staging.resize(c.po_ds.size());
        x.ready = true;
    }
    tg_perop_exec& x = *p->perop;
    CK(cudaSetDevice(x.dev));
    x.off.assign(c.po_ds.size(), -1);
    for (size_t t = 0; t < c.po_trace.size(); ++t) {
        const auto& e = c.po_trace[t];
        const int id = e.second;
        const uint64_t off = c.po_trace_off[t];  // static arena layout (planner_perop.cpp)
        switch (e.first) {
            case 0: {  // H2D of a piece: rows [r0, r1) of its DS
                x.off[id] = (int64_t)off;
                const Ds& d = g.ds[c.po_ds[id]];
                if (d.kind != DsKind::Temp) {
                    CK(copy_rows(x.arena + off, d.src, d, c.po_r0[id], c.po_r1[id], true, x.stream));
                } else {
                    if (x.staging[id].empty()) return fail(TG_E_STATE, "per-op executor: no host copy to load");
                    CK(cudaMemcpyAsync(x.arena + off, x.staging[id].data(), c.po_size[id], cudaMemcpyHostToDevice,
                                       x.stream));
                }
                break;
            }
            case 1: {  // run
                x.off[c.po_outs[id][0]] = (int64_t)off;
                cudaEvent_t a = nullptr, b = nullptr;
                if (x.profiling) {
                    cudaEventCreate(&a);
                    cudaEventCreate(&b);
                    cudaEventRecord(a, x.stream);
                }
                tg_status st = launch_node(g, c, x, id);
                if (st != TG_OK) return st;
                if (x.profiling) {
                    cudaEventRecord(b, x.stream);
                    x.prof.push_back({a, b});
                }
                ++p->launches;
                break;
            }
            case 2: {  // D2H: outputs into their rows of the host buffer, temporaries to staging
                const Ds& d = g.ds[c.po_ds[id]];
                if (c.po_kind[id] == TG_DS_OUTPUT) {
                    CK(copy_rows(d.dst, x.arena + x.off[id], d, c.po_r0[id], c.po_r1[id], false, x.stream));
                } else {
                    x.staging[id].resize(c.po_size[id] / 4);
                    CK(cudaMemcpyAsync(x.staging[id].data(), x.arena + x.off[id], c.po_size[id],
                                       cudaMemcpyDeviceToHost, x.stream));
                    CK(cudaStreamSynchronize(x.stream));  // staging is pageable
                }
                break;
            }
            default:  // free
                x.off[id] = -1;
        }
    }
    if (blocking) CK(cudaStreamSynchronize(x.stream));
    ++x.timing.executions;
    return TG_OK;
}

tg_status exec_timing_per_op(tg_plan* p, tg_timing* out) {
    tg_perop_exec* x = p->perop;
    if (!x) {
        *out = tg_timing{};
        return TG_OK;
    }
    for (auto& pr : x->prof) {
        CK(cudaEventSynchronize(pr.second));
        float ms = 0.f;
        CK(cudaEventElapsedTime(&ms, pr.first, pr.second));
        x->timing.kernel_ms[0] += ms;
        x->timing.unit_launches[0] += 1;
        x->timing.launches += 1;
        cudaEventDestroy(pr.first);
        cudaEventDestroy(pr.second);
    }
    x->prof.clear();
    *out = x->timing;
    return TG_OK;
}

void exec_set_profiling_per_op(tg_plan* p, bool on) {
    if (!p->perop) p->perop = new tg_perop_exec();
    p->perop->profiling = on;
    if (on) p->perop->timing = tg_timing{};
}

void exec_destroy_per_op(tg_plan* p) {
    tg_perop_exec* x = p->perop;
    if (!x) return;
    const Graph& g = p->graph->g;
    if (x->stream) cudaStreamSynchronize(x->stream);
    for (auto& pr : x->prof) {
        cudaEventDestroy(pr.first);
        cudaEventDestroy(pr.second);
    }
    if (x->arena) {
        if (x->own_arena)
            cudaFree(x->arena);
        else if (g.has_rt && g.rt.free)
            g.rt.free(x->arena, x->dev, g.rt.ctx);
    }
    if (x->own_stream && x->stream) cudaStreamDestroy(x->stream);
    cudaGetLastError();
    delete x;
    p->perop = nullptr;
}

}  // namespace tg
