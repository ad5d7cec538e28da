// engine_perop.cu -- executor of the paper-faithful plans (TG_PER_OP, TG_BASELINE).
//
// Replays the plan's schedule (planner_perop.cpp) literally on one stream, the way the paper
// ran its plans (no copy/compute overlap): H2D copies of whole data
// structures, one generic kernel per operator (the "operator library", Fig. 4), D2H copies
// of evicted or final data, and eager frees. Device memory is one arena of plan.arena_bytes
// carved with a first-fit allocator; data structures evicted to the host live in staging
// buffers owned by the plan.
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
    std::map<uint64_t, uint64_t> free_list;   // offset -> size
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

uint64_t a256(uint64_t x) { return (x + 255) / 256 * 256; }

bool arena_alloc(tg_perop_exec& x, uint64_t bytes, uint64_t& out) {
    bytes = a256(std::max<uint64_t>(bytes, 1));
    for (auto it = x.free_list.begin(); it != x.free_list.end(); ++it)
        if (it->second >= bytes) {
            out = it->first;
            const uint64_t rest = it->second - bytes;
            const uint64_t noff = it->first + bytes;
            x.free_list.erase(it);
            if (rest) x.free_list[noff] = rest;
            return true;
        }
    return false;
}

void arena_free(tg_perop_exec& x, uint64_t off, uint64_t bytes) {
    bytes = a256(std::max<uint64_t>(bytes, 1));
    auto it = x.free_list.emplace(off, bytes).first;
    auto nx = std::next(it);  // coalesce with the next and previous blocks
    if (nx != x.free_list.end() && it->first + it->second == nx->first) {
        it->second += nx->second;
        x.free_list.erase(nx);
    }
    if (it != x.free_list.begin()) {
        auto pv = std::prev(it);
        if (pv->first + pv->second == it->first) {
            pv->second += it->second;
            x.free_list.erase(it);
        }
    }
}

tg_status launch_node(const Graph& g, const PlanCore& c, tg_perop_exec& x, int op) {
    const Node& nd = g.nodes[c.po_ops[op]];
    auto dptr = [&](int gid) -> float* {
        for (size_t k = 0; k < c.po_ds.size(); ++k)
            if (c.po_ds[k] == gid) return x.off[k] < 0 ? nullptr : (float*)(x.arena + x.off[k]);
        return nullptr;
    };
    const Ds& Y = g.ds[nd.out];
    float* y = dptr(nd.out);
    if (!y) return fail(TG_E_STATE, "per-op executor: output not resident");
    cudaError_t e = cudaSuccess;
    switch (nd.op) {
        case OpKind::Conv: {
            const Ds& X = g.ds[nd.ins[0]];
            const Ds& K = g.ds[nd.ins[1]];
            GenConvArgs a{};
            a.x = dptr(nd.ins[0]);
            a.k = dptr(nd.ins[1]);
            a.y = y;
            a.n = X.d[0];
            a.ci = X.d[1];
            a.h = X.d[2];
            a.w = X.d[3];
            a.co = K.d[0];
            a.kh = K.d[2];
            a.kw = K.d[3];
            a.ho = Y.d[2];
            a.wo = Y.d[3];
            a.pt = nd.pad == TG_SAME ? (int)(K.d[2] - 1) / 2 : 0;
            a.pl = nd.pad == TG_SAME ? (int)(K.d[3] - 1) / 2 : 0;
            a.bias_kind = 0;
            if (nd.bias >= 0) {
                a.bias = dptr(nd.bias);
                a.bias_kind = g.ds[nd.bias].numel() == K.d[0] ? 1 : 2;
            }
            if (!a.x || !a.k || (nd.bias >= 0 && !a.bias)) return fail(TG_E_STATE, "per-op executor: input not resident");
            e = launch_gen_conv(a, x.stream);
            break;
        }
        case OpKind::Sub: {
            const Ds& X = g.ds[nd.ins[0]];
            GenSubArgs a{};
            a.x = dptr(nd.ins[0]);
            a.p = dptr(nd.ins[1]);
            a.y = y;
            a.n = X.d[0];
            a.c = X.d[1];
            a.h = X.d[2];
            a.w = X.d[3];
            a.ho = Y.d[2];
            a.wo = Y.d[3];
            a.s = nd.s;
            if (!a.x || !a.p) return fail(TG_E_STATE, "per-op executor: input not resident");
            e = launch_gen_sub(a, x.stream);
            break;
        }
        default: {
            GenElemArgs a{};
            a.nx = (int)nd.ins.size();
            for (int i = 0; i < a.nx; ++i) {
                a.xs[i] = dptr(nd.ins[i]);
                if (!a.xs[i]) return fail(TG_E_STATE, "per-op executor: input not resident");
            }
            a.y = y;
            a.numel = Y.numel();
            a.op = nd.op == OpKind::Tanh ? 4 : nd.op == OpKind::Max ? 5 : nd.elem;
            a.a = nd.a;
            a.b = nd.b;
            e = launch_gen_elem(a, x.stream);
        }
    }
    if (e != cudaSuccess) return fail(TG_E_CUDA, std::string("generic kernel launch failed: ") + cudaGetErrorString(e));
    return TG_OK;
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
    x.free_list.clear();
    x.free_list[0] = std::max<uint64_t>(c.arena_bytes, 256) / 256 * 256;
    x.off.assign(c.po_ds.size(), -1);
    auto host_src = [&](int sd) -> const float* {
        const Ds& d = g.ds[c.po_ds[sd]];
        if (d.kind != DsKind::Temp) return d.src;
        return x.staging[sd].empty() ? nullptr : x.staging[sd].data();
    };
    for (auto& e : c.po_trace) {
        const int id = e.second;
        switch (e.first) {
            case 0: {  // H2D
                if (x.off[id] < 0) {
                    uint64_t o;
                    if (!arena_alloc(x, c.po_size[id], o)) return fail(TG_E_OOM, "per-op arena fragmented (H2D)");
                    x.off[id] = (int64_t)o;
                }
                const float* src = host_src(id);
                if (!src) return fail(TG_E_STATE, "per-op executor: no host copy to load");
                CK(cudaMemcpyAsync(x.arena + x.off[id], src, c.po_size[id], cudaMemcpyHostToDevice, x.stream));
                break;
            }
            case 1: {  // run
                for (int32_t j : c.po_outs[id])
                    if (x.off[j] < 0) {
                        uint64_t o;
                        if (!arena_alloc(x, c.po_size[j], o)) return fail(TG_E_OOM, "per-op arena fragmented (output)");
                        x.off[j] = (int64_t)o;
                    }
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
            case 2: {  // D2H
                const Ds& d = g.ds[c.po_ds[id]];
                float* dst;
                if (c.po_kind[id] == TG_DS_OUTPUT) {
                    dst = d.dst;
                } else {
                    x.staging[id].resize(c.po_size[id] / 4);
                    dst = x.staging[id].data();
                }
                CK(cudaMemcpyAsync(dst, x.arena + x.off[id], c.po_size[id], cudaMemcpyDeviceToHost, x.stream));
                if (c.po_kind[id] != TG_DS_OUTPUT) CK(cudaStreamSynchronize(x.stream));  // staging is pageable
                break;
            }
            default:  // free
                if (x.off[id] >= 0) {
                    arena_free(x, (uint64_t)x.off[id], c.po_size[id]);
                    x.off[id] = -1;
                }
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
