// engine.cu -- the run-time library ("a simple run-time library to
// orchestrate execution") that executes a plan on one or more B200s.
//
// Per device: ONE arena of exactly plan.arena_bytes (parameters + `depth` chunk slots;
// a static layout, so the "fragmentation" margin of PAPER.md:409 is not needed), three
// streams (H2D copy engine, compute, D2H copy engine) and per-slot events. The host thread
// enqueues, for every chunk k of its shard, in slot s = k % depth:
//     H2D   waits compute(k - depth)          copy input rows (+halo, +streamed bias rows)
//     comp  waits H2D(k), D2H(k - depth)      fused offload-unit kernels
//     D2H   waits comp(k)                     copy output rows into the caller's buffer
// so copies of chunk k+1 / k-1 overlap the kernels of chunk k (the overlap the paper's
// GPUs could not do). Everything is asynchronous; tg_execute synchronizes
// once at the end. Several devices: one host thread per device over contiguous chunk
// ranges; no collective.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstdio>
#include <cstring>
#include <string>
#include <thread>
#include <vector>

#include "kernels/kernels.h"
#include "tg_internal.h"

using namespace tg;

namespace {

struct ProfRec {
    int kind;  // 0 edge, 1 U1, 2 U2, 3 U3, 10 h2d, 11 d2h
    cudaEvent_t a, b;
    int64_t chunk = -1;
};

struct DevState {
    int dev = 0;
    cudaStream_t st[3] = {nullptr, nullptr, nullptr};
    bool own_st[3] = {false, false, false};
    char* arena = nullptr;
    bool own_arena = false;
    std::vector<cudaEvent_t> ev_h2d, ev_comp, ev_d2h;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr, ev_params = nullptr;
    cudaEvent_t ev_caller = nullptr, ev_done = nullptr;  // ordering against the caller's stream
    int64_t c0 = 0, c1 = 0;
    std::vector<ProfRec> prof;
    std::vector<cudaEvent_t> ev_pool;
    int64_t launches = 0;
    bool params_resident = false;  // parameters uploaded by an earlier execution
    int64_t seq = 0;               // chunks enqueued on this device over all executions (slot ring)
    cudaGraphExec_t graph = nullptr;  // captured execution (tg_plan_set_graph), replayed on S1
    bool after_graph = false;         // the last work on this device was a graph replay
    int64_t graph_launches = 0;       // kernel launches one replay performs
};

}  // namespace

struct tg_exec {
    std::vector<DevState> devs;
    bool ready = false;
    std::vector<void*> registered;
    uint64_t registered_bytes = 0;
    bool profiling = false;
    bool graph_mode = false;   // replay a captured execution (tg_plan_set_graph)
    bool prof_copies = false;  // also time every copy (perturbs the copy engines)
    tg_timing timing{};
    std::vector<tg_trace_rec> trace;  // timeline collected from the profiling events
    std::vector<uint16_t> k3tc, k5tc;  // host copies of the bf16 tensor-core B operands
    std::vector<uint16_t> k3h3, k5h3;  // host copies of the 3xFP16 B operands (TG_FP32_TC)
    float k3_scale = 1.f, k5_scale = 1.f;  // their power-of-two weight scales
    std::vector<float> b5q4;  // C5 bias planes channel-quad interleaved [n5/4][h5][w5][4] (b5_quads)
};

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

const Graph& graph_of(const tg_plan* p) { return p->graph->g; }

cudaEvent_t pool_event(DevState& d) {
    if (!d.ev_pool.empty()) {
        cudaEvent_t e = d.ev_pool.back();
        d.ev_pool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
    return e;
}

tg_status init_device(tg_plan* p, DevState& d) {
    const Graph& g = graph_of(p);
    const PlanCore& c = p->core;
    CK(cudaSetDevice(d.dev));
    for (int w = 0; w < 3; ++w) {
        void* s = (g.has_rt && g.rt.stream) ? g.rt.stream(d.dev, w, g.rt.ctx) : nullptr;
        if (s) {
            d.st[w] = (cudaStream_t)s;
        } else {
            CK(cudaStreamCreateWithFlags(&d.st[w], cudaStreamNonBlocking));
            d.own_st[w] = true;
        }
    }
    const size_t bytes = std::max<uint64_t>(c.arena_bytes, 256);
    if (g.has_rt && g.rt.alloc) {
        d.arena = (char*)g.rt.alloc(bytes, d.dev, g.rt.ctx);
        if (!d.arena) return fail(TG_E_OOM, "runtime alloc of the device arena failed");
    } else {
        cudaError_t e = cudaMalloc((void**)&d.arena, bytes);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(TG_E_OOM, std::string("cudaMalloc of the device arena failed: ") + cudaGetErrorString(e));
        }
        d.own_arena = true;
    }
    const unsigned flags = cudaEventDisableTiming;
    d.ev_h2d.resize(c.depth);
    d.ev_comp.resize(c.depth);
    d.ev_d2h.resize(c.depth);
    for (int s = 0; s < c.depth; ++s) {
        CK(cudaEventCreateWithFlags(&d.ev_h2d[s], flags));
        CK(cudaEventCreateWithFlags(&d.ev_comp[s], flags));
        CK(cudaEventCreateWithFlags(&d.ev_d2h[s], flags));
    }
    CK(cudaEventCreateWithFlags(&d.ev_fork, flags));
    CK(cudaEventCreateWithFlags(&d.ev_join, flags));
    CK(cudaEventCreateWithFlags(&d.ev_params, flags));
    CK(cudaEventCreateWithFlags(&d.ev_caller, flags));
    CK(cudaEventCreateWithFlags(&d.ev_done, flags));
    return TG_OK;
}

// Register caller-owned pageable host buffers once, so async copies run at full speed. Only the
// span this process's shard touches is registered (tg_set_shard: a process may hold just its
// part of a global input and output, the rest of the nominal [n][c][h][w] range unmapped).
tg_status register_host(tg_plan* p, tg_exec* x) {
    const Graph& g = graph_of(p);
    const PlanCore& c = p->core;
    if (c.device_io || c.c1 <= c.c0) return TG_OK;
    const Template& t = c.t;
    const Ds& X = g.ds[t.input];
    const Ds& Y = g.ds[t.output];
    // [lo, hi) in floats of the input rows and output rows of chunks [c0, c1)
    const int64_t HW = t.H * t.W;
    const int64_t out_img = t.kind == Tmpl::Edge ? HW : 9 * t.h[5] * t.w[5];
    const int64_t out_plane = t.kind == Tmpl::Edge ? HW : t.h[5] * t.w[5];
    const int64_t w_out = t.kind == Tmpl::Edge ? t.W : t.w[5];
    const int64_t planes = t.kind == Tmpl::Edge ? 1 : 9;
    int64_t xlo = INT64_MAX, xhi = 0, ylo = INT64_MAX, yhi = 0;
    for (int64_t i = c.c0; i < c.c1; ++i) {
        const Chunk& ch = c.chunks[i];
        xlo = std::min(xlo, ch.img * HW + ch.in.a * t.W);
        xhi = std::max(xhi, (ch.img + ch.nimg - 1) * HW + ch.in.b * t.W);
        ylo = std::min(ylo, ch.img * out_img + ch.out.a * w_out);
        yhi = std::max(yhi, (ch.img + ch.nimg - 1) * out_img + (planes - 1) * out_plane + ch.out.b * w_out);
    }
    std::vector<std::pair<void*, size_t>> bufs;
    bufs.push_back({(void*)(X.src + xlo), (size_t)(xhi - xlo) * 4});
    bufs.push_back({(void*)(Y.dst + ylo), (size_t)(yhi - ylo) * 4});
    for (int id : c.param_ds) bufs.push_back({(void*)g.ds[id].src, (size_t)g.ds[id].numel() * 4});
    for (auto& b : bufs) {
        if (b.second < (1u << 20)) continue;  // small: pageable copies are fine
        cudaPointerAttributes at{};
        if (cudaPointerGetAttributes(&at, b.first) == cudaSuccess && at.type == cudaMemoryTypeHost) continue;
        cudaGetLastError();
        cudaError_t e = cudaHostRegister(b.first, b.second, cudaHostRegisterDefault);
        if (e != cudaSuccess) {
            // no silent fallback to pageable copies (a several-fold cliff of the host link):
            // the caller pins the buffer itself or fixes the overlap
            cudaGetLastError();
            char m[320];
            std::snprintf(m, sizeof m,
                          "cudaHostRegister of a %zu-byte caller host buffer failed: %s (pass page-locked memory, "
                          "e.g. cudaHostAlloc / torch pin_memory, or non-overlapping buffers)",
                          b.second, cudaGetErrorString(e));
            return fail(TG_E_CUDA, m);
        }
        x->registered.push_back(b.first);
        x->registered_bytes += b.second;
    }
    return TG_OK;
}

// The tensor-core U3 kernels read the resident C5 bias planes channel-quad interleaved,
// [n5/4][h5][w5][4]: a warp's 32 consecutive positions load 4 channels each with one 128-bit load
// (512 contiguous bytes), 4 loads per 16 channels instead of 16 scalar ones, with the same L1
// wavefronts. Same bytes as the plane layout, so the plan (offsets, budget) is
// unchanged; it needs n5 % 4 == 0 (the paper's 20 and 120; other n5 keep the planes).
inline bool b5_quads(const PlanCore& c) {
    return c.t.kind == Tmpl::Cnn && c.bias == "resident" && c.param_off[7] != UINT64_MAX && c.t.n5 % 4 == 0 &&
           (c.precision == TG_BF16_TC || c.precision == TG_FP32_TC);
}

inline char* slot_base(const PlanCore& c, DevState& d, int s) {
    return d.arena + c.param_bytes + (uint64_t)s * c.slot_bytes;
}

// Copies of chunk inputs into slot s (H2D stream).
tg_status enqueue_h2d(const tg_plan* p, DevState& d, const Chunk& ch, int s) {
    const Graph& g = graph_of(p);
    const PlanCore& c = p->core;
    const Template& t = c.t;
    const Ds& X = g.ds[t.input];
    char* base = slot_base(c, d, s);
    const size_t W = (size_t)t.W;
    const size_t rows = (size_t)ch.in.n();
    // input rows [in.a, in.b) of nimg images: one strided copy
    CK(cudaMemcpy2DAsync(base + c.slot.in, rows * W * 4, X.src + (size_t)ch.img * t.H * W + (size_t)ch.in.a * W,
                         (size_t)t.H * W * 4, rows * W * 4, (size_t)ch.nimg, cudaMemcpyHostToDevice, d.st[0]));
    if (t.kind == Tmpl::Cnn && c.bias == "streamed") {
        // bias rows of every level this chunk's outputs depend on (planes strided)
        struct B {
            int prm;
            uint64_t off;
            int64_t planes, row0, rows, h, w;
        } bs[4] = {{1, c.slot.b1, 8, ch.c1.a, ch.c1.n(), t.h[1], t.w[1]},
                   {4, c.slot.b3, 20, ch.c3.a, ch.c3.n(), t.h[3], t.w[3]},
                   {7, c.slot.b5, t.n5, ch.out.a, ch.out.n(), t.h[5], t.w[5]},
                   {9, c.slot.b6, 9, ch.out.a, ch.out.n(), t.h[5], t.w[5]}};
        for (const B& b : bs) {
            const float* src = g.ds[t.prm[b.prm]].src + (size_t)b.row0 * b.w;
            CK(cudaMemcpy2DAsync(base + b.off, (size_t)b.rows * b.w * 4, src, (size_t)b.h * b.w * 4,
                                 (size_t)b.rows * b.w * 4, (size_t)b.planes, cudaMemcpyHostToDevice, d.st[0]));
        }
    }
    return TG_OK;
}

tg_status enqueue_d2h(const tg_plan* p, DevState& d, const Chunk& ch, int s) {
    const Graph& g = graph_of(p);
    const PlanCore& c = p->core;
    const Template& t = c.t;
    const Ds& Y = g.ds[t.output];
    char* base = slot_base(c, d, s);
    if (t.kind == Tmpl::Edge) {
        const size_t W = (size_t)t.W, rows = (size_t)ch.out.n();
        CK(cudaMemcpy2DAsync(Y.dst + (size_t)ch.img * t.H * W + (size_t)ch.out.a * W, (size_t)t.H * W * 4,
                             base + c.slot.out, rows * W * 4, rows * W * 4, (size_t)ch.nimg, cudaMemcpyDeviceToHost,
                             d.st[2]));
    } else {
        const size_t w5 = (size_t)t.w[5], h5 = (size_t)t.h[5], rows = (size_t)ch.out.n();
        CK(cudaMemcpy2DAsync(Y.dst + (size_t)ch.img * 9 * h5 * w5 + (size_t)ch.out.a * w5, h5 * w5 * 4,
                             base + c.slot.out, rows * w5 * 4, rows * w5 * 4, (size_t)ch.nimg * 9,
                             cudaMemcpyDeviceToHost, d.st[2]));
    }
    return TG_OK;
}

struct KernelTimer {
    tg_exec* x;
    DevState& d;
    int kind;
    int64_t chunk;
    cudaEvent_t a = nullptr, b = nullptr;
    KernelTimer(tg_exec* x_, DevState& d_, int kind_, int64_t chunk_, cudaStream_t s)
        : x(x_), d(d_), kind(kind_), chunk(chunk_) {
        if (x->profiling) {
            a = pool_event(d);
            b = pool_event(d);
            if (a) cudaEventRecord(a, s);
        }
    }
    void done(cudaStream_t s) {
        if (x->profiling && a && b) {
            cudaEventRecord(b, s);
            d.prof.push_back({kind, a, b, chunk});
        }
    }
};

tg_status launch_units(tg_plan* p, tg_exec* x, DevState& d, const Chunk& ch, int s) {
    const Graph& g = graph_of(p);
    const PlanCore& c = p->core;
    const Template& t = c.t;
    char* base = slot_base(c, d, s);
    cudaStream_t cs = d.st[1];
    const int64_t ci = &ch - c.chunks.data();  // chunk index (trace records)
    auto param = [&](int i) -> const float* {
        return c.param_off[i] == UINT64_MAX ? nullptr : (const float*)(d.arena + c.param_off[i]);
    };
    const Ds& X = g.ds[t.input];
    const Ds& Y = g.ds[t.output];
    if (t.kind == Tmpl::Edge) {
        EdgeArgs a{};
        if (c.device_io) {
            a.in = X.src + (size_t)ch.img * t.H * t.W;
            a.in_img_stride = t.H * t.W;
            a.in_row0 = 0;
            a.in_rows = t.H;
            a.out = Y.dst + (size_t)ch.img * t.H * t.W + (size_t)ch.out.a * t.W;
            a.out_img_stride = t.H * t.W;
        } else {
            a.in = (const float*)(base + c.slot.in);
            a.in_img_stride = ch.in.n() * t.W;
            a.in_row0 = ch.in.a;
            a.in_rows = ch.in.n();
            a.out = (float*)(base + c.slot.out);
            a.out_img_stride = ch.out.n() * t.W;
        }
        a.out_row0 = ch.out.a;
        a.out_rows = ch.out.n();
        a.H = t.H;
        a.W = t.W;
        a.nimg = ch.nimg;
        for (int f = 0; f < t.nf; ++f) a.k_host[f] = g.ds[c.param_ds[f]].src;
        a.nf = t.nf;
        a.combine = t.combine;
        a.ks = t.ks;
        KernelTimer kt(x, d, 0, ci, cs);
        CK(launch_edge(a, cs));
        kt.done(cs);
        ++d.launches;
        return TG_OK;
    }
    // CNN: U1 -> U2 -> U3 on the compute stream; T2 and T4 stay in the slot
    const bool strm = c.bias == "streamed";
    const bool plane = c.bias != "scalar";
    const int64_t w1 = t.w[1], w2 = t.w[2], w3 = t.w[3], w4 = t.w[4], w5 = t.w[5];
    float* t2 = (float*)(base + c.slot.t2);
    float* t4 = (float*)(base + c.slot.t4);
    {
        CnnU1Args a{};
        if (c.device_io) {
            a.in = X.src + (size_t)ch.img * t.H * t.W;
            a.in_img_stride = t.H * t.W;
            a.in_row0 = 0;
        } else {
            a.in = (const float*)(base + c.slot.in);
            a.in_img_stride = ch.in.n() * t.W;
            a.in_row0 = ch.in.a;
        }
        a.W = t.W;
        a.k1_host = g.ds[t.prm[0]].src;
        a.b1_plane = plane;
        if (strm) {
            a.b1 = (const float*)(base + c.slot.b1);
            a.b1_row0 = ch.c1.a;
            a.b1_rows = ch.c1.n();
        } else {
            a.b1 = param(1);
            a.b1_row0 = 0;
            a.b1_rows = t.h[1];
        }
        a.p2_host = g.ds[t.prm[2]].src;
        a.t2 = t2;
        a.t2_img_stride = 8 * ch.t2.n() * w2;  // fp32 planes, or 2 fp16 parts x 8 channels (same bytes)
        a.t2_row0 = ch.t2.a;
        a.t2_rows = ch.t2.n();
        a.w1 = w1;
        a.w2 = w2;
        a.nimg = ch.nimg;
        a.bf16_out = c.precision == TG_BF16_TC;
        a.t2_h3 = c.precision == TG_FP32_TC;
        KernelTimer kt(x, d, 1, ci, cs);
        CK(launch_cnn_u1(a, cs));
        kt.done(cs);
        ++d.launches;
    }
    {
        CnnU2Args a{};
        a.t2 = t2;
        a.t2_img_stride = 8 * ch.t2.n() * w2;
        a.t2_row0 = ch.t2.a;
        a.t2_rows = ch.t2.n();
        a.w2 = w2;
        a.k3_host = g.ds[t.prm[3]].src;
        a.b3_plane = plane;
        if (strm) {
            a.b3 = (const float*)(base + c.slot.b3);
            a.b3_row0 = ch.c3.a;
            a.b3_rows = ch.c3.n();
        } else {
            a.b3 = param(4);
            a.b3_row0 = 0;
            a.b3_rows = t.h[3];
        }
        a.p4_host = g.ds[t.prm[5]].src;
        a.t4 = t4;
        a.t4_img_stride = (c.precision == TG_FP32_TC ? 24 : 20) * ch.t4.n() * w4;
        a.t4_row0 = ch.t4.a;
        a.t4_rows = ch.t4.n();
        a.w3 = w3;
        a.w4 = w4;
        a.nimg = ch.nimg;
        a.bf16_tc = c.precision == TG_BF16_TC;
        a.k3_tc = c.k3tc_off == UINT64_MAX ? nullptr : (const uint16_t*)(d.arena + c.k3tc_off);
        a.p4_dev = param(5);
        if (c.precision == TG_FP32_TC) {
            a.k3_h3 = (const uint16_t*)(d.arena + c.k3tc_off);
            a.w_unscale = 1.f / (cnn_h3_act_scale() * x->k3_scale);
        }
        KernelTimer kt(x, d, 2, ci, cs);
        CK(a.bf16_tc ? launch_cnn_u2_tc(a, cs)
                     : c.precision == TG_FP32_TC ? launch_cnn_u2_h3(a, cs) : launch_cnn_u2(a, cs));
        kt.done(cs);
        ++d.launches;
    }
    {
        CnnU3Args a{};
        a.t4 = t4;
        a.t4_img_stride = (c.precision == TG_FP32_TC ? 24 : 20) * ch.t4.n() * w4;
        a.t4_row0 = ch.t4.a;
        a.t4_rows = ch.t4.n();
        a.w4 = w4;
        a.k5 = param(6);
        a.k6 = param(8);
        a.b5_plane = a.b6_plane = plane;
        a.b5_q4 = b5_quads(c) ? 1 : 0;
        if (strm) {
            a.b5 = (const float*)(base + c.slot.b5);
            a.b6 = (const float*)(base + c.slot.b6);
            a.b5_row0 = a.b6_row0 = ch.out.a;
            a.b5_rows = a.b6_rows = ch.out.n();
        } else {
            a.b5 = param(7);
            a.b6 = param(9);
            a.b5_row0 = a.b6_row0 = 0;
            a.b5_rows = a.b6_rows = t.h[5];
        }
        if (c.device_io) {
            a.out = Y.dst + (size_t)ch.img * 9 * t.h[5] * w5 + (size_t)ch.out.a * w5;
            a.out_img_stride = 9 * t.h[5] * w5;
            a.out_plane_stride = t.h[5] * w5;
        } else {
            a.out = (float*)(base + c.slot.out);
            a.out_img_stride = 9 * ch.out.n() * w5;
            a.out_plane_stride = ch.out.n() * w5;
        }
        a.out_row0 = ch.out.a;
        a.out_rows = ch.out.n();
        a.w5 = w5;
        a.n5 = t.n5;
        a.nimg = ch.nimg;
        a.bf16_tc = c.precision == TG_BF16_TC;
        a.k5_tc = c.k5tc_off == UINT64_MAX ? nullptr : (const uint16_t*)(d.arena + c.k5tc_off);
        a.w_unscale = c.precision == TG_FP32_TC ? 1.f / (cnn_h3_act_scale() * x->k5_scale) : 1.f;
        a.n_pad = cnn_n5_pad(t.n5);
        a.k6_host = g.ds[t.prm[8]].src;
        KernelTimer kt(x, d, 3, ci, cs);
        CK(a.bf16_tc ? launch_cnn_u3_tc(a, cs)
                     : c.precision == TG_FP32_TC ? launch_cnn_u3_h3(a, cs) : launch_cnn_u3(a, cs));
        kt.done(cs);
        ++d.launches;
    }
    return TG_OK;
}

tg_status run_device(tg_plan* p, tg_exec* x, DevState& d, bool blocking, cudaStream_t caller, bool ordered,
                     bool capturing = false) {
    const Graph& g = graph_of(p);
    const PlanCore& c = p->core;
    CK(cudaSetDevice(d.dev));
    cudaStream_t S0 = d.st[0], S1 = d.st[1], S2 = d.st[2];
    // The caller's stream: the execution starts after the work enqueued on it so far
    // (device-resident inputs may be produced there) and later work on it starts after the
    // execution (device-resident outputs may be consumed there).
    if (ordered) {
        CK(cudaEventRecord(d.ev_caller, caller));
        CK(cudaStreamWaitEvent(S1, d.ev_caller, 0));
    }
    // Fork: the copy streams are ordered after earlier work on the compute stream only where
    // they need to be -- device-resident I/O (inputs may come from earlier kernels) and a
    // parameter (re-)upload (earlier kernels may still read the old parameters). Otherwise a
    // new execution's H2D copies only wait for their slot to be free (the slot ring and its
    // events persist across executions), so back-to-back executions of one plan pipeline:
    // the next batch uploads while the previous one's last chunks compute and download.
    // (when the execution is being captured into a graph, the copy streams always fork from S1
    // -- that is how they join the capture -- and the slot ring starts afresh: graph replays on
    // S1 are serialised, so no chunk waits for a slot of an earlier execution)
    // A direct execution after a graph replay does the same: the slot events were last recorded
    // inside the capture, so they neither order against the replays nor may be waited on.
    // A device-resident plan moves no data on the copy streams (only a parameter upload on S0), so
    // it forks them only for that upload and never joins them: its captured graph is then just the
    // kernels on S1 (configs[0]: fewer graph nodes, less launch overhead per step).
    const bool fresh = capturing || d.after_graph;
    d.after_graph = false;
    const bool fork = c.device_io ? !d.params_resident : (!d.params_resident || fresh);
    if (fork) {
        CK(cudaEventRecord(d.ev_fork, S1));
        CK(cudaStreamWaitEvent(S0, d.ev_fork, 0));
        CK(cudaStreamWaitEvent(S2, d.ev_fork, 0));
    }
    // parameters (never split): uploaded by the first execution and kept
    // resident in the arena for later ones (tg_plan_invalidate_params forces a re-upload)
    if (!d.params_resident) {
        ProfRec pr{10, nullptr, nullptr};
        if (x->prof_copies) {
            pr.a = pool_event(d);
            pr.b = pool_event(d);
            cudaEventRecord(pr.a, S0);
        }
        for (size_t i = 0; i < c.param_ds.size(); ++i) {
            if (c.param_off[i] == UINT64_MAX) continue;
            const Ds& P = g.ds[c.param_ds[i]];
            const float* src = (i == 7 && b5_quads(c)) ? x->b5q4.data() : P.src;
            CK(cudaMemcpyAsync(d.arena + c.param_off[i], src, (size_t)P.numel() * 4, cudaMemcpyHostToDevice, S0));
        }
        if (c.k5tc_off != UINT64_MAX) {
            // tensor-core B operands (bf16, or fp16-split for TG_FP32_TC), prepared on the host
            // by exec_run before any device thread starts (prepare_tc_operands)
            const std::vector<uint16_t>& k3 = c.precision == TG_FP32_TC ? x->k3h3 : x->k3tc;
            const std::vector<uint16_t>& k5 = c.precision == TG_FP32_TC ? x->k5h3 : x->k5tc;
            CK(cudaMemcpyAsync(d.arena + c.k3tc_off, k3.data(), k3.size() * 2, cudaMemcpyHostToDevice, S0));
            CK(cudaMemcpyAsync(d.arena + c.k5tc_off, k5.data(), k5.size() * 2, cudaMemcpyHostToDevice, S0));
        }
        if (x->prof_copies) {
            cudaEventRecord(pr.b, S0);
            d.prof.push_back(pr);
        }
        CK(cudaEventRecord(d.ev_params, S0));
        CK(cudaStreamWaitEvent(S1, d.ev_params, 0));
        d.params_resident = true;
    }
    const int D = c.depth;
    for (int64_t k = 0; k < d.c1 - d.c0; ++k, ++d.seq) {
        const Chunk& ch = c.chunks[d.c0 + k];
        const int64_t sq = fresh ? k : d.seq;  // position in the slot ring
        const int s = (int)(sq % D);
        if (!c.device_io) {
            if (sq >= D) CK(cudaStreamWaitEvent(S0, d.ev_comp[s], 0));
            ProfRec pr{10, nullptr, nullptr, d.c0 + k};
            if (x->prof_copies) {
                pr.a = pool_event(d);
                pr.b = pool_event(d);
                cudaEventRecord(pr.a, S0);
            }
            tg_status st = enqueue_h2d(p, d, ch, s);
            if (st != TG_OK) return st;
            if (x->prof_copies) {
                cudaEventRecord(pr.b, S0);
                d.prof.push_back(pr);
            }
            CK(cudaEventRecord(d.ev_h2d[s], S0));
            CK(cudaStreamWaitEvent(S1, d.ev_h2d[s], 0));
            if (sq >= D) CK(cudaStreamWaitEvent(S1, d.ev_d2h[s], 0));
        }
        tg_status st = launch_units(p, x, d, ch, s);
        if (st != TG_OK) return st;
        CK(cudaEventRecord(d.ev_comp[s], S1));
        if (!c.device_io) {
            CK(cudaStreamWaitEvent(S2, d.ev_comp[s], 0));
            ProfRec pr{11, nullptr, nullptr, d.c0 + k};
            if (x->prof_copies) {
                pr.a = pool_event(d);
                pr.b = pool_event(d);
                cudaEventRecord(pr.a, S2);
            }
            st = enqueue_d2h(p, d, ch, s);
            if (st != TG_OK) return st;
            if (x->prof_copies) {
                cudaEventRecord(pr.b, S2);
                d.prof.push_back(pr);
            }
            CK(cudaEventRecord(d.ev_d2h[s], S2));
        }
    }
    // join: the compute stream waits for the last D2H, so it marks the end of everything
    // (device-resident I/O: nothing ran on the copy streams but a parameter upload, which S1
    // already waited for through ev_params)
    if (!c.device_io) {
        CK(cudaEventRecord(d.ev_join, S2));
        CK(cudaStreamWaitEvent(S1, d.ev_join, 0));
    }
    if (ordered) {
        CK(cudaEventRecord(d.ev_done, S1));
        CK(cudaStreamWaitEvent(caller, d.ev_done, 0));
    }
    if (blocking) CK(cudaStreamSynchronize(S1));
    return TG_OK;
}

// Host copies of the tensor-core B operands, derived from the parameters once per plan (and
// again after tg_plan_invalidate_params) on the calling thread, before any per-device thread
// reads them.
void prepare_tc_operands(tg_plan* p, tg_exec* x) {
    const Graph& g = graph_of(p);
    const PlanCore& c = p->core;
    if (c.k5tc_off == UINT64_MAX) return;
    if (b5_quads(c) && x->b5q4.empty()) {  // [n5][hw] -> [n5/4][hw][4]
        const float* src = g.ds[c.t.prm[7]].src;
        const int64_t n5 = c.t.n5, hw = c.t.h[5] * c.t.w[5];
        x->b5q4.resize((size_t)(n5 * hw));
        for (int64_t ch = 0; ch < n5; ++ch)
            for (int64_t q = 0; q < hw; ++q) x->b5q4[((ch >> 2) * hw + q) * 4 + (ch & 3)] = src[ch * hw + q];
    }
    const Ds& K3 = g.ds[c.t.prm[3]];
    const Ds& K5 = g.ds[c.t.prm[6]];
    if (c.precision == TG_FP32_TC && x->k5h3.empty()) {
        x->k3_scale = cnn_h3_weight_scale(K3.src, (size_t)K3.numel());
        x->k5_scale = cnn_h3_weight_scale(K5.src, (size_t)K5.numel());
        x->k3h3.resize(cnn_k3_h3_bytes() / 2);
        cnn_prepare_k3_h3(K3.src, x->k3_scale, x->k3h3.data());
        x->k5h3.resize(cnn_k5_h3_bytes(c.t.n5) / 2);
        cnn_prepare_k5_h3(K5.src, c.t.n5, x->k5_scale, x->k5h3.data());
    }
    if (c.precision == TG_BF16_TC && x->k5tc.empty()) {
        x->k3tc.resize(cnn_k3_tc_bytes() / 2);
        x->k5tc.resize(cnn_k5_tc_bytes(c.t.n5) / 2);
        cnn_prepare_k3_tc(K3.src, x->k3tc.data());
        cnn_prepare_k5_tc(K5.src, c.t.n5, x->k5tc.data());
    }
}

}  // namespace

namespace tg {

tg_status exec_run(tg_plan* p, bool blocking, void* caller_stream, bool has_caller) {
    if (!p->exec) p->exec = new tg_exec();
    tg_exec* x = p->exec;
    const Graph& g = graph_of(p);
    const PlanCore& c = p->core;
    if (!x->ready) {
        std::vector<int32_t> devs = g.devices;
        if (devs.empty()) {
            int cur = 0;
            CK(cudaGetDevice(&cur));
            devs.push_back(cur);
        }
        x->devs.resize(devs.size());
        const int64_t n = c.c1 - c.c0, nd = (int64_t)devs.size();
        for (size_t i = 0; i < devs.size(); ++i) {
            DevState& d = x->devs[i];
            d.dev = devs[i];
            d.c0 = c.c0 + n * (int64_t)i / nd;
            d.c1 = c.c0 + n * (int64_t)(i + 1) / nd;
            tg_status st = init_device(p, d);
            if (st != TG_OK) return st;
        }
        tg_status st = register_host(p, x);
        if (st != TG_OK) return st;
        x->ready = true;
    }
    bool any_upload = false;
    for (auto& d : x->devs) any_upload |= !d.params_resident;
    if (any_upload) prepare_tc_operands(p, x);
    // caller-stream ordering: an explicit stream (tg_execute_on), or for device-resident I/O
    // the legacy default stream (where PyTorch's default stream and plain CUDA code enqueue)
    const bool ordered = has_caller || c.device_io;
    const cudaStream_t caller = has_caller ? (cudaStream_t)caller_stream : cudaStreamLegacy;
    if (ordered && x->devs.size() > 1)
        return fail(TG_E_UNSUPPORTED, "execute: ordering against a caller stream needs a one-device plan");
    tg_status result = TG_OK;
    if (x->graph_mode && x->devs.size() == 1 && !any_upload && !x->profiling) {
        // CUDA-graph replay: the execution's whole enqueue sequence (copies, kernels, events on
        // the three streams) captured once, then launched as one graph on the compute stream
        DevState& d = x->devs[0];
        CK(cudaSetDevice(d.dev));
        cudaStream_t S1 = d.st[1];
        if (!d.graph) {
            const int64_t l0 = d.launches;
            CK(cudaStreamBeginCapture(S1, cudaStreamCaptureModeRelaxed));
            tg_status st = run_device(p, x, d, false, nullptr, false, true);
            cudaGraph_t gr = nullptr;
            cudaError_t e = cudaStreamEndCapture(S1, &gr);
            if (st != TG_OK) {
                if (gr) cudaGraphDestroy(gr);
                return st;
            }
            if (e != cudaSuccess) return fail(TG_E_CUDA, std::string("graph capture: ") + cudaGetErrorString(e));
            e = cudaGraphInstantiate(&d.graph, gr, 0);
            cudaGraphDestroy(gr);
            if (e != cudaSuccess) {
                d.graph = nullptr;
                return fail(TG_E_CUDA, std::string("graph instantiate: ") + cudaGetErrorString(e));
            }
            d.graph_launches = d.launches - l0;
            d.launches = l0;
        }
        if (ordered) {
            CK(cudaEventRecord(d.ev_caller, caller));
            CK(cudaStreamWaitEvent(S1, d.ev_caller, 0));
        }
        CK(cudaGraphLaunch(d.graph, S1));
        d.launches += d.graph_launches;
        d.after_graph = true;
        if (ordered) {
            CK(cudaEventRecord(d.ev_done, S1));
            CK(cudaStreamWaitEvent(caller, d.ev_done, 0));
        }
        if (blocking) CK(cudaStreamSynchronize(S1));
    } else if (x->devs.size() == 1) {
        result = run_device(p, x, x->devs[0], blocking, caller, ordered);
    } else {
        std::vector<tg_status> sts(x->devs.size(), TG_OK);
        std::vector<std::string> errs(x->devs.size());
        std::vector<std::thread> th;
        for (size_t i = 0; i < x->devs.size(); ++i)
            th.emplace_back([&, i] {
                sts[i] = run_device(p, x, x->devs[i], blocking, nullptr, false);
                if (sts[i] != TG_OK) errs[i] = tg_last_error();
            });
        for (auto& t : th) t.join();
        for (size_t i = 0; i < sts.size(); ++i)
            if (sts[i] != TG_OK) {
                result = fail(sts[i], errs[i]);
                break;
            }
    }
    int64_t l = 0;
    for (auto& d : x->devs) l += d.launches;
    p->launches = l;
    ++x->timing.executions;
    return result;
}

tg_status exec_set_profiling(tg_plan* p, int level) {
    if (!p->exec) p->exec = new tg_exec();
    const bool on = level != 0;
    p->exec->profiling = on;
    p->exec->prof_copies = level == 1;
    if (on) {
        p->exec->timing = tg_timing{};
        p->exec->trace.clear();
    }
    return TG_OK;
}

tg_status exec_timing(tg_plan* p, tg_timing* out) {
    if (!p->exec) {
        *out = tg_timing{};
        return TG_OK;
    }
    tg_exec* x = p->exec;
    for (auto& d : x->devs) {
        CK(cudaSetDevice(d.dev));
        for (auto& r : d.prof) {
            CK(cudaEventSynchronize(r.b));
            float ms = 0.f, t0 = 0.f;
            CK(cudaEventElapsedTime(&ms, r.a, r.b));
            CK(cudaEventElapsedTime(&t0, d.prof.front().a, r.a));
            x->trace.push_back({d.dev, r.kind, r.chunk, (double)t0, (double)t0 + ms});
            if (r.kind < 4) {
                x->timing.kernel_ms[r.kind] += ms;
                x->timing.unit_launches[r.kind] += 1;
                x->timing.launches += 1;
            } else if (r.kind == 10) {
                x->timing.h2d_ms += ms;
            } else {
                x->timing.d2h_ms += ms;
            }
            d.ev_pool.push_back(r.a);
            d.ev_pool.push_back(r.b);
        }
        d.prof.clear();
    }
    *out = x->timing;
    return TG_OK;
}

void exec_destroy(tg_plan* p) {
    tg_exec* x = p->exec;
    if (!x) return;
    const Graph& g = graph_of(p);
    for (auto& d : x->devs) {
        if (cudaSetDevice(d.dev) != cudaSuccess) continue;
        if (d.st[1]) cudaStreamSynchronize(d.st[1]);
        for (auto& r : d.prof) {
            cudaEventDestroy(r.a);
            cudaEventDestroy(r.b);
        }
        for (auto e : d.ev_pool) cudaEventDestroy(e);
        for (auto* v : {&d.ev_h2d, &d.ev_comp, &d.ev_d2h})
            for (auto e : *v)
                if (e) cudaEventDestroy(e);
        if (d.graph) cudaGraphExecDestroy(d.graph);
        for (auto e : {d.ev_fork, d.ev_join, d.ev_params, d.ev_caller, d.ev_done})
            if (e) cudaEventDestroy(e);
        if (d.arena) {
            if (d.own_arena)
                cudaFree(d.arena);
            else if (g.has_rt && g.rt.free)
                g.rt.free(d.arena, d.dev, g.rt.ctx);
        }
        for (int w = 0; w < 3; ++w)
            if (d.own_st[w] && d.st[w]) cudaStreamDestroy(d.st[w]);
    }
    for (void* ptr : x->registered) cudaHostUnregister(ptr);
    cudaGetLastError();
    delete x;
    p->exec = nullptr;
}

tg_status exec_trace(tg_plan* p, tg_trace_rec* out, size_t cap, size_t* n) {
    tg_timing t{};
    tg_status st = exec_timing(p, &t);  // collects pending records into the trace
    if (st != TG_OK) return st;
    *n = 0;
    if (!p->exec) return TG_OK;
    const std::vector<tg_trace_rec>& tr = p->exec->trace;
    *n = tr.size();
    for (size_t i = 0; i < tr.size() && i < cap; ++i) out[i] = tr[i];
    return TG_OK;
}

uint64_t exec_registered_bytes(const tg_plan* p) { return p->exec ? p->exec->registered_bytes : 0; }

tg_status exec_set_graph(tg_plan* p, bool on) {
    if (!p->exec) p->exec = new tg_exec();
    tg_exec* x = p->exec;
    x->graph_mode = on;
    for (auto& d : x->devs)
        if (d.graph) {
            if (cudaSetDevice(d.dev) == cudaSuccess) cudaStreamSynchronize(d.st[1]);
            cudaGraphExecDestroy(d.graph);
            d.graph = nullptr;
        }
    return TG_OK;
}

void exec_invalidate_params(tg_plan* p) {
    if (!p->exec) return;
    // a captured graph holds the kernels' weight parameters by value: recapture after the upload
    if (p->exec->graph_mode) exec_set_graph(p, true);
    for (auto& d : p->exec->devs) d.params_resident = false;
    p->exec->k3tc.clear();  // the bf16 tensor-core operands are re-derived from the new values
    p->exec->k5tc.clear();
    p->exec->k5h3.clear();
    p->exec->k3h3.clear();
    p->exec->b5q4.clear();
}

}  // namespace tg
