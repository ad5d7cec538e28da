// tg_internal.h -- graph IR, plan and executor structures behind include/tg.h.
// Product code: shares nothing with oracle/.
#pragma once

#include <cstdint>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/tg.h"

namespace tg {

// ----------------------------------------------------------------------------- errors
void set_error(const std::string& msg);
tg_status fail(tg_status code, const std::string& msg);

// ----------------------------------------------------------------------------- graph IR
enum class DsKind { Input, Param, Temp };
enum class Loc { None, Host, Device };

struct Ds {
    int64_t d[4] = {1, 1, 1, 1};  // n, c, h, w
    DsKind kind = DsKind::Temp;
    const float* src = nullptr;   // input/param source (host or device)
    Loc src_loc = Loc::None;
    float* dst = nullptr;         // bound output destination
    Loc dst_loc = Loc::None;
    int producer = -1;            // node id
    std::vector<float> owned;     // library-derived parameter (e.g. rot90 kernel)
    int64_t numel() const { return d[0] * d[1] * d[2] * d[3]; }
};

enum class OpKind { Conv, Elem, Tanh, Max, Sub, Matmul };

struct Node {
    OpKind op;
    std::vector<int> ins;  // DS ids (conv: x, k; sub: x, p; matmul: a, b)
    int out = -1;
    int32_t pad = TG_VALID;  // conv
    int32_t bias = -1;       // conv bias DS id or -1
    int32_t elem = 0;        // elementwise op
    float a = 1.f, b = 0.f;  // affine
    int32_t s = 2;           // subsample window/stride
};

struct Graph {
    std::vector<Ds> ds;
    std::vector<Node> nodes;
    // target parameters
    std::vector<int32_t> devices;
    uint64_t budget = 0;
    int32_t precision = TG_FP32;
    int64_t max_chunk_px = int64_t(1) << 25;
    int32_t depth = 3;
    int32_t rank = 0, world = 1;
    tg_runtime rt{};
    bool has_rt = false;
};

// ----------------------------------------------------------------------------- templates
enum class Tmpl { Edge, Cnn };

struct RowRange {
    int64_t a = 0, b = 0;
    int64_t n() const { return b - a; }
};

struct Chunk {
    int64_t img = 0, nimg = 1;
    RowRange in, c1, t2, c3, t4, out;  // edge uses in/out only
};

struct Template {
    Tmpl kind = Tmpl::Edge;
    int input = -1, output = -1;
    int64_t n = 0, H = 0, W = 0;
    // edge
    int ks = 16;
    int k1 = -1, k2 = -1;  // kernel DS ids (fold order E1, E2, -E1, -E2)
    int nf = 2;            // convolutions (orientations with remaps = 2 nf)
    int kk[4] = {-1, -1, -1, -1};
    int combine = 0;       // 0 max with remaps, 1 sum, 2 max |.|, 3 max
    // cnn
    int n5 = 0;
    bool bias_plane = true;
    int prm[10] = {-1, -1, -1, -1, -1, -1, -1, -1, -1, -1};
    int64_t h[6] = {0}, w[6] = {0};  // level 0 input, 1 C1, 2 S2, 3 C3, 4 S4, 5 C5/C6
};

// slot layout inside the arena (byte offsets relative to the slot base)
struct SlotLayout {
    uint64_t in = 0, t2 = 0, t4 = 0, out = 0, b1 = 0, b3 = 0, b5 = 0, b6 = 0;
    uint64_t bytes = 0;
};

struct PlanCore {
    Template t;
    int32_t mode = TG_FUSED;
    int32_t precision = TG_FP32;
    bool device_io = false;
    std::string bias = "none";  // none | resident | streamed | scalar
    std::string split;          // batch | rows
    int64_t B = 1, R = 0;
    int32_t depth = 3;
    uint64_t budget = 0;
    int64_t max_chunk_px = 0;
    uint64_t param_bytes = 0, slot_bytes = 0, arena_bytes = 0;
    std::vector<uint64_t> param_off;  // offset of each param (template order) in param region
    std::vector<int> param_ds;        // DS ids in template order
    std::vector<bool> param_streamed; // true: bias rows streamed per chunk
    uint64_t k3tc_off = UINT64_MAX, k5tc_off = UINT64_MAX;  // bf16 tensor-core B operands
    SlotLayout slot;
    std::vector<Chunk> chunks;        // global chunk list
    int64_t c0 = 0, c1 = 0;           // this process's shard
    int32_t rank = 0, world = 1;
    uint64_t h2d = 0, d2h = 0, io_lb = 0, total = 0;
    // H2D split (fused): parameter floats uploaded (streamed bias planes excluded), operands
    // derived from them on the host (tensor-core B operands), chunk rows (+ streamed bias rows)
    uint64_t h2d_param = 0, h2d_derived = 0, h2d_chunk = 0;
    uint64_t io_lb_data = 0;      // io_lb without the parameters (images in + outputs out)
    int64_t chunk_cap = 0;        // the policy's cap on B (batch) or R (rows)
    uint64_t slot_bytes_next = 0; // slot bytes at B + 1 / R + 1 (0 when at the cap)
    int64_t nops = 0, nds = 0;
    int64_t n_units = 1;
    // per-operator modes (TG_PER_OP, TG_BASELINE): the abstract schedule over graph DS/nodes
    std::vector<int> po_ds;       // sched DS id -> graph DS id
    std::vector<uint64_t> po_size;
    std::vector<int32_t> po_kind;
    std::vector<int> po_ops;      // sched op id -> graph node id
    std::vector<std::vector<int32_t>> po_ins, po_outs;
    std::vector<int32_t> po_order;
    std::vector<std::pair<int32_t, int32_t>> po_trace;  // (0 h2d | 1 run | 2 d2h | 3 free, id)
    uint64_t po_capacity = 0;
    // operator splitting (TG_PER_OP, R19): sched DS k is rows
    // [po_r0[k], po_r1[k]) of graph DS po_ds[k]; sched op j is piece po_piece[j] of node po_ops[j]
    std::vector<int64_t> po_r0, po_r1;
    std::vector<int32_t> po_piece;
    std::vector<int32_t> po_k;    // split factor per graph node (0: not needed)
    std::vector<uint64_t> po_trace_off;  // arena offset of the DS each trace step touches (static
                                         // layout, PAPER.md:409 fragmentation margin)
};

tg_status recognise(const Graph& g, Template& t);
tg_status make_plan_per_op(const Graph& g, int32_t mode, PlanCore& p);
tg_status make_plan(const Graph& g, int32_t mode, PlanCore& p);
std::string plan_json(const PlanCore& p);
std::string plan_json_per_op(const PlanCore& p);

}  // namespace tg

// abstract operator graph of the transfer scheduler (sched.cpp)
struct tg_sched {
    struct D {
        uint64_t size;
        int32_t kind;  // TG_DS_*
    };
    struct O {
        std::vector<int32_t> ins, outs;
    };
    std::vector<D> ds;
    std::vector<O> ops;
};

namespace tg {
std::vector<int32_t> sched_dfs(const tg_sched& s);
// trace kinds: 0 H2D ds, 1 run op, 2 D2H ds, 3 (frees only) ds leaves the GPU
uint64_t sched_transfers(const tg_sched& s, const std::vector<int32_t>& order, uint64_t capacity,
                         std::vector<std::pair<int32_t, int32_t>>* trace, bool frees);
}  // namespace tg

// opaque handles
struct tg_graph {
    tg::Graph g;
};

struct tg_exec;         // engine state (engine.cu)
struct tg_perop_exec;   // per-operator executor state (engine_perop.cu)

struct tg_plan {
    const tg_graph* graph = nullptr;
    tg::PlanCore core;
    tg_exec* exec = nullptr;
    tg_perop_exec* perop = nullptr;
    int64_t launches = 0;
};

namespace tg {
tg_status exec_run(tg_plan* p, bool blocking, void* caller_stream = nullptr, bool has_caller = false);
tg_status exec_set_profiling(tg_plan* p, int level);
tg_status exec_set_graph(tg_plan* p, bool on);
tg_status exec_timing(tg_plan* p, tg_timing* out);
tg_status exec_trace(tg_plan* p, tg_trace_rec* out, size_t cap, size_t* n);
void exec_destroy(tg_plan* p);
uint64_t exec_registered_bytes(const tg_plan* p);
void exec_invalidate_params(tg_plan* p);
tg_status exec_run_per_op(tg_plan* p, bool blocking);
tg_status exec_timing_per_op(tg_plan* p, tg_timing* out);
void exec_set_profiling_per_op(tg_plan* p, bool on);
void exec_destroy_per_op(tg_plan* p);
// descriptor of sched op `op` of a per-op plan given the arena offsets of its pieces
bool oplib_desc(const Graph& g, const PlanCore& c, int op, const std::vector<int64_t>& off, const char* arena,
                tg_oplib_op& d);
// operator library (oplib.cu): one operator piece on `stream` (a cudaStream_t)
tg_status oplib_run(const tg_oplib_op& op, void* stream);
// code generator (codegen.cpp)
std::string plan_codegen(const tg_plan* p);
}  // namespace tg
