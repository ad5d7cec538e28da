// api.cpp -- the C ABI of include/tg.h: graph building, target parameters, plan handles.
// Graph nodes follow the paper's operator graph (vertices are parallel
// computations, edges data dependencies; footprints statically known).
#include <cuda_runtime.h>

#include <cmath>
#include <cstring>
#include <new>
#include <string>

#include "kernels/kernels.h"
#include "tg_internal.h"

namespace tg {
static thread_local std::string g_last_error;
void set_error(const std::string& msg) { g_last_error = msg; }
tg_status fail(tg_status code, const std::string& msg) {
    g_last_error = msg;
    return code;
}
}  // namespace tg

using namespace tg;

#define TG_GUARD_BEGIN try {
#define TG_GUARD_END                                                   \
    }                                                                  \
    catch (const std::bad_alloc&) {                                    \
        return fail(TG_E_OOM, "host allocation failed");               \
    }                                                                  \
    catch (const std::exception& e) {                                  \
        return fail(TG_E_ARG, std::string("internal error: ") + e.what()); \
    }

static bool valid_id(const Graph& g, tg_id id) { return id >= 0 && id < (tg_id)g.ds.size(); }

static tg_id add_ds(Graph& g, const int64_t d[4], DsKind kind) {
    Ds x;
    for (int i = 0; i < 4; ++i) x.d[i] = d[i];
    x.kind = kind;
    g.ds.push_back(std::move(x));
    return (tg_id)g.ds.size() - 1;
}

extern "C" {

const char* tg_last_error(void) { return g_last_error.c_str(); }
const char* tg_version(void) { return "tg 0.2 sm_100a"; }

tg_status tg_probe_fp32_peak(int32_t device, double* tflops) {
    if (!tflops) return fail(TG_E_ARG, "tg_probe_fp32_peak: NULL out pointer");
    TG_GUARD_BEGIN
    cudaError_t e = probe_fp32_peak(device, tflops);
    if (e != cudaSuccess) return fail(TG_E_CUDA, std::string("tg_probe_fp32_peak: ") + cudaGetErrorString(e));
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_graph_create(tg_graph** g) {
    if (!g) return fail(TG_E_ARG, "tg_graph_create: NULL out pointer");
    TG_GUARD_BEGIN
    *g = new tg_graph();
    return TG_OK;
    TG_GUARD_END
}

void tg_graph_destroy(tg_graph* g) { delete g; }

static tg_status input_common(tg_graph* g, int64_t n, int64_t c, int64_t h, int64_t w,
                              const float* p, Loc loc, tg_id* out) {
    if (!g || !p || !out) return fail(TG_E_ARG, "tg_input: NULL argument");
    if (n <= 0 || c <= 0 || h <= 0 || w <= 0) return fail(TG_E_SHAPE, "tg_input: non-positive dim");
    TG_GUARD_BEGIN
    int64_t d[4] = {n, c, h, w};
    tg_id id = add_ds(g->g, d, DsKind::Input);
    g->g.ds[id].src = p;
    g->g.ds[id].src_loc = loc;
    *out = id;
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_input(tg_graph* g, int64_t n, int64_t c, int64_t h, int64_t w, const float* host,
                   tg_id* out) {
    return input_common(g, n, c, h, w, host, Loc::Host, out);
}

tg_status tg_input_device(tg_graph* g, int64_t n, int64_t c, int64_t h, int64_t w,
                          const float* dev, tg_id* out) {
    return input_common(g, n, c, h, w, dev, Loc::Device, out);
}

tg_status tg_param(tg_graph* g, int64_t d0, int64_t d1, int64_t d2, int64_t d3, const float* host,
                   tg_id* out) {
    if (!g || !host || !out) return fail(TG_E_ARG, "tg_param: NULL argument");
    if (d0 <= 0 || d1 <= 0 || d2 <= 0 || d3 <= 0) return fail(TG_E_SHAPE, "tg_param: non-positive dim");
    TG_GUARD_BEGIN
    int64_t d[4] = {d0, d1, d2, d3};
    tg_id id = add_ds(g->g, d, DsKind::Param);
    g->g.ds[id].src = host;
    g->g.ds[id].src_loc = Loc::Host;
    *out = id;
    return TG_OK;
    TG_GUARD_END
}

static tg_id add_node(Graph& g, Node nd, const int64_t d[4]) {
    tg_id y = add_ds(g, d, DsKind::Temp);
    nd.out = y;
    g.nodes.push_back(nd);
    g.ds[y].producer = (int)g.nodes.size() - 1;
    return y;
}

tg_status tg_conv2d(tg_graph* g, tg_id x, tg_id k, tg_id bias, int32_t pad, tg_id* y) {
    if (!g || !y) return fail(TG_E_ARG, "tg_conv2d: NULL argument");
    Graph& G = g->g;
    if (!valid_id(G, x) || !valid_id(G, k) || (bias != -1 && !valid_id(G, bias)))
        return fail(TG_E_ARG, "tg_conv2d: unknown DS id");
    if (pad != TG_VALID && pad != TG_SAME) return fail(TG_E_ARG, "tg_conv2d: pad must be TG_VALID or TG_SAME");
    const Ds& X = G.ds[x];
    const Ds& K = G.ds[k];
    if (K.kind != DsKind::Param) return fail(TG_E_ARG, "tg_conv2d: kernel must be a parameter");
    const int64_t co = K.d[0], ci = K.d[1], kh = K.d[2], kw = K.d[3];
    if (ci != X.d[1]) return fail(TG_E_SHAPE, "tg_conv2d: kernel input channels != input planes");
    int64_t ho = X.d[2], wo = X.d[3];
    if (pad == TG_VALID) {
        ho = X.d[2] - kh + 1;
        wo = X.d[3] - kw + 1;
    }
    if (ho <= 0 || wo <= 0) return fail(TG_E_SHAPE, "tg_conv2d: kernel larger than input");
    if (bias != -1) {
        const Ds& B = G.ds[bias];
        const bool scalar = B.numel() == co && (B.d[0] * B.d[1] * B.d[2] == 1 || B.d[1] * B.d[2] * B.d[3] == 1);
        const bool plane = B.d[0] == 1 && B.d[1] == co && B.d[2] == ho && B.d[3] == wo;
        if (B.kind != DsKind::Param || (!scalar && !plane))
            return fail(TG_E_SHAPE, "tg_conv2d: bias must be a [co] or [1][co][ho][wo] parameter");
    }
    TG_GUARD_BEGIN
    Node nd;
    nd.op = OpKind::Conv;
    nd.ins = {x, k};
    nd.pad = pad;
    nd.bias = bias;
    int64_t d[4] = {X.d[0], co, ho, wo};
    *y = add_node(G, nd, d);
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_elementwise(tg_graph* g, int32_t op, const tg_id* xs, int32_t nx, float a, float b,
                         tg_id* y) {
    if (!g || !xs || !y || nx <= 0) return fail(TG_E_ARG, "tg_elementwise: bad argument");
    Graph& G = g->g;
    if (op < TG_ADD || op > TG_ABS) return fail(TG_E_ARG, "tg_elementwise: unknown op");
    if (op != TG_ADD && nx != 1) return fail(TG_E_ARG, "tg_elementwise: unary op takes one input");
    for (int i = 0; i < nx; ++i) {
        if (!valid_id(G, xs[i])) return fail(TG_E_ARG, "tg_elementwise: unknown DS id");
        for (int j = 0; j < 4; ++j)
            if (G.ds[xs[i]].d[j] != G.ds[xs[0]].d[j]) return fail(TG_E_SHAPE, "tg_elementwise: shape mismatch");
    }
    TG_GUARD_BEGIN
    Node nd;
    nd.op = OpKind::Elem;
    nd.ins.assign(xs, xs + nx);
    nd.elem = op;
    nd.a = a;
    nd.b = b;
    *y = add_node(G, nd, G.ds[xs[0]].d);
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_tanh(tg_graph* g, tg_id x, tg_id* y) {
    if (!g || !y) return fail(TG_E_ARG, "tg_tanh: NULL argument");
    Graph& G = g->g;
    if (!valid_id(G, x)) return fail(TG_E_ARG, "tg_tanh: unknown DS id");
    TG_GUARD_BEGIN
    Node nd;
    nd.op = OpKind::Tanh;
    nd.ins = {x};
    *y = add_node(G, nd, G.ds[x].d);
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_max_combine(tg_graph* g, const tg_id* xs, int32_t nx, tg_id* y) {
    if (!g || !xs || !y || nx <= 0) return fail(TG_E_ARG, "tg_max_combine: bad argument");
    Graph& G = g->g;
    for (int i = 0; i < nx; ++i) {
        if (!valid_id(G, xs[i])) return fail(TG_E_ARG, "tg_max_combine: unknown DS id");
        for (int j = 0; j < 4; ++j)
            if (G.ds[xs[i]].d[j] != G.ds[xs[0]].d[j]) return fail(TG_E_SHAPE, "tg_max_combine: shape mismatch");
    }
    TG_GUARD_BEGIN
    Node nd;
    nd.op = OpKind::Max;
    nd.ins.assign(xs, xs + nx);
    *y = add_node(G, nd, G.ds[xs[0]].d);
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_subsample(tg_graph* g, tg_id x, tg_id p, int32_t s, tg_id* y) {
    if (!g || !y) return fail(TG_E_ARG, "tg_subsample: NULL argument");
    Graph& G = g->g;
    if (!valid_id(G, x) || !valid_id(G, p)) return fail(TG_E_ARG, "tg_subsample: unknown DS id");
    if (s <= 0) return fail(TG_E_ARG, "tg_subsample: window must be positive");
    const Ds& X = G.ds[x];
    const Ds& P = G.ds[p];
    if (P.kind != DsKind::Param || P.numel() != X.d[1] * s * s)
        return fail(TG_E_SHAPE, "tg_subsample: kernel must be a [c][s][s] parameter");
    if (X.d[2] < s || X.d[3] < s) return fail(TG_E_SHAPE, "tg_subsample: input smaller than window");
    TG_GUARD_BEGIN
    Node nd;
    nd.op = OpKind::Sub;
    nd.ins = {x, p};
    nd.s = s;
    int64_t d[4] = {X.d[0], X.d[1], (X.d[2] - s) / s + 1, (X.d[3] - s) / s + 1};
    *y = add_node(G, nd, d);
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_matmul(tg_graph* g, tg_id a, tg_id b, tg_id* y) {
    if (!g || !y) return fail(TG_E_ARG, "tg_matmul: NULL argument");
    Graph& G = g->g;
    if (!valid_id(G, a) || !valid_id(G, b)) return fail(TG_E_ARG, "tg_matmul: unknown DS id");
    const Ds& A = G.ds[a];
    const Ds& B = G.ds[b];
    if (A.d[0] * A.d[1] != 1 || B.d[0] * B.d[1] != 1)
        return fail(TG_E_SHAPE, "tg_matmul: operands must be matrices [1][1][m][k] and [1][1][k][n]");
    if (A.d[3] != B.d[2]) return fail(TG_E_SHAPE, "tg_matmul: inner dimensions differ");
    TG_GUARD_BEGIN
    Node nd;
    nd.op = OpKind::Matmul;
    nd.ins = {a, b};
    int64_t d[4] = {1, 1, A.d[2], B.d[3]};
    *y = add_node(G, nd, d);
    return TG_OK;
    TG_GUARD_END
}

static tg_status output_common(tg_graph* g, tg_id y, float* dst, Loc loc) {
    if (!g || !dst) return fail(TG_E_ARG, "tg_output: NULL argument");
    Graph& G = g->g;
    if (!valid_id(G, y)) return fail(TG_E_ARG, "tg_output: unknown DS id");
    if (G.ds[y].producer < 0) return fail(TG_E_ARG, "tg_output: DS is not produced by an operator");
    G.ds[y].dst = dst;
    G.ds[y].dst_loc = loc;
    return TG_OK;
}

tg_status tg_output(tg_graph* g, tg_id y, float* host_dst) { return output_common(g, y, host_dst, Loc::Host); }
tg_status tg_output_device(tg_graph* g, tg_id y, float* dev_dst) { return output_common(g, y, dev_dst, Loc::Device); }

tg_status tg_shape(const tg_graph* g, tg_id id, int64_t dims[4]) {
    if (!g || !dims) return fail(TG_E_ARG, "tg_shape: NULL argument");
    if (!valid_id(g->g, id)) return fail(TG_E_ARG, "tg_shape: unknown DS id");
    for (int i = 0; i < 4; ++i) dims[i] = g->g.ds[id].d[i];
    return TG_OK;
}

// find_edges(Image, Kernel, num_orientations, Combine_op): orientations at
// 0 and 90 degrees are convolutions with the kernel and its rot90 (precomputed host data,
// the 2 x 256 kernel floats of Table 1), 180 and 270 degrees are remaps.
// Kernel rotated counter-clockwise by `deg` about its centre: multiples of 90 degrees are exact
// index permutations (90: R[i][j] = K[j][k-1-i], as numpy.rot90); other angles sample K
// bilinearly at the rotated position (zero outside) -- DESIGN.md reading R18.
static std::vector<float> rotate_kernel(const float* K, int64_t k, int deg) {
    std::vector<float> r(k * k, 0.f);
    deg = ((deg % 360) + 360) % 360;
    if (deg % 90 == 0) {
        for (int64_t i = 0; i < k; ++i)
            for (int64_t j = 0; j < k; ++j) {
                int64_t si = i, sj = j;
                for (int q = 0; q < deg / 90; ++q) {  // apply rot90 q times
                    const int64_t ti = sj, tj = k - 1 - si;
                    si = ti;
                    sj = tj;
                }
                r[i * k + j] = K[si * k + sj];
            }
        return r;
    }
    const double th = deg * 3.14159265358979323846 / 180.0, c0 = (k - 1) / 2.0;
    const double cs = std::cos(th), sn = std::sin(th);
    for (int64_t i = 0; i < k; ++i)
        for (int64_t j = 0; j < k; ++j) {
            const double y = i - c0, x = j - c0;
            const double sr = c0 + y * cs + x * sn, sc = c0 - y * sn + x * cs;
            const int64_t r0 = (int64_t)std::floor(sr), q0 = (int64_t)std::floor(sc);
            const double fr = sr - r0, fc = sc - q0;
            double v = 0.0;
            for (int dr = 0; dr < 2; ++dr)
                for (int dc = 0; dc < 2; ++dc) {
                    const int64_t rr = r0 + dr, cc = q0 + dc;
                    if (rr < 0 || rr >= k || cc < 0 || cc >= k) continue;
                    v += (dr ? fr : 1 - fr) * (dc ? fc : 1 - fc) * K[rr * k + cc];
                }
            r[i * k + j] = (float)v;
        }
    return r;
}

// find_edges(Image, Kernel, num_orientations, Combine_op): orientations are
// rotations of the filter in steps of 360/num_orientations degrees; the first half are
// convolutions with the rotated kernel (precomputed host data, the kernel floats of Table 1),
// the second half are remaps (negations) of the first. Combine: TG_MAX over
// all orientations, TG_MAXABS = max |response| of the convolutions, TG_SUM = sum of the
// convolutions' responses (adding the remaps would cancel them).
tg_status tg_find_edges(tg_graph* g, tg_id img, tg_id kernel, int32_t num_orientations,
                        int32_t combine_op, tg_id* edge_map) {
    if (!g || !edge_map) return fail(TG_E_ARG, "tg_find_edges: NULL argument");
    Graph& G = g->g;
    if (!valid_id(G, img) || !valid_id(G, kernel)) return fail(TG_E_ARG, "tg_find_edges: unknown DS id");
    if (num_orientations != 2 && num_orientations != 4 && num_orientations != 8)
        return fail(TG_E_ARG, "tg_find_edges: num_orientations must be 2, 4 or 8");
    if (combine_op != TG_MAX && combine_op != TG_SUM && combine_op != TG_MAXABS)
        return fail(TG_E_ARG, "tg_find_edges: combine_op must be TG_MAX, TG_SUM or TG_MAXABS");
    const Ds& K = G.ds[kernel];
    if (K.kind != DsKind::Param || K.d[0] != 1 || K.d[1] != 1 || K.d[2] != K.d[3])
        return fail(TG_E_SHAPE, "tg_find_edges: kernel must be a square [1][1][k][k] parameter");
    if (G.ds[img].d[1] != 1) return fail(TG_E_SHAPE, "tg_find_edges: image must have one plane");
    if (K.src_loc != Loc::Host) return fail(TG_E_ARG, "tg_find_edges: kernel must be host data");
    TG_GUARD_BEGIN
    const int64_t k = K.d[2];
    const int nconv = num_orientations / 2, step = 360 / num_orientations;
    std::vector<tg_id> resp;
    tg_status st;
    for (int f = 0; f < nconv; ++f) {
        tg_id kid = kernel;
        if (f > 0) {
            int64_t d[4] = {1, 1, k, k};
            kid = add_ds(G, d, DsKind::Param);
            G.ds[kid].owned = rotate_kernel(G.ds[kernel].src, k, f * step);
            G.ds[kid].src = G.ds[kid].owned.data();
            G.ds[kid].src_loc = Loc::Host;
        }
        tg_id e;
        if ((st = tg_conv2d(g, img, kid, -1, TG_SAME, &e)) != TG_OK) return st;
        resp.push_back(e);
    }
    tg_id out;
    if (combine_op == TG_SUM) {
        if ((st = tg_elementwise(g, TG_ADD, resp.data(), (int32_t)resp.size(), 1.f, 0.f, &out)) != TG_OK) return st;
    } else if (combine_op == TG_MAXABS) {
        std::vector<tg_id> ab;
        for (tg_id e : resp) {
            tg_id a;
            if ((st = tg_elementwise(g, TG_ABS, &e, 1, 0.f, 0.f, &a)) != TG_OK) return st;
            ab.push_back(a);
        }
        if ((st = tg_max_combine(g, ab.data(), (int32_t)ab.size(), &out)) != TG_OK) return st;
    } else {
        std::vector<tg_id> all = resp;
        for (tg_id e : resp) {
            tg_id r;
            if ((st = tg_elementwise(g, TG_NEG, &e, 1, 0.f, 0.f, &r)) != TG_OK) return st;
            all.push_back(r);
        }
        if ((st = tg_max_combine(g, all.data(), (int32_t)all.size(), &out)) != TG_OK) return st;
    }
    *edge_map = out;
    return TG_OK;
    TG_GUARD_END
}

// CNN template (4 convolutional, 2 sub-sampling and 5 tanh layers; layer
// widths and kernel sizes as reconstructed in SURVEY F2).
tg_status tg_cnn(tg_graph* g, tg_id img, int32_t n5, const tg_id params[10], int32_t bias_mode,
                 tg_id* out) {
    if (!g || !params || !out) return fail(TG_E_ARG, "tg_cnn: NULL argument");
    if (n5 < 1 || n5 > 128) return fail(TG_E_ARG, "tg_cnn: n5 must be in [1, 128]");
    if (bias_mode != TG_BIAS_PLANE && bias_mode != TG_BIAS_SCALAR) return fail(TG_E_ARG, "tg_cnn: bad bias mode");
    tg_id x = img, y;
    tg_status st;
    auto conv = [&](int ki, int bi) -> tg_status {
        st = tg_conv2d(g, x, params[ki], params[bi], TG_VALID, &y);
        x = y;
        return st;
    };
    auto tanh_ = [&]() -> tg_status {
        st = tg_tanh(g, x, &y);
        x = y;
        return st;
    };
    auto sub = [&](int pi) -> tg_status {
        st = tg_subsample(g, x, params[pi], 2, &y);
        x = y;
        return st;
    };
    if ((st = conv(0, 1)) || (st = tanh_()) || (st = sub(2)) || (st = tanh_()) || (st = conv(3, 4)) ||
        (st = tanh_()) || (st = sub(5)) || (st = tanh_()) || (st = conv(6, 7)) || (st = tanh_()) ||
        (st = conv(8, 9)))
        return st;
    *out = x;
    return TG_OK;
}

tg_status tg_set_devices(tg_graph* g, const int32_t* ordinals, int32_t n) {
    if (!g || !ordinals || n <= 0 || n > 8) return fail(TG_E_ARG, "tg_set_devices: 1..8 devices");
    g->g.devices.assign(ordinals, ordinals + n);
    return TG_OK;
}

tg_status tg_set_device_budget(tg_graph* g, uint64_t bytes) {
    if (!g) return fail(TG_E_ARG, "tg_set_device_budget: NULL graph");
    g->g.budget = bytes;
    return TG_OK;
}

tg_status tg_set_precision(tg_graph* g, int32_t prec) {
    if (!g || (prec != TG_FP32 && prec != TG_BF16_TC && prec != TG_FP32_TC))
        return fail(TG_E_ARG, "tg_set_precision: bad precision");
    g->g.precision = prec;
    return TG_OK;
}

tg_status tg_set_chunking(tg_graph* g, int64_t max_chunk_px, int32_t depth) {
    if (!g || max_chunk_px <= 0 || depth < 1 || depth > 8) return fail(TG_E_ARG, "tg_set_chunking: bad argument");
    g->g.max_chunk_px = max_chunk_px;
    g->g.depth = depth;
    return TG_OK;
}

tg_status tg_set_shard(tg_graph* g, int32_t rank, int32_t world) {
    if (!g || world < 1 || rank < 0 || rank >= world) return fail(TG_E_ARG, "tg_set_shard: need 0 <= rank < world");
    g->g.rank = rank;
    g->g.world = world;
    return TG_OK;
}

tg_status tg_set_runtime(tg_graph* g, const tg_runtime* rt) {
    if (!g) return fail(TG_E_ARG, "tg_set_runtime: NULL graph");
    if (rt) {
        g->g.rt = *rt;
        g->g.has_rt = true;
    } else {
        g->g.rt = tg_runtime{};
        g->g.has_rt = false;
    }
    return TG_OK;
}

tg_status tg_plan_create(const tg_graph* g, int32_t mode, tg_plan** plan) {
    if (!g || !plan) return fail(TG_E_ARG, "tg_plan_create: NULL argument");
    if (mode != TG_FUSED && mode != TG_PER_OP && mode != TG_BASELINE)
        return fail(TG_E_ARG, "tg_plan_create: mode must be TG_FUSED, TG_PER_OP or TG_BASELINE");
    TG_GUARD_BEGIN
    auto* p = new tg_plan();
    p->graph = g;
    tg_status st = mode == TG_FUSED ? make_plan(g->g, mode, p->core) : make_plan_per_op(g->g, mode, p->core);
    if (st != TG_OK) {
        delete p;
        return st;
    }
    *plan = p;
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_plan_stats_get(const tg_plan* p, tg_plan_stats* out) {
    if (!p || !out) return fail(TG_E_ARG, "tg_plan_stats_get: NULL argument");
    std::memset(out, 0, sizeof(*out));
    const PlanCore& c = p->core;
    out->h2d_bytes = c.h2d;
    out->d2h_bytes = c.d2h;
    out->io_lower_bound_bytes = c.io_lb;
    out->total_temp_bytes = c.total;
    const size_t nd = p->graph->g.devices.empty() ? 1 : p->graph->g.devices.size();
    for (size_t i = 0; i < nd && i < 8; ++i) out->peak_device_bytes[i] = c.arena_bytes;
    out->n_chunks = (int64_t)c.chunks.size();
    out->n_units = c.n_units;
    out->n_ops_fig7 = c.nops;
    out->n_ds_fig7 = c.nds;
    out->chunk_begin = c.c0;
    out->chunk_end = c.c1;
    out->host_registered_bytes = exec_registered_bytes(p);
    // steady state: parameters stay resident after the first execution
    out->h2d_bytes_steady = c.device_io ? 0 : (c.mode == TG_FUSED ? c.h2d_chunk : c.h2d);
    out->io_lower_bound_data_bytes = c.mode == TG_FUSED ? c.io_lb_data : c.io_lb;
    return TG_OK;
}

tg_status tg_plan_dump_json(const tg_plan* p, char* buf, size_t cap, size_t* needed) {
    if (!p) return fail(TG_E_ARG, "tg_plan_dump_json: NULL plan");
    TG_GUARD_BEGIN
    std::string s = plan_json(p->core);
    if (needed) *needed = s.size() + 1;
    if (!buf || cap < s.size() + 1) return fail(TG_E_ARG, "tg_plan_dump_json: buffer too small");
    std::memcpy(buf, s.c_str(), s.size() + 1);
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_plan_codegen(const tg_plan* p, char* buf, size_t cap, size_t* needed) {
    if (!p) return fail(TG_E_ARG, "tg_plan_codegen: NULL plan");
    if (p->core.mode == TG_FUSED)
        return fail(TG_E_UNSUPPORTED, "tg_plan_codegen: generates TG_PER_OP / TG_BASELINE plans");
    TG_GUARD_BEGIN
    std::string s = plan_codegen(p);
    if (s.empty()) return fail(TG_E_STATE, "tg_plan_codegen: inconsistent plan");
    if (needed) *needed = s.size() + 1;
    if (!buf || cap < s.size() + 1) return fail(TG_E_ARG, "tg_plan_codegen: buffer too small");
    std::memcpy(buf, s.c_str(), s.size() + 1);
    return TG_OK;
    TG_GUARD_END
}

tg_status tg_execute(tg_plan* p) {
    if (!p) return fail(TG_E_ARG, "tg_execute: NULL plan");
    TG_GUARD_BEGIN
    if (p->core.mode != TG_FUSED) return exec_run_per_op(p, true);
    return exec_run(p, true);
    TG_GUARD_END
}

tg_status tg_execute_async(tg_plan* p) {
    if (!p) return fail(TG_E_ARG, "tg_execute_async: NULL plan");
    TG_GUARD_BEGIN
    if (p->core.mode != TG_FUSED) return exec_run_per_op(p, false);
    return exec_run(p, false);
    TG_GUARD_END
}

tg_status tg_execute_on(tg_plan* p, void* stream, int32_t blocking) {
    if (!p) return fail(TG_E_ARG, "tg_execute_on: NULL plan");
    TG_GUARD_BEGIN
    if (p->core.mode != TG_FUSED) return fail(TG_E_UNSUPPORTED, "tg_execute_on: fused plans only");
    return exec_run(p, blocking != 0, stream, true);
    TG_GUARD_END
}

tg_status tg_plan_set_graph(tg_plan* p, int32_t on) {
    if (!p) return fail(TG_E_ARG, "tg_plan_set_graph: NULL plan");
    if (p->core.mode != TG_FUSED) return fail(TG_E_UNSUPPORTED, "tg_plan_set_graph: fused plans only");
    TG_GUARD_BEGIN
    return exec_set_graph(p, on != 0);
    TG_GUARD_END
}

tg_status tg_plan_set_profiling(tg_plan* p, int32_t on) {
    if (!p) return fail(TG_E_ARG, "tg_plan_set_profiling: NULL plan");
    TG_GUARD_BEGIN
    if (p->core.mode != TG_FUSED) {
        exec_set_profiling_per_op(p, on != 0);
        return TG_OK;
    }
    return exec_set_profiling(p, on);
    TG_GUARD_END
}

tg_status tg_plan_timing_get(tg_plan* p, tg_timing* out) {
    if (!p || !out) return fail(TG_E_ARG, "tg_plan_timing_get: NULL argument");
    TG_GUARD_BEGIN
    if (p->core.mode != TG_FUSED) return exec_timing_per_op(p, out);
    return exec_timing(p, out);
    TG_GUARD_END
}

tg_status tg_plan_trace_get(tg_plan* p, tg_trace_rec* out, size_t cap, size_t* n) {
    if (!p || !n || (cap && !out)) return fail(TG_E_ARG, "tg_plan_trace_get: NULL argument");
    TG_GUARD_BEGIN
    if (p->core.mode != TG_FUSED) return fail(TG_E_UNSUPPORTED, "tg_plan_trace_get: fused plans only");
    return exec_trace(p, out, cap, n);
    TG_GUARD_END
}

int64_t tg_plan_launch_count(const tg_plan* p) { return p ? p->launches : 0; }

tg_status tg_plan_invalidate_params(tg_plan* p) {
    if (!p) return fail(TG_E_ARG, "tg_plan_invalidate_params: NULL plan");
    exec_invalidate_params(p);
    return TG_OK;
}

void tg_plan_destroy(tg_plan* p) {
    if (!p) return;
    exec_destroy(p);
    exec_destroy_per_op(p);
    delete p;
}

}  // extern "C"
