// planner.cpp -- offload-unit recognition, operator splitting into halo-correct chunks,
// chunk schedule, sharding and byte accounting (pure host code, no CUDA calls).
//
// Paper steps: represent the template as a parallel operator graph; split
// operators whose footprint exceeds GPU memory, with the input extents
// of every split piece inferred "by traversing the split graph from the leaves to the root"
// (PAPER.md:367); partition the graph into offload units; schedule offloads
// and transfers to minimise host<->GPU bytes.
//
// B200 design ("Offload units"): the whole edge template is ONE
// offload unit (the paper's "best possible"); the CNN is three units
// U1 = C1 T S2 T, U2 = C3 T S4 T, U3 = C5 T C6. Chunks are row bands (or whole-image
// batches) sized so that `depth` chunks are in flight (H2D / compute / D2H) within the
// budget. The rule is restated in oracle/planner.py::fused_plan and the two must agree
// bit-exactly (tests/test_plan_parity.py).
#include <algorithm>
#include <cstdio>
#include <sstream>

#include "kernels/kernels.h"
#include "tg_internal.h"

namespace tg {

static uint64_t a256(uint64_t x) { return (x + 255) / 256 * 256; }

// ----------------------------------------------------------------------------- recognition
static const Node* producer(const Graph& g, int ds) {
    if (ds < 0 || ds >= (int)g.ds.size() || g.ds[ds].producer < 0) return nullptr;
    return &g.nodes[g.ds[ds].producer];
}

static bool is_same_conv_1ch(const Graph& g, const Node* n) {
    if (!n || n->op != OpKind::Conv || n->pad != TG_SAME || n->bias != -1) return false;
    const Ds& K = g.ds[n->ins[1]];
    return K.d[0] == 1 && K.d[1] == 1 && K.d[2] == K.d[3] && K.d[2] >= 1 && K.d[2] <= 16;
}

// Edge template (Fig. 1(b)): 1..4 SAME convolutions of one image combined by
//   max over the responses and their remaps (negations)   [combine 0, the paper's template]
//   sum of the responses                                   [combine 1, "addition"]
//   max of |response|                                      [combine 2, "max absolute value"]
//   max of the responses                                   [combine 3]
static tg_status recognise_edge(const Graph& g, int out, Template& t) {
    const Node* top = producer(g, out);
    if (!top) return TG_E_UNSUPPORTED;
    const bool is_max = top->op == OpKind::Max;
    const bool is_sum = top->op == OpKind::Elem && top->elem == TG_ADD;
    if (!is_max && !is_sum) return TG_E_UNSUPPORTED;
    std::vector<const Node*> convs;
    std::vector<int> conv_out, negated, absed;
    for (int x : top->ins) {
        const Node* p = producer(g, x);
        if (is_same_conv_1ch(g, p)) {
            convs.push_back(p);
            conv_out.push_back(x);
        } else if (p && p->op == OpKind::Elem && p->elem == TG_NEG) {
            negated.push_back(p->ins[0]);
        } else if (p && p->op == OpKind::Elem && p->elem == TG_ABS) {
            absed.push_back(p->ins[0]);
        } else {
            return TG_E_UNSUPPORTED;
        }
    }
    int combine;
    if (is_sum) {
        if (!negated.empty() || !absed.empty()) return TG_E_UNSUPPORTED;
        combine = 1;
    } else if (!absed.empty()) {
        if (!convs.empty() || !negated.empty()) return TG_E_UNSUPPORTED;
        for (int x : absed) {
            const Node* p = producer(g, x);
            if (!is_same_conv_1ch(g, p)) return TG_E_UNSUPPORTED;
            convs.push_back(p);
            conv_out.push_back(x);
        }
        combine = 2;
    } else if (!negated.empty()) {
        // the remaps must negate exactly the convolution outputs (each once)
        std::vector<int> a = negated, b = conv_out;
        std::sort(a.begin(), a.end());
        std::sort(b.begin(), b.end());
        if (a != b || std::adjacent_find(a.begin(), a.end()) != a.end()) return TG_E_UNSUPPORTED;
        combine = 0;
    } else {
        combine = 3;
    }
    if (convs.empty() || convs.size() > 4) return TG_E_UNSUPPORTED;
    const int x = convs[0]->ins[0];
    const Ds& X = g.ds[x];
    if (X.kind != DsKind::Input || X.d[1] != 1) return TG_E_UNSUPPORTED;
    for (const Node* c : convs)
        if (c->ins[0] != x || g.ds[c->ins[1]].d[2] != g.ds[convs[0]->ins[1]].d[2]) return TG_E_UNSUPPORTED;
    t.kind = Tmpl::Edge;
    t.input = x;
    t.output = out;
    t.n = X.d[0];
    t.H = X.d[2];
    t.W = X.d[3];
    t.ks = (int)g.ds[convs[0]->ins[1]].d[2];
    t.nf = (int)convs.size();
    t.combine = combine;
    for (int f = 0; f < t.nf; ++f) t.kk[f] = convs[f]->ins[1];
    t.k1 = t.kk[0];
    t.k2 = t.nf > 1 ? t.kk[1] : -1;
    return TG_OK;
}

static tg_status recognise_cnn(const Graph& g, int out, Template& t) {
    // walk back: C6 T5 C5 T4 S4 T3 C3 T2 S2 T1 C1 <- input
    const OpKind want[11] = {OpKind::Conv, OpKind::Tanh, OpKind::Conv, OpKind::Tanh, OpKind::Sub, OpKind::Tanh,
                             OpKind::Conv, OpKind::Tanh, OpKind::Sub, OpKind::Tanh, OpKind::Conv};
    const Node* chain[11];
    int cur = out;
    for (int i = 0; i < 11; ++i) {
        const Node* p = producer(g, cur);
        if (!p || p->op != want[i]) return TG_E_UNSUPPORTED;
        chain[i] = p;
        cur = p->ins[0];
    }
    const Ds& X = g.ds[cur];
    if (X.kind != DsKind::Input || X.d[1] != 1) return TG_E_UNSUPPORTED;
    const Node *c6 = chain[0], *c5 = chain[2], *s4 = chain[4], *c3 = chain[6], *s2 = chain[8], *c1 = chain[10];
    auto kd = [&](const Node* n, int i) { return g.ds[n->ins[1]].d[i]; };
    for (const Node* c : {c1, c3, c5, c6})
        if (c->pad != TG_VALID || c->bias < 0) return TG_E_UNSUPPORTED;
    if (kd(c1, 0) != 8 || kd(c1, 1) != 1 || kd(c1, 2) != 5 || kd(c1, 3) != 5) return TG_E_UNSUPPORTED;
    if (kd(c3, 0) != 20 || kd(c3, 1) != 8 || kd(c3, 2) != 5 || kd(c3, 3) != 5) return TG_E_UNSUPPORTED;
    const int64_t n5 = kd(c5, 0);
    if (n5 < 1 || n5 > 128 || kd(c5, 1) != 20 || kd(c5, 2) != 5 || kd(c5, 3) != 5) return TG_E_UNSUPPORTED;
    if (kd(c6, 0) != 9 || kd(c6, 1) != n5 || kd(c6, 2) != 1 || kd(c6, 3) != 1) return TG_E_UNSUPPORTED;
    if (s2->s != 2 || s4->s != 2) return TG_E_UNSUPPORTED;
    // bias kind must be uniform: all planes [1][co][ho][wo] or all scalars [co] (a 1x1 plane
    // is both)
    int plane_ok = 0, scalar_ok = 0;
    for (const Node* c : {c1, c3, c5, c6}) {
        const Ds& B = g.ds[c->bias];
        const Ds& O = g.ds[c->out];
        plane_ok += (B.d[0] == 1 && B.d[1] == O.d[1] && B.d[2] == O.d[2] && B.d[3] == O.d[3]) ? 1 : 0;
        scalar_ok += (B.numel() == O.d[1]) ? 1 : 0;
    }
    if (plane_ok != 4 && scalar_ok != 4) return TG_E_UNSUPPORTED;
    const int planes = plane_ok == 4 ? 4 : 0;
    t.kind = Tmpl::Cnn;
    t.input = cur;
    t.output = out;
    t.n = X.d[0];
    t.H = X.d[2];
    t.W = X.d[3];
    t.n5 = (int)n5;
    t.bias_plane = planes == 4;
    const int prm[10] = {c1->ins[1], c1->bias, s2->ins[1], c3->ins[1], c3->bias,
                         s4->ins[1], c5->ins[1], c5->bias, c6->ins[1], c6->bias};
    for (int i = 0; i < 10; ++i) t.prm[i] = prm[i];
    t.h[0] = t.H;
    t.w[0] = t.W;
    t.h[1] = t.H - 4;
    t.w[1] = t.W - 4;
    t.h[2] = (t.h[1] - 2) / 2 + 1;
    t.w[2] = (t.w[1] - 2) / 2 + 1;
    t.h[3] = t.h[2] - 4;
    t.w[3] = t.w[2] - 4;
    t.h[4] = (t.h[3] - 2) / 2 + 1;
    t.w[4] = (t.w[3] - 2) / 2 + 1;
    t.h[5] = t.h[4] - 4;
    t.w[5] = t.w[4] - 4;
    if (t.h[5] <= 0 || t.w[5] <= 0) return TG_E_SHAPE;
    return TG_OK;
}

tg_status recognise(const Graph& g, Template& t) {
    int out = -1, nout = 0;
    for (int i = 0; i < (int)g.ds.size(); ++i)
        if (g.ds[i].dst) {
            out = i;
            ++nout;
        }
    if (nout != 1) return fail(TG_E_STATE, "plan: bind exactly one template output with tg_output/tg_output_device");
    if (recognise_edge(g, out, t) == TG_OK) return TG_OK;
    tg_status st = recognise_cnn(g, out, t);
    if (st == TG_OK) return TG_OK;
    if (st == TG_E_SHAPE) return fail(TG_E_SHAPE, "plan: image too small for the CNN template");
    return fail(TG_E_UNSUPPORTED,
                "plan: TG_FUSED recognises the edge template (2 SAME convs, 2 remaps, 4-way max) and the "
                "11-layer CNN template; other graphs need TG_PER_OP (not in this round)");
}

// ----------------------------------------------------------------------------- halos
// Walk a chain of row-local operators from the output band back to the input
// (PAPER.md:367). kinds: 'v' VALID conv (p = k), 's' SAME conv (p = k, clipped to [0,H)),
// 'u' subsample (p = window = stride), 'e' elementwise.
struct LayerRule {
    char kind;
    int64_t p;
};

static std::vector<RowRange> back_propagate(const std::vector<LayerRule>& layers, int64_t r0, int64_t r1,
                                            int64_t H_in) {
    std::vector<RowRange> ranges(layers.size() + 1);
    int64_t a = r0, b = r1;
    ranges[layers.size()] = {a, b};
    for (int i = (int)layers.size() - 1; i >= 0; --i) {
        const LayerRule& L = layers[i];
        switch (L.kind) {
            case 'v': b = b + L.p - 1; break;
            case 's':
                a = std::max<int64_t>(0, a - (L.p - 1) / 2);
                b = std::min<int64_t>(H_in, b + L.p / 2);
                break;
            case 'u':
                a = L.p * a;
                b = L.p * b;
                break;
            default: break;
        }
        ranges[i] = {a, b};
    }
    return ranges;
}

static const std::vector<LayerRule> kCnnLayers = {{'v', 5}, {'e', 0}, {'u', 2}, {'e', 0}, {'v', 5}, {'e', 0},
                                                  {'u', 2}, {'e', 0}, {'v', 5}, {'e', 0}, {'v', 1}};

static Chunk rows_of(const Template& t, int64_t img, int64_t nimg, int64_t r0, int64_t r1) {
    Chunk c;
    c.img = img;
    c.nimg = nimg;
    if (t.kind == Tmpl::Edge) {
        auto rg = back_propagate({{'s', t.ks}}, r0, r1, t.H);
        c.in = rg[0];
        c.out = rg[1];
    } else {
        auto rg = back_propagate(kCnnLayers, r0, r1, t.H);
        // levels: 0 in, 1 C1, 2 T1, 3 S2, 4 T2, 5 C3, 6 T3, 7 S4, 8 T4, 9 C5, 10 T5, 11 C6
        c.in = rg[0];
        c.c1 = rg[1];
        c.t2 = rg[4];
        c.c3 = rg[5];
        c.t4 = rg[8];
        c.out = rg[11];
    }
    return c;
}

// ----------------------------------------------------------------------------- chunk rule
namespace {
struct Sizer {
    const Template& t;
    bool device_io;
    int64_t n5;
    uint64_t t4_words;  // 4-byte words per T4 pixel: 20 (fp32 planes; bf16 blocks fit), 24 for
                        // TG_FP32_TC (2 fp16 parts x 3 blocks of 8 channels)
    // slot layout for B images x R output rows with the given row ranges
    SlotLayout slot(int64_t B, int64_t R, const Chunk& rg, bool streamed) const {
        SlotLayout s;
        uint64_t off = 0;
        auto put = [&](uint64_t& field, uint64_t bytes) {
            field = off;
            off += a256(bytes);
        };
        const uint64_t f = 4;
        if (!device_io) put(s.in, (uint64_t)B * rg.in.n() * t.W * f);
        if (t.kind == Tmpl::Cnn) {
            put(s.t2, (uint64_t)B * 8 * rg.t2.n() * t.w[2] * f);
            put(s.t4, (uint64_t)B * t4_words * rg.t4.n() * t.w[4] * f);
            if (!device_io) put(s.out, (uint64_t)B * 9 * R * t.w[5] * f);
            if (streamed) {
                put(s.b1, (uint64_t)8 * rg.c1.n() * t.w[1] * f);
                put(s.b3, (uint64_t)20 * rg.c3.n() * t.w[3] * f);
                put(s.b5, (uint64_t)n5 * R * t.w[5] * f);
                put(s.b6, (uint64_t)9 * R * t.w[5] * f);
            }
        } else if (!device_io) {
            put(s.out, (uint64_t)B * R * t.W * f);
        }
        s.bytes = off;
        return s;
    }
    Chunk widest(int64_t R) const {
        if (t.kind == Tmpl::Edge) {
            Chunk c;
            c.in = {0, std::min<int64_t>(t.H, R + t.ks - 1)};
            c.out = {0, R};
            return c;
        }
        return rows_of(t, 0, 1, 0, R);
    }
};
}  // namespace

tg_status make_plan(const Graph& g, int32_t mode, PlanCore& p) {
    tg_status st = recognise(g, p.t);
    if (st != TG_OK) return st;
    const Template& t = p.t;
    p.mode = mode;
    p.precision = g.precision;
    p.budget = g.budget;
    p.max_chunk_px = g.max_chunk_px;
    p.depth = g.depth;
    const Ds& X = g.ds[t.input];
    const Ds& Y = g.ds[t.output];
    p.device_io = X.src_loc == Loc::Device && Y.dst_loc == Loc::Device;
    if ((X.src_loc == Loc::Device) != (Y.dst_loc == Loc::Device))
        return fail(TG_E_UNSUPPORTED, "plan: input and output must both be host or both be device resident");
    if (p.device_io) {
        // device-resident buffers live on ONE device: every device thread would dereference them
        for (size_t i = 1; i < g.devices.size(); ++i)
            if (g.devices[i] != g.devices[0])
                return fail(TG_E_UNSUPPORTED, "plan: device-resident I/O needs a one-device plan (tg_set_devices)");
    }
    const uint64_t f = 4;
    const int64_t H = t.H, W = t.W, n = t.n;
    const int64_t h_out = t.kind == Tmpl::Edge ? H : t.h[5];
    const int64_t w_out = t.kind == Tmpl::Edge ? W : t.w[5];
    const int64_t in_per_out = t.kind == Tmpl::Edge ? 1 : 4;

    // parameters in template order, and which are bias planes
    std::vector<int> prm;
    std::vector<bool> is_bias;
    if (t.kind == Tmpl::Edge) {
        prm.assign(t.kk, t.kk + t.nf);
        is_bias.assign(t.nf, false);
    } else {
        prm.assign(t.prm, t.prm + 10);
        is_bias = {false, true, false, false, true, false, false, true, false, true};
    }
    uint64_t all_pb = 0, nonbias_pb = 0;
    for (size_t i = 0; i < prm.size(); ++i) {
        const uint64_t b = a256((uint64_t)g.ds[prm[i]].numel() * f);
        all_pb += b;
        if (!is_bias[i]) nonbias_pb += b;
    }
    // tensor-core path: bf16 B operands of C3 and C5 prepared once and kept with the params
    uint64_t tc_bytes = 0;
    if (t.kind == Tmpl::Cnn && g.precision == TG_BF16_TC) {
        tc_bytes = a256(cnn_k3_tc_bytes()) + a256(cnn_k5_tc_bytes(t.n5));
        all_pb += tc_bytes;
        nonbias_pb += tc_bytes;
    }
    // 3xFP16 path: the fp16-split B operands of C3 and C5, kept with the parameters
    if (t.kind == Tmpl::Cnn && g.precision == TG_FP32_TC) {
        tc_bytes = a256(cnn_k3_h3_bytes()) + a256(cnn_k5_h3_bytes(t.n5));
        all_pb += tc_bytes;
        nonbias_pb += tc_bytes;
    }
    int32_t depth = p.device_io ? 1 : g.depth;
    p.depth = depth;
    Sizer sz{t, p.device_io, t.n5, (uint64_t)(t.kind == Tmpl::Cnn && g.precision == TG_FP32_TC ? 24 : 20)};
    auto fits = [&](uint64_t pb, uint64_t sb) { return g.budget == 0 || pb + (uint64_t)depth * sb <= g.budget; };

    auto chunk_list = [&](bool batch, int64_t B, int64_t R) {
        std::vector<Chunk> out;
        if (batch) {
            for (int64_t b0 = 0; b0 < n; b0 += B) out.push_back(rows_of(t, b0, std::min(B, n - b0), 0, h_out));
        } else {
            for (int64_t b0 = 0; b0 < n; ++b0)
                for (int64_t r0 = 0; r0 < h_out; r0 += R) out.push_back(rows_of(t, b0, 1, r0, std::min(h_out, r0 + R)));
        }
        return out;
    };
    // exact bytes the parameter uploads move (resident parameters; streamed bias planes travel
    // with the chunks) and the tensor-core operands derived from them
    uint64_t all_pexact = 0, nonbias_pexact = 0;
    for (size_t i = 0; i < prm.size(); ++i) {
        const uint64_t b = (uint64_t)g.ds[prm[i]].numel() * f;
        all_pexact += b;
        if (!is_bias[i]) nonbias_pexact += b;
    }
    uint64_t derived_exact = 0;
    if (t.kind == Tmpl::Cnn && g.precision == TG_BF16_TC) derived_exact = cnn_k3_tc_bytes() + cnn_k5_tc_bytes(t.n5);
    if (t.kind == Tmpl::Cnn && g.precision == TG_FP32_TC) derived_exact = cnn_k3_h3_bytes() + cnn_k5_h3_bytes(t.n5);
    auto chunk_h2d = [&](const std::vector<Chunk>& cs, size_t c0, size_t c1, bool streamed) -> uint64_t {
        if (p.device_io) return 0;
        uint64_t s = 0;
        for (size_t i = c0; i < c1; ++i) {
            const Chunk& c = cs[i];
            s += (uint64_t)c.nimg * c.in.n() * W * f;
            if (streamed) {
                s += (uint64_t)8 * c.c1.n() * t.w[1] * f + (uint64_t)20 * c.c3.n() * t.w[3] * f;
                s += (uint64_t)(t.n5 + 9) * c.out.n() * t.w[5] * f;
            }
        }
        return s;
    };
    auto h2d_of = [&](const std::vector<Chunk>& cs, size_t c0, size_t c1, bool streamed) -> uint64_t {
        if (p.device_io) return 0;
        return (streamed ? nonbias_pexact : all_pexact) + derived_exact + chunk_h2d(cs, c0, c1, streamed);
    };

    const std::string base_bias = t.kind == Tmpl::Edge ? "none" : (t.bias_plane ? "resident" : "scalar");
    bool have = false, batch = false, streamed = false;
    int64_t B = 1, R = h_out;
    uint64_t pb = all_pb;
    SlotLayout slot;
    std::string bias_mode = base_bias;
    // 1. batch mode. Host I/O: at least 2 x depth chunks over each shard's share of the images
    // (n_share = ceil(n / world)), so copies of some chunks overlap the kernels of others
    const int64_t n_share = (n + g.world - 1) / g.world;
    int64_t bcap = 0;
    if (p.device_io)
        bcap = n;
    else if (H * W <= g.max_chunk_px)
        bcap = std::min({n, g.max_chunk_px / (H * W), std::max<int64_t>(1, (n_share + 2 * depth - 1) / (2 * depth))});
    for (int64_t b = bcap; b >= 1; --b) {
        SlotLayout s = sz.slot(b, h_out, rows_of(t, 0, b, 0, h_out), false);
        if (fits(all_pb, s.bytes)) {
            have = batch = true;
            B = b;
            R = h_out;
            slot = s;
            p.chunk_cap = bcap;
            p.slot_bytes_next = b < bcap ? sz.slot(b + 1, h_out, rows_of(t, 0, b + 1, 0, h_out), false).bytes : 0;
            break;
        }
    }
    // 2. row mode
    if (!have) {
        // at most max_chunk_px input pixels per chunk, and (host I/O) at least 2 x depth chunks
        // over each shard's images
        int64_t rcap = std::min<int64_t>(h_out, std::max<int64_t>(1, g.max_chunk_px / (W * in_per_out)));
        if (!p.device_io) {
            const int64_t per_img = (2 * depth + n_share - 1) / n_share;  // chunks wanted per image
            rcap = std::min<int64_t>(rcap, (h_out + per_img - 1) / per_img);
        }
        struct Cand {
            uint64_t h2d;
            int64_t R;
            std::string bm;
            uint64_t pb;
            SlotLayout slot;
        };
        std::vector<Cand> cands;
        std::vector<std::string> modes = {base_bias};
        if (base_bias == "resident") modes.push_back("streamed");
        for (const std::string& bm : modes) {
            const bool strm = bm == "streamed";
            const uint64_t pbm = strm ? nonbias_pb : all_pb;
            int64_t lo = 1, hi = rcap, best = 0;
            while (lo <= hi) {  // slot bytes grow monotonically with R
                const int64_t mid = (lo + hi) / 2;
                if (fits(pbm, sz.slot(1, mid, sz.widest(mid), strm).bytes)) {
                    best = mid;
                    lo = mid + 1;
                } else {
                    hi = mid - 1;
                }
            }
            if (best) {
                auto cs = chunk_list(false, 1, best);
                cands.push_back({h2d_of(cs, 0, cs.size(), strm), best, bm, pbm, sz.slot(1, best, sz.widest(best), strm)});
            }
        }
        if (cands.empty()) {
            char msg[256];
            std::snprintf(msg, sizeof msg,
                          "plan: budget %llu B cannot hold %d slots of the smallest chunk (1 output row) plus parameters",
                          (unsigned long long)g.budget, depth);
            return fail(TG_E_INFEASIBLE, msg);
        }
        std::stable_sort(cands.begin(), cands.end(), [](const Cand& a, const Cand& b) { return a.h2d < b.h2d; });
        const Cand& c = cands.front();
        have = true;
        batch = false;
        B = 1;
        R = c.R;
        bias_mode = c.bm;
        pb = c.pb;
        slot = c.slot;
        streamed = c.bm == "streamed";
        p.chunk_cap = rcap;
        p.slot_bytes_next = R < rcap ? sz.slot(1, R + 1, sz.widest(R + 1), streamed).bytes : 0;
    }
    p.split = batch ? "batch" : "rows";
    p.B = B;
    p.R = R;
    p.bias = bias_mode;
    p.param_bytes = pb;
    p.slot = slot;
    p.slot_bytes = slot.bytes;
    p.arena_bytes = pb + (uint64_t)depth * slot.bytes;
    // parameter region layout (streamed bias planes live in the slots instead)
    p.param_ds = prm;
    p.param_off.assign(prm.size(), UINT64_MAX);
    p.param_streamed.assign(prm.size(), false);
    uint64_t off = 0;
    for (size_t i = 0; i < prm.size(); ++i) {
        if (streamed && is_bias[i]) {
            p.param_streamed[i] = true;
            continue;
        }
        p.param_off[i] = off;
        off += a256((uint64_t)g.ds[prm[i]].numel() * f);
    }
    p.k3tc_off = p.k5tc_off = UINT64_MAX;
    if (tc_bytes && g.precision == TG_BF16_TC) {
        p.k3tc_off = off;
        off += a256(cnn_k3_tc_bytes());
        p.k5tc_off = off;
        off += a256(cnn_k5_tc_bytes(t.n5));
    } else if (tc_bytes) {  // TG_FP32_TC
        p.k3tc_off = off;
        off += a256(cnn_k3_h3_bytes());
        p.k5tc_off = off;
        off += a256(cnn_k5_h3_bytes(t.n5));
    }
    p.chunks = chunk_list(batch, B, R);
    const int64_t C = (int64_t)p.chunks.size();
    p.rank = g.rank;
    p.world = g.world;
    p.c0 = (C * g.rank) / g.world;
    p.c1 = (C * (g.rank + 1)) / g.world;
    p.h2d_param = p.device_io ? 0 : (streamed ? nonbias_pexact : all_pexact);
    p.h2d_derived = p.device_io ? 0 : derived_exact;
    p.h2d_chunk = chunk_h2d(p.chunks, p.c0, p.c1, streamed);
    p.h2d = p.h2d_param + p.h2d_derived + p.h2d_chunk;
    p.d2h = 0;
    if (!p.device_io) {
        const int64_t planes_out = t.kind == Tmpl::Cnn ? 9 : 1;
        for (int64_t i = p.c0; i < p.c1; ++i) {
            const Chunk& c = p.chunks[i];
            p.d2h += (uint64_t)c.nimg * planes_out * c.out.n() * w_out * f;
        }
    }
    // Table 1 accounting at Fig. 7 granularity
    uint64_t param_floats = 0;
    for (int id : prm) param_floats += (uint64_t)g.ds[id].numel();
    if (t.kind == Tmpl::Edge) {
        const uint64_t S = (uint64_t)H * W, k = (uint64_t)t.nf;
        // per image: Im, the k responses, k remaps / abs (combine 0, 2), the combined output
        const uint64_t planes = (t.combine == 0 || t.combine == 2) ? 2 * k + 2 : k + 2;
        p.io_lb = ((uint64_t)n * 2 * S + param_floats) * f;
        p.io_lb_data = (uint64_t)n * 2 * S * f;
        p.total = ((uint64_t)n * planes * S + param_floats) * f;  // 4 orientations: Im E1 E2 E5 E6 E
        p.nops = (int64_t)(planes - 1);                            // convolutions (+remaps) + combine
        p.nds = (int64_t)(planes + k);                             // + the k kernels
        p.n_units = 1;
    } else {
        const uint64_t A0 = (uint64_t)H * W, A1 = (uint64_t)t.h[1] * t.w[1], A2 = (uint64_t)t.h[2] * t.w[2],
                       A3 = (uint64_t)t.h[3] * t.w[3], A4 = (uint64_t)t.h[4] * t.w[4], A5 = (uint64_t)t.h[5] * t.w[5];
        const uint64_t n5 = (uint64_t)t.n5;
        // Fig. 7 per layer (n_in -> n_out, c = n_in*n_out pairs): c conv outputs L, c - n_out
        // partial sums S, n_out outputs O; tanh: one output per plane; subsample: one output
        // per plane (parameters counted separately).
        auto conv_temp = [](uint64_t nin, uint64_t nout, uint64_t A) { return (nin * nout + (nin * nout - nout) + nout) * A; };
        const uint64_t per_img = A0 + conv_temp(1, 8, A1) + 8 * A1 + 8 * A2 + 8 * A2 + conv_temp(8, 20, A3) + 20 * A3 +
                                 20 * A4 + 20 * A4 + conv_temp(20, n5, A5) + n5 * A5 + conv_temp(n5, 9, A5);
        p.io_lb = ((uint64_t)n * (A0 + 9 * A5) + param_floats) * f;
        p.io_lb_data = (uint64_t)n * (A0 + 9 * A5) * f;
        p.total = ((uint64_t)n * per_img + param_floats) * f;
        // ops: conv 2c, tanh 1/plane, subsample 1/plane; DS: conv 3c + n_out, tanh 1/plane,
        // subsample 2/plane, plus the input plane
        const uint64_t c1 = 8, c3 = 160, c5 = 20 * n5, c6 = 9 * n5;
        p.nops = (int64_t)(2 * (c1 + c3 + c5 + c6) + 8 + 8 + 8 + 20 + 20 + 20 + n5);
        p.nds = (int64_t)(1 + (3 * c1 + 8) + 8 + 16 + 8 + (3 * c3 + 20) + 20 + 40 + 20 + (3 * c5 + n5) + n5 + (3 * c6 + 9));
        p.n_units = 3;
    }
    return TG_OK;
}

// ----------------------------------------------------------------------------- JSON
static void jrange(std::ostringstream& o, const char* k, const RowRange& r) {
    o << "\"" << k << "\": [" << r.a << ", " << r.b << "]";
}

std::string plan_json(const PlanCore& p) {
    if (p.mode != TG_FUSED) return plan_json_per_op(p);
    const Template& t = p.t;
    std::ostringstream o;
    o << "{";
    o << "\"template\": \"" << (t.kind == Tmpl::Edge ? "edge" : "cnn") << "\", ";
    o << "\"n\": " << t.n << ", \"H\": " << t.H << ", \"W\": " << t.W << ", ";
    o << "\"ks\": " << (t.kind == Tmpl::Edge ? t.ks : 0) << ", \"n5\": " << (t.kind == Tmpl::Cnn ? t.n5 : 0) << ", ";
    static const char* kComb[4] = {"max", "sum", "maxabs", "maxplain"};
    o << "\"nf\": " << (t.kind == Tmpl::Edge ? t.nf : 0) << ", \"combine\": \"" << (t.kind == Tmpl::Edge ? kComb[t.combine] : "none") << "\", ";
    o << "\"budget\": " << p.budget << ", \"depth\": " << p.depth << ", \"max_chunk_px\": " << p.max_chunk_px << ", ";
    o << "\"device_io\": " << (p.device_io ? "true" : "false") << ", ";
    o << "\"precision\": \"" << (t.kind != Tmpl::Cnn ? "fp32" : p.precision == TG_BF16_TC ? "bf16_tc" : p.precision == TG_FP32_TC ? "fp32_tc" : "fp32") << "\", ";
    o << "\"bias\": \"" << p.bias << "\", \"split\": \"" << p.split << "\", ";
    o << "\"B\": " << p.B << ", \"R\": " << p.R << ", ";
    o << "\"param_bytes\": " << p.param_bytes << ", \"slot_bytes\": " << p.slot_bytes
      << ", \"arena_bytes\": " << p.arena_bytes << ", ";
    o << "\"chunk_cap\": " << p.chunk_cap << ", \"slot_bytes_next\": " << p.slot_bytes_next << ", ";
    {  // slot buffers: [offset, end) of each buffer present in this plan's slot
        const SlotLayout& L = p.slot;
        const uint64_t offs[8] = {L.in, L.t2, L.t4, L.out, L.b1, L.b3, L.b5, L.b6};
        const char* names[8] = {"in", "t2", "t4", "out", "b1", "b3", "b5", "b6"};
        const bool cnn = t.kind == Tmpl::Cnn, strm = p.bias == "streamed";
        const bool present[8] = {!p.device_io, cnn, cnn, !p.device_io, strm, strm, strm, strm};
        std::vector<std::pair<uint64_t, int>> ord;
        for (int i = 0; i < 8; ++i)
            if (present[i]) ord.push_back({offs[i], i});
        std::sort(ord.begin(), ord.end());
        o << "\"slot\": {";
        for (size_t k = 0; k < ord.size(); ++k) {
            const uint64_t end = k + 1 < ord.size() ? ord[k + 1].first : p.slot_bytes;
            o << (k ? ", " : "") << "\"" << names[ord[k].second] << "\": [" << ord[k].first << ", " << end << "]";
        }
        o << "}, ";
    }
    o << "\"n_chunks\": " << p.chunks.size() << ", \"chunks\": [";
    for (size_t i = 0; i < p.chunks.size(); ++i) {
        const Chunk& c = p.chunks[i];
        if (i) o << ", ";
        o << "{\"img\": " << c.img << ", \"nimg\": " << c.nimg << ", ";
        jrange(o, "in", c.in);
        o << ", ";
        if (t.kind == Tmpl::Cnn) {
            jrange(o, "c1", c.c1);
            o << ", ";
            jrange(o, "t2", c.t2);
            o << ", ";
            jrange(o, "c3", c.c3);
            o << ", ";
            jrange(o, "t4", c.t4);
            o << ", ";
        }
        jrange(o, "out", c.out);
        o << "}";
    }
    o << "], ";
    o << "\"shard\": [" << p.rank << ", " << p.world << ", " << p.c0 << ", " << p.c1 << "], ";
    o << "\"h2d_bytes\": " << p.h2d << ", \"d2h_bytes\": " << p.d2h << ", ";
    o << "\"h2d_param_bytes\": " << p.h2d_param << ", \"h2d_derived_bytes\": " << p.h2d_derived
      << ", \"h2d_chunk_bytes\": " << p.h2d_chunk << ", ";
    o << "\"io_lower_bound_bytes\": " << p.io_lb << ", \"io_lower_bound_data_bytes\": " << p.io_lb_data
      << ", \"total_temp_bytes\": " << p.total << ", ";
    o << "\"n_ops_fig7\": " << p.nops << ", \"n_ds_fig7\": " << p.nds;
    o << "}";
    return o.str();
}

}  // namespace tg
