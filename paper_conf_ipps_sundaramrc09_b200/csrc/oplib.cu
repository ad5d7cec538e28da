// oplib.cu -- tg_oplib_run: the operator library of Fig. 4 behind the C ABI.
// Validates a tg_oplib_op descriptor (one operator piece, device pointers) and launches the
// generic kernel for it (kernels/generic.cu). The per-operator executor (engine_perop.cu) and
// the generated programs of tg_plan_codegen (codegen.cpp) both run operators through here.
#include <cuda_runtime.h>

#include <string>

#include "kernels/kernels.h"
#include "tg_internal.h"

namespace tg {

static bool to_view(const tg_oplib_view& in, GenView& v) {
    if (in.nseg < 1 || in.nseg > kGenMaxSeg) return false;
    v = GenView{};
    v.nseg = in.nseg;
    for (int i = 0; i < in.nseg; ++i) {
        if (!in.seg[i].p || in.seg[i].r1 < in.seg[i].r0) return false;
        v.seg[i] = GenSeg{in.seg[i].p, in.seg[i].r0, in.seg[i].r1};
    }
    return true;
}

// a whole parameter (kernel, subsample weights): one piece from row 0
static const float* whole(const tg_oplib_view& v, int64_t h) {
    return (v.nseg == 1 && v.seg[0].r0 == 0 && v.seg[0].r1 == h) ? v.seg[0].p : nullptr;
}

tg_status oplib_run(const tg_oplib_op& op, void* stream_) {
    cudaStream_t stream = (cudaStream_t)stream_;
    if (op.nin < 1 || op.nin > TG_OPLIB_MAX_IN || !op.y || op.r1 < op.r0 || op.r0 < 0 || op.r1 > op.y_dims[2])
        return fail(TG_E_ARG, "tg_oplib_run: malformed descriptor");
    if (op.r1 == op.r0) return TG_OK;
    GenView v[TG_OPLIB_MAX_IN];
    for (int i = 0; i < op.nin; ++i)
        if ((op.kind != TG_OPLIB_CONV || i != 1) && (op.kind != TG_OPLIB_SUB || i != 1) && !to_view(op.in[i], v[i]))
            return fail(TG_E_ARG, "tg_oplib_run: bad input view");
    const int64_t* X = op.in_dims[0];
    const int64_t* Y = op.y_dims;
    cudaError_t e = cudaSuccess;
    switch (op.kind) {
        case TG_OPLIB_CONV: {
            if (op.nin < 2 || op.nin > 3) return fail(TG_E_ARG, "tg_oplib_run: conv takes x, kernel[, bias]");
            const int64_t* K = op.in_dims[1];
            GenConvArgs a{};
            a.x = v[0];
            a.k = whole(op.in[1], K[2]);
            if (!a.k) return fail(TG_E_ARG, "tg_oplib_run: the kernel must be one whole piece");
            a.y = op.y;
            a.r0 = op.r0;
            a.r1 = op.r1;
            a.n = X[0];
            a.ci = X[1];
            a.h = X[2];
            a.w = X[3];
            a.co = K[0];
            a.kh = K[2];
            a.kw = K[3];
            a.wo = Y[3];
            a.pt = op.pad == TG_SAME ? (int)(K[2] - 1) / 2 : 0;
            a.pl = op.pad == TG_SAME ? (int)(K[3] - 1) / 2 : 0;
            if (op.nin == 3) {
                a.bias = v[2];
                const int64_t* B = op.in_dims[2];
                a.bias_kind = B[0] * B[1] * B[2] * B[3] == K[0] ? 1 : 2;
            }
            e = launch_gen_conv(a, stream);
            break;
        }
        case TG_OPLIB_SUB: {
            if (op.nin != 2 || op.s < 1) return fail(TG_E_ARG, "tg_oplib_run: subsample takes x, p and s >= 1");
            GenSubArgs a{};
            a.x = v[0];
            a.p = whole(op.in[1], op.in_dims[1][2]);
            if (!a.p) return fail(TG_E_ARG, "tg_oplib_run: subsample weights must be one whole piece");
            a.y = op.y;
            a.r0 = op.r0;
            a.r1 = op.r1;
            a.n = X[0];
            a.c = X[1];
            a.h = X[2];
            a.w = X[3];
            a.wo = Y[3];
            a.s = op.s;
            e = launch_gen_sub(a, stream);
            break;
        }
        case TG_OPLIB_MATMUL: {
            if (op.nin != 2) return fail(TG_E_ARG, "tg_oplib_run: matmul takes a, b");
            GenMatmulArgs a{};
            a.a = v[0];
            a.b = v[1];
            a.c = op.y;
            a.r0 = op.r0;
            a.r1 = op.r1;
            a.k = X[3];
            a.n = Y[3];
            e = launch_gen_matmul(a, stream);
            break;
        }
        case TG_OPLIB_ELEM: {
            if (op.elem < 0 || op.elem > 5) return fail(TG_E_ARG, "tg_oplib_run: unknown elementwise op");
            GenElemArgs a{};
            a.nx = op.nin;
            for (int i = 0; i < a.nx; ++i) a.xs[i] = v[i];
            a.y = op.y;
            a.r0 = op.r0;
            a.r1 = op.r1;
            a.planes = Y[0] * Y[1];
            a.w = Y[3];
            a.op = op.elem;
            a.a = op.a;
            a.b = op.b;
            e = launch_gen_elem(a, stream);
            break;
        }
        default:
            return fail(TG_E_ARG, "tg_oplib_run: unknown operator kind");
    }
    if (e != cudaSuccess) return fail(TG_E_CUDA, std::string("tg_oplib_run: launch failed: ") + cudaGetErrorString(e));
    return TG_OK;
}

}  // namespace tg

extern "C" tg_status tg_oplib_run(const tg_oplib_op* op, void* stream) {
    if (!op) return tg::fail(TG_E_ARG, "tg_oplib_run: NULL descriptor");
    return tg::oplib_run(*op, stream);
}
