// generic.cu -- one kernel per graph operator, for the paper-faithful execution modes
// (TG_PER_OP: each operator is its own offload unit, "In our implementation, the
// individual operators are taken to be the offload units"; TG_BASELINE: PAPER.md:613). These
// are the "operator library" of Fig. 4: straightforward, correct sm_100a
// kernels over whole data structures; the fused units (edge.cu, cnn_*.cu) are the fast path.
#include <cuda_runtime.h>

#include "kernels.h"

namespace tg {
namespace {

__device__ __forceinline__ float tanh_f(float x) {
    x = fminf(fmaxf(x, -15.f), 15.f);
    const float e = __expf(2.f * x);
    return 1.f - __fdividef(2.f, 1.f + e);
}

// y[n][co][r][c] = sum_ci sum_i sum_j x[n][ci][r+i-pt][c+j-pl] * K[co][ci][i][j] (+ bias)
__global__ void conv_kernel(GenConvArgs a) {
    const int64_t total = a.n * a.co * a.ho * a.wo;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = idx % a.wo;
        int64_t t = idx / a.wo;
        const int64_t r = t % a.ho;
        t /= a.ho;
        const int64_t co = t % a.co;
        const int64_t n = t / a.co;
        float acc = 0.f;
        for (int64_t ci = 0; ci < a.ci; ++ci) {
            const float* xp = a.x + (n * a.ci + ci) * a.h * a.w;
            const float* kp = a.k + (co * a.ci + ci) * a.kh * a.kw;
            for (int i = 0; i < a.kh; ++i) {
                const int64_t rr = r + i - a.pt;
                if (rr < 0 || rr >= a.h) continue;
                for (int j = 0; j < a.kw; ++j) {
                    const int64_t cc = c + j - a.pl;
                    if (cc < 0 || cc >= a.w) continue;
                    acc = fmaf(xp[rr * a.w + cc], kp[i * a.kw + j], acc);
                }
            }
        }
        if (a.bias_kind == 1) acc += a.bias[co];
        if (a.bias_kind == 2) acc += a.bias[(co * a.ho + r) * a.wo + c];
        a.y[idx] = acc;
    }
}

__global__ void elem_kernel(GenElemArgs a) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.numel;
         i += (int64_t)gridDim.x * blockDim.x) {
        float v;
        switch (a.op) {
            case 0:  // TG_ADD: left fold
                v = a.xs[0][i];
                for (int k = 1; k < a.nx; ++k) v += a.xs[k][i];
                break;
            case 1: v = -a.xs[0][i]; break;                     // TG_NEG
            case 2: v = fmaf(a.a, a.xs[0][i], a.b); break;     // TG_AFFINE
            case 3: v = fabsf(a.xs[0][i]); break;               // TG_ABS
            case 4: v = tanh_f(a.xs[0][i]); break;              // tanh
            default: {                                          // max: (x > m) ? x : m
                v = a.xs[0][i];
                for (int k = 1; k < a.nx; ++k) {
                    const float x = a.xs[k][i];
                    v = (x > v) ? x : v;
                }
            }
        }
        a.y[i] = v;
    }
}

__global__ void sub_kernel(GenSubArgs a) {
    const int64_t total = a.n * a.c * a.ho * a.wo;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t cc = idx % a.wo;
        int64_t t = idx / a.wo;
        const int64_t r = t % a.ho;
        t /= a.ho;
        const int64_t ch = t % a.c;
        const int64_t n = t / a.c;
        const float* xp = a.x + (n * a.c + ch) * a.h * a.w;
        const float* pp = a.p + ch * a.s * a.s;
        float acc = 0.f;
        for (int i = 0; i < a.s; ++i)
            for (int j = 0; j < a.s; ++j) acc = fmaf(pp[i * a.s + j], xp[(a.s * r + i) * a.w + a.s * cc + j], acc);
        a.y[idx] = acc;
    }
}

unsigned blocks_for(int64_t n) {
    const int64_t b = (n + 255) / 256;
    return (unsigned)(b < 148 * 32 ? (b > 0 ? b : 1) : 148 * 32);
}

}  // namespace

cudaError_t launch_gen_conv(const GenConvArgs& a, cudaStream_t s) {
    conv_kernel<<<blocks_for(a.n * a.co * a.ho * a.wo), 256, 0, s>>>(a);
    return cudaGetLastError();
}
cudaError_t launch_gen_elem(const GenElemArgs& a, cudaStream_t s) {
    elem_kernel<<<blocks_for(a.numel), 256, 0, s>>>(a);
    return cudaGetLastError();
}
cudaError_t launch_gen_sub(const GenSubArgs& a, cudaStream_t s) {
    sub_kernel<<<blocks_for(a.n * a.c * a.ho * a.wo), 256, 0, s>>>(a);
    return cudaGetLastError();
}

}  // namespace tg
