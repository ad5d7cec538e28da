// generic.cu -- one kernel per graph operator, for the paper-faithful execution modes
// (TG_PER_OP: each operator is its own offload unit, "In our implementation, the
// individual operators are taken to be the offload units"; TG_BASELINE: PAPER.md:613). These
// are the "operator library" of Fig. 4: straightforward, correct sm_100a
// kernels; the fused units (edge.cu, cnn_*.cu) are the fast path.
//
// Every kernel computes the output rows [r0, r1) of one operator -- one piece of a split
// operator or the whole operator -- reading its inputs through views of
// the input pieces resident in the arena. An output element is computed by the same
// arithmetic in the same order whichever piece it falls in, so split execution is bit-exact
// with unsplit execution.
#include <cuda_runtime.h>

#include "kernels.h"
#include "tanh_fp32.cuh"

namespace tg {
namespace {

__device__ __forceinline__ float tanh_f(float x) { return tanh_fp32(x); }

// row r of plane `plane` (= n * c + ch) of a DS of row width w, from the first piece that
// holds it (nullptr if none does: the planner guarantees that never happens for rows inside
// the image)
__device__ __forceinline__ const float* vrow(const GenView& v, int64_t plane, int64_t r, int64_t w) {
    for (int s = 0; s < v.nseg; ++s) {
        const GenSeg& g = v.seg[s];
        if (r >= g.r0 && r < g.r1) return g.p + (plane * (g.r1 - g.r0) + (r - g.r0)) * w;
    }
    return nullptr;
}

// y[n][co][r][c] = sum_ci sum_i sum_j x[n][ci][r+i-pt][c+j-pl] * K[co][ci][i][j] (+ bias),
// zero outside the image (SAME), for r in [r0, r1)
__global__ void conv_kernel(GenConvArgs a) {
    const int64_t rows = a.r1 - a.r0;
    const int64_t total = a.n * a.co * rows * a.wo;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = idx % a.wo;
        int64_t t = idx / a.wo;
        const int64_t r = a.r0 + t % rows;
        t /= rows;
        const int64_t co = t % a.co;
        const int64_t n = t / a.co;
        float acc = 0.f;
        for (int64_t ci = 0; ci < a.ci; ++ci) {
            const float* kp = a.k + (co * a.ci + ci) * a.kh * a.kw;
            for (int i = 0; i < a.kh; ++i) {
                const int64_t rr = r + i - a.pt;
                if (rr < 0 || rr >= a.h) continue;
                const float* xr = vrow(a.x, n * a.ci + ci, rr, a.w);
                for (int j = 0; j < a.kw; ++j) {
                    const int64_t cc = c + j - a.pl;
                    if (cc < 0 || cc >= a.w) continue;
                    acc = fmaf(xr[cc], kp[i * a.kw + j], acc);
                }
            }
        }
        if (a.bias_kind == 1) acc += vrow(a.bias, 0, 0, a.co)[co];
        if (a.bias_kind == 2) acc += vrow(a.bias, co, r, a.wo)[c];
        a.y[idx] = acc;
    }
}

__global__ void elem_kernel(GenElemArgs a) {
    const int64_t rows = a.r1 - a.r0;
    const int64_t total = a.planes * rows * a.w;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = i % a.w;
        const int64_t t = i / a.w;
        const int64_t r = a.r0 + t % rows;
        const int64_t pl = t / rows;
        auto X = [&](int k) { return vrow(a.xs[k], pl, r, a.w)[c]; };
        float v;
        switch (a.op) {
            case 0:  // TG_ADD: left fold
                v = X(0);
                for (int k = 1; k < a.nx; ++k) v += X(k);
                break;
            case 1: v = -X(0); break;                     // TG_NEG
            case 2: v = fmaf(a.a, X(0), a.b); break;      // TG_AFFINE
            case 3: v = fabsf(X(0)); break;               // TG_ABS
            case 4: v = tanh_f(X(0)); break;              // tanh
            default: {                                    // max: (x > m) ? x : m
                v = X(0);
                for (int k = 1; k < a.nx; ++k) {
                    const float x = X(k);
                    v = (x > v) ? x : v;
                }
            }
        }
        a.y[i] = v;
    }
}

__global__ void sub_kernel(GenSubArgs a) {
    const int64_t rows = a.r1 - a.r0;
    const int64_t total = a.n * a.c * rows * a.wo;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t cc = idx % a.wo;
        int64_t t = idx / a.wo;
        const int64_t r = a.r0 + t % rows;
        t /= rows;
        const int64_t ch = t % a.c;
        const int64_t n = t / a.c;
        const float* pp = a.p + ch * a.s * a.s;
        float acc = 0.f;
        for (int i = 0; i < a.s; ++i) {
            const float* xr = vrow(a.x, n * a.c + ch, a.s * r + i, a.w);
            for (int j = 0; j < a.s; ++j) acc = fmaf(pp[i * a.s + j], xr[a.s * cc + j], acc);
        }
        a.y[idx] = acc;
    }
}

// C rows [r0, r1) = A rows [r0, r1) x B: 64 x 64 output tiles, 16-deep k slices staged in
// shared memory, 4 x 4 outputs per thread; every element accumulates l = 0..k-1 in order
// (fmaf), so a row's value does not depend on the tile or piece that computes it.
constexpr int MB = 64, NB = 64, KB = 16;
__global__ __launch_bounds__(256) void matmul_kernel(GenMatmulArgs a) {
    __shared__ float As[KB][MB + 4];
    __shared__ float Bs[KB][NB + 4];
    const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
    const int64_t m0 = a.r0 + (int64_t)blockIdx.y * MB, n0 = (int64_t)blockIdx.x * NB;
    float acc[4][4] = {};
    for (int64_t k0 = 0; k0 < a.k; k0 += KB) {
        for (int e = 0; e < 4; ++e) {
            const int idx = threadIdx.x + e * 256;
            const int mr = idx / KB, kk = idx % KB;
            const int64_t row = m0 + mr, col = k0 + kk;
            As[kk][mr] = (row < a.r1 && col < a.k) ? vrow(a.a, 0, row, a.k)[col] : 0.f;
            const int kb = idx / NB, nc = idx % NB;
            Bs[kb][nc] = (k0 + kb < a.k && n0 + nc < a.n) ? vrow(a.b, 0, k0 + kb, a.n)[n0 + nc] : 0.f;
        }
        __syncthreads();
        const int kl = (int)((a.k - k0) < KB ? (a.k - k0) : KB);
        for (int kk = 0; kk < kl; ++kk) {
            float av[4], bv[4];
            for (int i = 0; i < 4; ++i) av[i] = As[kk][ty * 4 + i];
            for (int j = 0; j < 4; ++j) bv[j] = Bs[kk][tx * 4 + j];
            for (int i = 0; i < 4; ++i)
                for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
        }
        __syncthreads();
    }
    for (int i = 0; i < 4; ++i) {
        const int64_t row = m0 + ty * 4 + i;
        if (row >= a.r1) break;
        for (int j = 0; j < 4; ++j) {
            const int64_t col = n0 + tx * 4 + j;
            if (col < a.n) a.c[(row - a.r0) * a.n + col] = acc[i][j];
        }
    }
}

unsigned blocks_for(int64_t n) {
    const int64_t b = (n + 255) / 256;
    return (unsigned)(b < 148 * 32 ? (b > 0 ? b : 1) : 148 * 32);
}

}  // namespace

cudaError_t launch_gen_conv(const GenConvArgs& a, cudaStream_t s) {
    conv_kernel<<<blocks_for(a.n * a.co * (a.r1 - a.r0) * a.wo), 256, 0, s>>>(a);
    return cudaGetLastError();
}
cudaError_t launch_gen_elem(const GenElemArgs& a, cudaStream_t s) {
    elem_kernel<<<blocks_for(a.planes * (a.r1 - a.r0) * a.w), 256, 0, s>>>(a);
    return cudaGetLastError();
}
cudaError_t launch_gen_sub(const GenSubArgs& a, cudaStream_t s) {
    sub_kernel<<<blocks_for(a.n * a.c * (a.r1 - a.r0) * a.wo), 256, 0, s>>>(a);
    return cudaGetLastError();
}
cudaError_t launch_gen_matmul(const GenMatmulArgs& a, cudaStream_t s) {
    const dim3 grid((unsigned)((a.n + NB - 1) / NB), (unsigned)((a.r1 - a.r0 + MB - 1) / MB));
    if (grid.x == 0 || grid.y == 0) return cudaSuccess;
    matmul_kernel<<<grid, 256, 0, s>>>(a);
    return cudaGetLastError();
}

}  // namespace tg
