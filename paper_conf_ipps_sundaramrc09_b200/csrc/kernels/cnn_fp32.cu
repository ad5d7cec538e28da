// cnn_fp32.cu -- the three fused CNN offload units on FP32 CUDA cores (sm_100a).
//
// CNN of PAPER.md:635 (reconstructed in SURVEY F2): C1(1->8,5x5) T S2 T C3(8->20,5x5) T S4 T
// C5(20->n5,5x5) T C6(n5->9,1x1). The paper expands each conv layer into per-pair
// convolutions, partial-sum adds and a bias-plane add (Fig. 7); here one
// kernel per offload unit keeps all of those temporaries in registers:
//   U1: C1 + bias + tanh + S2 + tanh   -> T2 (8 planes)
//   U2: C3 + bias + tanh + S4 + tanh   -> T4 (20 planes)
//   U3: C5 + bias + tanh + C6 + bias   -> output (9 planes); T5 never leaves registers
// Row coordinates are global level rows; a chunk's buffers start at the row0 the planner
// back-propagated. Every output pixel is computed by the same instruction
// sequence in the same order wherever its tile or chunk starts, so split runs are
// bit-identical to unsplit runs.
//
// tanh: 1 - 2/(1 + e^{2x}) with MUFU ex2/rcp (x clamped to +-15): absolute error < 3e-7,
// well inside the normwise 1e-5 parity bound.
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstring>

#include "kernels.h"
#include "tanh_fp32.cuh"
#include "tma_util.cuh"

namespace tg {
namespace {

__device__ __forceinline__ float tanh_f(float x) { return tanh_fp32(x); }
// hi/lo fp16 pairs of two consecutive channels (element 0 in the low half): the 3xFP16 split
__device__ __forceinline__ void split_f16x2(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    const __half2 h = __floats2half2_rn(x0, x1);
    const float2 hf = __half22float2(h);
    const __half2 l = __floats2half2_rn(x0 - hf.x, x1 - hf.y);
    hi = *reinterpret_cast<const uint32_t*>(&h);
    lo = *reinterpret_cast<const uint32_t*>(&l);
}

// MUFU.TANH (one SFU op, relative error ~2^-11): only where the result is rounded to bf16
// anyway (U1 feeding the tensor-core path), never on the fp32 path.
__device__ __forceinline__ float tanh_mufu(float x) {
    float y;
    asm("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// ============================================================================ U1
// One thread per T2 pixel and all 8 channels: the 2x2 C1 pixels under it (4 x 8 x 25 FFMA
// from a 6x6 input window), bias, tanh, the 2x2 subsample, tanh. Weights travel in the
// constant bank (kernel parameter) so FFMAs take them as uniform operands.
struct U1W {
    float k1[25][8];  // [tap][ch]: channel pairs are adjacent (one FFMA2 operand)
    float p2[8][4];
};

constexpr int U1_TR = 8, U1_TC = 16;                // T2 tile (rows x cols) = 128 threads
constexpr int U1_IR = 2 * U1_TR + 4, U1_IC = 2 * U1_TC + 4;  // 20 x 36 input window

template <bool kBf16>
__global__ void __launch_bounds__(128, 4) cnn_u1_kernel(const CnnU1Args a, const __grid_constant__ U1W w) {
    __shared__ __align__(16) float xs[U1_IR * U1_IC];
    const int tid = threadIdx.x, ty = tid / U1_TC, tx = tid % U1_TC;
    const int64_t img = blockIdx.z;
    const int64_t r2_0 = a.t2_row0 + (int64_t)blockIdx.y * U1_TR;  // global T2 row of the tile
    const int64_t c2_0 = (int64_t)blockIdx.x * U1_TC;
    const int64_t ir0 = 2 * r2_0, ic0 = 2 * c2_0;                  // global input row/col
    const float* inb = a.in + img * a.in_img_stride;
    const int64_t in_rows_avail = a.in_img_stride / a.W;
    for (int idx = tid; idx < U1_IR * U1_IC; idx += 128) {
        const int r = idx / U1_IC, c = idx - r * U1_IC;
        const int64_t br = ir0 + r - a.in_row0, gc = ic0 + c;
        xs[idx] = (br >= 0 && br < in_rows_avail && gc < a.W) ? __ldg(inb + br * a.W + gc) : 0.f;
    }
    __syncthreads();
    const int64_t R2 = r2_0 + ty, C2 = c2_0 + tx;
    if (R2 >= a.t2_row0 + a.t2_rows || C2 >= a.w2) return;

    // bias of the 2x2 C1 pixels under this T2 pixel, loaded before the FMA sweep so the
    // loads are in flight while it runs (one 8-byte load per channel and row when aligned)
    float2 bb[8][2];
    if (a.b1_plane) {
        const bool v2 = (a.w1 & 1) == 0 && (reinterpret_cast<uintptr_t>(a.b1) & 7) == 0;
#pragma unroll
        for (int ch = 0; ch < 8; ++ch)
#pragma unroll
            for (int ra = 0; ra < 2; ++ra) {
                const float* bp = a.b1 + ((int64_t)ch * a.b1_rows + (2 * R2 + ra - a.b1_row0)) * a.w1 + 2 * C2;
                bb[ch][ra] = v2 ? __ldg(reinterpret_cast<const float2*>(bp)) : make_float2(__ldg(bp), __ldg(bp + 1));
            }
    } else {
#pragma unroll
        for (int ch = 0; ch < 8; ++ch) {
            const float b = __ldg(a.b1 + ch);
            bb[ch][0] = bb[ch][1] = make_float2(b, b);
        }
    }

    // FFMA2 over channel pairs (2c, 2c+1): each lane rounds exactly like fmaf
    float2 acc2[4][4];
#pragma unroll
    for (int cp = 0; cp < 4; ++cp)
#pragma unroll
        for (int p = 0; p < 4; ++p) acc2[cp][p] = make_float2(0.f, 0.f);
#pragma unroll
    for (int i = 0; i < 6; ++i) {
        float x[6];
        const float2* xr = reinterpret_cast<const float2*>(&xs[(2 * ty + i) * U1_IC + 2 * tx]);
#pragma unroll
        for (int v = 0; v < 3; ++v) {
            const float2 t = xr[v];
            x[2 * v] = t.x;
            x[2 * v + 1] = t.y;
        }
#pragma unroll
        for (int ra = 0; ra < 2; ++ra) {
            const int ki = i - ra;  // kernel row for C1 row 2*R2 + ra
            if (ki < 0 || ki > 4) continue;
#pragma unroll
            for (int cp = 0; cp < 4; ++cp)
#pragma unroll
                for (int kj = 0; kj < 5; ++kj) {
                    const float2 wv = make_float2(w.k1[ki * 5 + kj][2 * cp], w.k1[ki * 5 + kj][2 * cp + 1]);
#pragma unroll
                    for (int cb = 0; cb < 2; ++cb)
                        acc2[cp][ra * 2 + cb] = __ffma2_rn(make_float2(x[cb + kj], x[cb + kj]), wv, acc2[cp][ra * 2 + cb]);
                }
        }
    }
    float* t2 = a.t2 + img * a.t2_img_stride;
    const int64_t plane = a.t2_rows * a.w2;
    float tv[8];
#pragma unroll
    for (int ch = 0; ch < 8; ++ch) {
        float s = 0.f;
#pragma unroll
        for (int p = 0; p < 4; ++p) {
            const float b = (p & 1) ? bb[ch][p >> 1].y : bb[ch][p >> 1].x;
            const float av = (ch & 1) ? acc2[ch >> 1][p].y : acc2[ch >> 1][p].x;
            const float t = kBf16 ? tanh_mufu(av + b) : tanh_f(av + b);
            s = fmaf(w.p2[ch][p], t, s);
        }
        tv[ch] = kBf16 ? tanh_mufu(s) : tanh_f(s);
    }
    if (kBf16) {  // one 16-byte pixel of 8 bf16 channels (the tensor-core U2's operand rows)
        uint4* d = reinterpret_cast<uint4*>(a.t2) + (img * a.t2_rows + (R2 - a.t2_row0)) * a.w2 + C2;
        uint32_t p[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            asm("cvt.rn.bf16x2.f32 %0, %1, %2;\n" : "=r"(p[k]) : "f"(tv[2 * k + 1]), "f"(tv[2 * k]));
        }
        *d = make_uint4(p[0], p[1], p[2], p[3]);
    } else if (a.t2_h3) {  // fp16-split pixels (x 2^4) for the 3xFP16 U2: [part][rows][w2][8]
        uint4* d = reinterpret_cast<uint4*>(a.t2) + img * 2 * plane + (R2 - a.t2_row0) * a.w2 + C2;
        uint32_t hi[4], lo[4];
#pragma unroll
        for (int m = 0; m < 4; ++m) split_f16x2(16.f * tv[2 * m], 16.f * tv[2 * m + 1], hi[m], lo[m]);
        d[0] = make_uint4(hi[0], hi[1], hi[2], hi[3]);
        d[plane] = make_uint4(lo[0], lo[1], lo[2], lo[3]);
    } else {
#pragma unroll
        for (int ch = 0; ch < 8; ++ch) t2[ch * plane + (R2 - a.t2_row0) * a.w2 + C2] = tv[ch];
    }
}

// ---------------------------------------------------------------------------- U1, TMA path
// Persistent variant (W % 4 == 0): each CTA walks T2 tiles of 8 rows x 32 columns; thread
// (ty, tx) owns T2 pixels (ty, 2tx) and (ty, 2tx+1), i.e. a 2 x 4 block of C1 pixels x 8
// channels (32 FFMA2 accumulators) from a 6 x 8 input window (two LDS.128 per row). One
// thread stages the NEXT tile with two TMA loads -- the 20 x 68 input window and the
// 8 x 16 x 64 bias block of the plane -- into the other shared-memory stage while the CTA
// computes the current one (OOB zero fill = the image edge). Same FFMA order per output as
// the fallback kernel above, so the two give identical bits.
constexpr int U1T_R = 8, U1T_C = 32;
constexpr int U1T_IR = 2 * U1T_R + 4, U1T_IC = 2 * U1T_C + 4;  // 20 x 68 input window
constexpr int U1T_BR = 2 * U1T_R, U1T_BC = 2 * U1T_C;          // 16 x 64 C1 bias block per channel
constexpr int U1T_XBYTES = U1T_IR * U1T_IC * 4;                 // 5440
constexpr int U1T_XSTRIDE = (U1T_XBYTES + 127) / 128 * 128;
constexpr int U1T_BBYTES = 8 * U1T_BR * U1T_BC * 4;             // 32768
constexpr int U1T_STAGE = U1T_XSTRIDE + U1T_BBYTES;

template <bool kBf16, bool kPlane>
__global__ void __launch_bounds__(128, 3)
    cnn_u1_tma_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap bmap,
                      const CnnU1Args a, const __grid_constant__ U1W w, const int tiles_c, const int tiles_r,
                      const int64_t ntiles) {
    extern __shared__ __align__(128) uint8_t smraw[];
    uint8_t* base = smraw + ((128 - (tma_smem_u32(smraw) & 127)) & 127);
    __shared__ __align__(8) uint64_t full[2];
    const int tid = threadIdx.x, ty = tid >> 4, tx = tid & 15;
    if (tid == 0) {
        tma_prefetch_map(&xmap);
        if (kPlane) tma_prefetch_map(&bmap);
        tma_mbar_init(&full[0], 1);
        tma_mbar_init(&full[1], 1);
        tma_fence_init();
    }
    __syncthreads();
    // tile -> (image, first T2 row, first T2 column) in 32-bit arithmetic (the launcher checks
    // that tile counts fit; 64-bit division is a long software sequence)
    const uint32_t per = (uint32_t)tiles_c * (uint32_t)tiles_r;
    auto coords = [&](int64_t t, int64_t& img, int64_t& r2_0, int64_t& c2_0) {
        const uint32_t tu = (uint32_t)t, im = tu / per, rem = tu - im * per, ry = rem / (uint32_t)tiles_c;
        img = im;
        r2_0 = a.t2_row0 + (int64_t)ry * U1T_R;
        c2_0 = (int64_t)(rem - ry * (uint32_t)tiles_c) * U1T_C;
    };
    auto issue = [&](int64_t t, int b) {
        int64_t img, r2_0, c2_0;
        coords(t, img, r2_0, c2_0);
        uint8_t* st = base + b * U1T_STAGE;
        tma_expect_tx(&full[b], U1T_XBYTES + (kPlane ? U1T_BBYTES : 0));
        tma_load_3d(st, &xmap, (int)(2 * c2_0), (int)(2 * r2_0 - a.in_row0), (int)img, &full[b]);
        if (kPlane) tma_load_3d(st + U1T_XSTRIDE, &bmap, (int)(2 * c2_0), (int)(2 * r2_0 - a.b1_row0), 0, &full[b]);
    };
    const int64_t plane = a.t2_rows * a.w2;
    int64_t t = blockIdx.x;
    if (tid == 0 && t < ntiles) issue(t, 0);
    for (int k = 0; t < ntiles; ++k, t += gridDim.x) {
        const int b = k & 1;
        if (tid == 0 && t + gridDim.x < ntiles) issue(t + gridDim.x, b ^ 1);
        tma_wait(&full[b], (uint32_t)((k >> 1) & 1));
        const float* xs = reinterpret_cast<const float*>(base + b * U1T_STAGE);
        const float* bs = reinterpret_cast<const float*>(base + b * U1T_STAGE + U1T_XSTRIDE);
        int64_t img, r2_0, c2_0;
        coords(t, img, r2_0, c2_0);

        float2 acc[4][2][4];  // [channel pair][C1 row ra][C1 column cb]
#pragma unroll
        for (int cp = 0; cp < 4; ++cp)
#pragma unroll
            for (int ra = 0; ra < 2; ++ra)
#pragma unroll
                for (int cb = 0; cb < 4; ++cb) acc[cp][ra][cb] = make_float2(0.f, 0.f);
#pragma unroll
        for (int i = 0; i < 6; ++i) {
            float x[8];
            const float4* xr = reinterpret_cast<const float4*>(&xs[(2 * ty + i) * U1T_IC + 4 * tx]);
            const float4 u = xr[0], v = xr[1];
            x[0] = u.x; x[1] = u.y; x[2] = u.z; x[3] = u.w;
            x[4] = v.x; x[5] = v.y; x[6] = v.z; x[7] = v.w;
#pragma unroll
            for (int ra = 0; ra < 2; ++ra) {
                const int ki = i - ra;
                if (ki < 0 || ki > 4) continue;
#pragma unroll
                for (int cp = 0; cp < 4; ++cp)
#pragma unroll
                    for (int kj = 0; kj < 5; ++kj) {
                        const float2 wv = make_float2(w.k1[ki * 5 + kj][2 * cp], w.k1[ki * 5 + kj][2 * cp + 1]);
#pragma unroll
                        for (int cb = 0; cb < 4; ++cb)
                            acc[cp][ra][cb] = __ffma2_rn(make_float2(x[cb + kj], x[cb + kj]), wv, acc[cp][ra][cb]);
                    }
            }
        }
        const int64_t R2 = r2_0 + ty;
        const bool row_ok = R2 < a.t2_row0 + a.t2_rows;
        // bias, tanh, the 2x2 subsample, tanh -- per channel PAIR, the same pair the FFMA2
        // accumulators hold, with paired FP32 arithmetic (each lane rounds like the scalar ops, so
        // the bits equal a per-channel loop)
        float tv[2][8];
#pragma unroll
        for (int cp = 0; cp < 4; ++cp) {
            float4 b4[2][2];  // [channel parity][C1 row]
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const int ch = 2 * cp + e;
                if (kPlane) {
#pragma unroll
                    for (int ra = 0; ra < 2; ++ra)
                        b4[e][ra] = *reinterpret_cast<const float4*>(&bs[(ch * U1T_BR + 2 * ty + ra) * U1T_BC + 4 * tx]);
                } else {
                    const float bv = __ldg(a.b1 + ch);
                    b4[e][0] = b4[e][1] = make_float4(bv, bv, bv, bv);
                }
            }
#pragma unroll
            for (int q = 0; q < 2; ++q) {
                float2 s = make_float2(0.f, 0.f);
#pragma unroll
                for (int p = 0; p < 4; ++p) {
                    const int ra = p >> 1, cb = 2 * q + (p & 1);
                    auto pick = [&](const float4& bb) { return cb == 0 ? bb.x : cb == 1 ? bb.y : cb == 2 ? bb.z : bb.w; };
                    const float2 av = __fadd2_rn(acc[cp][ra][cb], make_float2(pick(b4[0][ra]), pick(b4[1][ra])));
                    const float2 th = kBf16 ? make_float2(tanh_mufu(av.x), tanh_mufu(av.y)) : tanh_fp32x2(av);
                    s = __ffma2_rn(make_float2(w.p2[2 * cp][p], w.p2[2 * cp + 1][p]), th, s);
                }
                const float2 t = kBf16 ? make_float2(tanh_mufu(s.x), tanh_mufu(s.y)) : tanh_fp32x2(s);
                tv[q][2 * cp] = t.x;
                tv[q][2 * cp + 1] = t.y;
            }
        }
        __syncthreads();  // stage b is free for the prefetch issued in iteration k+1
        if (row_ok) {
            const int64_t C2 = c2_0 + 2 * tx;
            if (kBf16) {
                uint4* d = reinterpret_cast<uint4*>(a.t2) + (img * a.t2_rows + (R2 - a.t2_row0)) * a.w2 + C2;
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    if (C2 + q >= a.w2) continue;
                    uint32_t pk[4];
#pragma unroll
                    for (int m = 0; m < 4; ++m)
                        asm("cvt.rn.bf16x2.f32 %0, %1, %2;\n" : "=r"(pk[m]) : "f"(tv[q][2 * m + 1]), "f"(tv[q][2 * m]));
                    d[q] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
                }
            } else if (a.t2_h3) {  // fp16-split pixels (x 2^4): [part][rows][w2][8]
                uint4* d = reinterpret_cast<uint4*>(a.t2) + img * 2 * plane + (R2 - a.t2_row0) * a.w2 + C2;
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    if (C2 + q >= a.w2) continue;
                    uint32_t hi[4], lo[4];
#pragma unroll
                    for (int m = 0; m < 4; ++m)
                        split_f16x2(16.f * tv[q][2 * m], 16.f * tv[q][2 * m + 1], hi[m], lo[m]);
                    d[q] = make_uint4(hi[0], hi[1], hi[2], hi[3]);
                    d[plane + q] = make_uint4(lo[0], lo[1], lo[2], lo[3]);
                }
            } else {
                float* t2 = a.t2 + img * a.t2_img_stride + (R2 - a.t2_row0) * a.w2 + C2;
#pragma unroll
                for (int ch = 0; ch < 8; ++ch) {
                    if (C2 + 1 < a.w2)
                        *reinterpret_cast<float2*>(t2 + ch * plane) = make_float2(tv[0][ch], tv[1][ch]);
                    else if (C2 < a.w2)
                        t2[ch * plane] = tv[0][ch];
                }
            }
        }
    }
}

// ============================================================================ U2
// One thread per T4 pixel and all 20 channels (the 2x2 C3 pixels under it: 80
// accumulators). Loop over the 8 input planes; per plane a fully unrolled 6-row sweep of
// the 6x6 window (2000 FFMA). The 20x8x25 weights are a kernel parameter (constant bank).
// The T2 window and, in bias-plane mode, the C3 bias block under the tile reach shared
// memory as one batch of asynchronous copies (LDGSTS, zero fill outside the chunk), so a
// CTA waits one memory latency before computing, and the other resident CTA covers it.
struct U2W {
    float k3[8][25][20];  // [ci][tap][co]: the 20 output channels of one tap are contiguous
    float p4[20][4];
};

constexpr int U2_TR = 8, U2_TC = 16;
constexpr int U2_IR = 2 * U2_TR + 4, U2_IC = 2 * U2_TC + 4;  // 20 x 36 per plane
constexpr int U2_BR = 2 * U2_TR, U2_BC = 2 * U2_TC;           // C3 bias block 16 x 32 per channel

__device__ __forceinline__ void cp_async4(uint32_t dst, const float* src, bool valid) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"(dst), "l"(src), "r"(valid ? 4 : 0)
                 : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }

__global__ void __launch_bounds__(128, 2) cnn_u2_kernel(const CnnU2Args a, const __grid_constant__ U2W w) {
    extern __shared__ __align__(16) float u2sm[];
    float* xs = u2sm;                      // [8][U2_IR * U2_IC]
    float* bs = xs + 8 * U2_IR * U2_IC;    // [20][U2_BR][U2_BC] (bias-plane mode)
    const int tid = threadIdx.x, ty = tid / U2_TC, tx = tid % U2_TC;
    const int64_t img = blockIdx.z;
    const int64_t r4_0 = a.t4_row0 + (int64_t)blockIdx.y * U2_TR;
    const int64_t c4_0 = (int64_t)blockIdx.x * U2_TC;
    const int64_t ir0 = 2 * r4_0, ic0 = 2 * c4_0;  // global T2 row/col of the window (= C3 row/col of the bias block)
    const float* t2b = a.t2 + img * a.t2_img_stride;
    const int64_t plane = a.t2_rows * a.w2;
    for (int rem = tid; rem < U2_IR * U2_IC; rem += 128) {
        const int r = rem / U2_IC, c = rem - r * U2_IC;
        const int64_t br = ir0 + r - a.t2_row0, gc = ic0 + c;
        const bool ok = br >= 0 && br < a.t2_rows && gc < a.w2;
        const float* src = ok ? t2b + br * a.w2 + gc : a.t2;
        const uint32_t dst = (uint32_t)__cvta_generic_to_shared(xs + rem);
#pragma unroll
        for (int ci = 0; ci < 8; ++ci)
            cp_async4(dst + 4u * ci * (U2_IR * U2_IC), ok ? src + ci * plane : src, ok);
    }
    if (a.b3_plane) {
        const int64_t b3_plane = a.b3_rows * a.w3;
        for (int rem = tid; rem < U2_BR * U2_BC; rem += 128) {
            const int r = rem / U2_BC, c = rem - r * U2_BC;
            const int64_t br = ir0 + r - a.b3_row0, gc = ic0 + c;
            const bool ok = br >= 0 && br < a.b3_rows && gc < a.w3;
            const float* src = ok ? a.b3 + br * a.w3 + gc : a.b3;
            const uint32_t dst = (uint32_t)__cvta_generic_to_shared(bs + rem);
#pragma unroll 4
            for (int co = 0; co < 20; ++co)
                cp_async4(dst + 4u * co * (U2_BR * U2_BC), ok ? src + co * b3_plane : src, ok);
        }
    }
    cp_async_commit();
    cp_async_wait_all();
    __syncthreads();
    const int64_t R4 = r4_0 + ty, C4 = c4_0 + tx;
    if (R4 >= a.t4_row0 + a.t4_rows || C4 >= a.w4) return;

    float2 acc2[10][4];  // channel pairs (2c, 2c+1), FFMA2
#pragma unroll
    for (int cp = 0; cp < 10; ++cp)
#pragma unroll
        for (int p = 0; p < 4; ++p) acc2[cp][p] = make_float2(0.f, 0.f);
#pragma unroll 1
    for (int ci = 0; ci < 8; ++ci) {
#pragma unroll
        for (int i = 0; i < 6; ++i) {
            float x[6];
            const float2* xr = reinterpret_cast<const float2*>(&xs[ci * (U2_IR * U2_IC) + (2 * ty + i) * U2_IC + 2 * tx]);
#pragma unroll
            for (int v = 0; v < 3; ++v) {
                const float2 t = xr[v];
                x[2 * v] = t.x;
                x[2 * v + 1] = t.y;
            }
#pragma unroll
            for (int ra = 0; ra < 2; ++ra) {
                const int ki = i - ra;
                if (ki < 0 || ki > 4) continue;
#pragma unroll
                for (int kj = 0; kj < 5; ++kj)
#pragma unroll
                    for (int cp = 0; cp < 10; ++cp) {
                        const float2 wv = make_float2(w.k3[ci][ki * 5 + kj][2 * cp], w.k3[ci][ki * 5 + kj][2 * cp + 1]);
                        acc2[cp][ra * 2 + 0] = __ffma2_rn(make_float2(x[kj], x[kj]), wv, acc2[cp][ra * 2 + 0]);
                        acc2[cp][ra * 2 + 1] = __ffma2_rn(make_float2(x[kj + 1], x[kj + 1]), wv, acc2[cp][ra * 2 + 1]);
                    }
            }
        }
    }
    float* t4 = a.t4 + img * a.t4_img_stride;
    const int64_t oplane = a.t4_rows * a.w4;
    float tv[20];
#pragma unroll
    for (int co = 0; co < 20; ++co) {
        float bq[4];
        if (a.b3_plane) {
#pragma unroll
            for (int ra = 0; ra < 2; ++ra) {
                const float2 bb = *reinterpret_cast<const float2*>(&bs[(co * U2_BR + 2 * ty + ra) * U2_BC + 2 * tx]);
                bq[2 * ra] = bb.x;
                bq[2 * ra + 1] = bb.y;
            }
        } else {
            const float b = __ldg(a.b3 + co);
            bq[0] = bq[1] = bq[2] = bq[3] = b;
        }
        float s = 0.f;
#pragma unroll
        for (int p = 0; p < 4; ++p) {
            const float av = (co & 1) ? acc2[co >> 1][p].y : acc2[co >> 1][p].x;
            s = fmaf(w.p4[co][p], tanh_f(av + bq[p]), s);
        }
        tv[co] = tanh_f(s);
    }
    const int64_t px = (R4 - a.t4_row0) * a.w4 + C4;
#pragma unroll
    for (int co = 0; co < 20; ++co) t4[co * oplane + px] = tv[co];
}

// ============================================================================ U3
// C5 + bias + tanh + C6 + bias. One CTA (256 threads, one per SM: ~150 KB of shared memory)
// per work item of 1024 output positions; a thread owns 4 consecutive positions of a row and
// loops over the C5 channels in groups of 8 (4 px x 8 ch accumulators over 20 planes x 25
// taps, channel-paired FFMA2 with broadcast LDS.128 weights), then bias + tanh and the
// group's contribution to the 9 C6 dot products (C6 is 1x1: a dot product over n5), so T5
// never exists in memory. All loads into shared memory are asynchronous (LDGSTS with zero
// fill for halo and out-of-range positions): the band of T4 once per item, the weights of
// group g+1 while group g computes (double buffer), and the bias-plane values of a group are
// fetched into registers before its tap loop so their latency hides behind it.
// Two item geometries (chosen per launch by the fraction of wasted positions):
//  - narrow images (padded T4 pitch P = round4(w4) <= 256): positions are flattened over
//    (row, col) with pitch P, an item is 1024 consecutive flattened positions, and the
//    shared band holds the flattened range [p0, p0 + 1024 + 4P + 8) of every T4 plane; the
//    P - w5 columns past the row end are computed and dropped (2-5 % at VGA width, instead
//    of the 20 % a 64-column tile loses on 153 columns);
//  - wide images: 16 x 64 output tiles, T4 window 20 x 68 per plane.
// Every output is the same FFMA sequence (ci, i, j order) wherever its item starts, so split
// runs stay bit-identical to unsplit runs.
constexpr int U3_THREADS = 256, U3_POS = 4 * U3_THREADS, U3_P = 4, U3_G = 8;
constexpr int U3W_TR = 16, U3W_TC = 64, U3W_PITCH = U3W_TC + 4;  // wide tile (pitch 68)
constexpr int U3_NARROW_MAX_PITCH = 256;


struct U3Geom {
    int narrow;             // 1: flattened items, 0: 16 x 64 tiles
    int pitch;              // shared-memory row pitch (floats)
    int cs;                 // shared-memory plane stride (floats)
    int stage;              // floats staged per plane
    int tiles_c;            // wide: column tiles
    int64_t items_per_img;
};

__global__ void __launch_bounds__(U3_THREADS, 1) cnn_u3_kernel(const CnnU3Args a, const U3Geom gm) {
    extern __shared__ __align__(16) float sm[];
    const int n5 = a.n5, n5p = (n5 + U3_G - 1) / U3_G * U3_G;
    float* xs = sm;                             // [20][cs]
    float* ws = xs + 20 * gm.cs;                // [2][20*25][8] group weights (double buffer)
    float* k6s = ws + 2 * 20 * 25 * U3_G;       // [n5p][12]: the 9 C6 weights of a channel
    const int tid = threadIdx.x;
    const int64_t img = blockIdx.x / gm.items_per_img;
    const int64_t item = blockIdx.x - img * gm.items_per_img;
    const float* t4b = a.t4 + img * a.t4_img_stride;
    const int64_t plane = a.t4_rows * a.w4;

    // geometry of the staged band and of this thread's 4 positions
    int64_t R5, C5;  // global C5 row, column of the first position
    int sb;          // shared offset of the first position (tap (0,0)) within a plane
    int64_t p0 = 0, r0 = 0, c0 = 0;
    if (gm.narrow) {
        p0 = item * U3_POS;
        const int64_t p = p0 + 4 * tid;
        R5 = a.out_row0 + p / gm.pitch;
        C5 = p % gm.pitch;
        sb = 4 * tid;
    } else {
        const int64_t tr = item / gm.tiles_c, tc = item - tr * gm.tiles_c;
        r0 = a.out_row0 + tr * U3W_TR;
        c0 = tc * U3W_TC;
        const int ty = tid / (U3W_TC / U3_P), tg = tid % (U3W_TC / U3_P);
        R5 = r0 + ty;
        C5 = c0 + tg * U3_P;
        sb = ty * U3W_PITCH + tg * U3_P;
    }
    const bool row_ok = R5 < a.out_row0 + a.out_rows;

    auto stage_weights = [&](int g0, int buf) {
        float* wd = ws + buf * (20 * 25 * U3_G);
        for (int idx = tid; idx < 20 * 25 * U3_G; idx += U3_THREADS) {
            const int ch = idx / 500, k = idx - ch * 500;  // coalesced over k within a channel
            const bool ok = g0 + ch < n5;
            cp_async4((uint32_t)__cvta_generic_to_shared(wd + k * U3_G + ch),
                      ok ? a.k5 + (int64_t)(g0 + ch) * 500 + k : a.k5, ok);
        }
    };
    stage_weights(0, 0);
    // the band of every T4 plane (rows are global T4 rows; zero outside the chunk's rows)
    for (int s = tid; s < gm.stage; s += U3_THREADS) {
        int64_t gr, gc;
        if (gm.narrow) {
            const int64_t q = p0 + s;
            gr = a.out_row0 + q / gm.pitch;
            gc = q % gm.pitch;
        } else {
            const int rr = s / U3W_PITCH;
            gr = r0 + rr;
            gc = c0 + (s - rr * U3W_PITCH);
        }
        const int64_t br = gr - a.t4_row0;
        const bool ok = br >= 0 && br < a.t4_rows && gc < a.w4;
        const float* src = ok ? t4b + br * a.w4 + gc : a.t4;
        const uint32_t dst = (uint32_t)__cvta_generic_to_shared(xs + s);
#pragma unroll 4
        for (int ci = 0; ci < 20; ++ci) cp_async4(dst + 4u * ci * gm.cs, ok ? src + ci * plane : src, ok);
    }
    cp_async_commit();
    for (int idx = tid; idx < n5p * 12; idx += U3_THREADS) {
        const int ch = idx / 12, o = idx - ch * 12;
        k6s[idx] = (ch < n5 && o < 9) ? __ldg(a.k6 + o * n5 + ch) : 0.f;
    }

    float c6[9][U3_P];
#pragma unroll
    for (int o = 0; o < 9; ++o)
#pragma unroll
        for (int p = 0; p < U3_P; ++p) c6[o][p] = 0.f;

    const int ngroups = n5p / U3_G;
    for (int gi = 0; gi < ngroups; ++gi) {
        const int g0 = gi * U3_G;
        cp_async_wait_all();
        __syncthreads();  // weights of group gi (and the band) visible; group gi-1 fully consumed
        if (gi + 1 < ngroups) stage_weights(g0 + U3_G, (gi + 1) & 1);
        cp_async_commit();
        // this group's bias values (their latency hides behind the tap loop)
        float bv[U3_G][U3_P];
#pragma unroll
        for (int c = 0; c < U3_G; ++c) {
            const int ch = min(g0 + c, n5 - 1);
#pragma unroll
            for (int p = 0; p < U3_P; ++p) {
                if (a.b5_plane)
                    bv[c][p] = (row_ok && C5 + p < a.w5)
                                   ? __ldg(a.b5 + ((int64_t)ch * a.b5_rows + (R5 - a.b5_row0)) * a.w5 + C5 + p)
                                   : 0.f;
                else
                    bv[c][p] = __ldg(a.b5 + ch);
            }
        }
        const float* wg = ws + (gi & 1) * (20 * 25 * U3_G);
        float2 acc2[U3_G / 2][U3_P];  // channel pairs, FFMA2
#pragma unroll
        for (int c = 0; c < U3_G / 2; ++c)
#pragma unroll
            for (int p = 0; p < U3_P; ++p) acc2[c][p] = make_float2(0.f, 0.f);
#pragma unroll 1
        for (int ci = 0; ci < 20; ++ci) {
#pragma unroll
            for (int i = 0; i < 5; ++i) {
                float x[8];
                const float4* xr = reinterpret_cast<const float4*>(&xs[ci * gm.cs + sb + i * gm.pitch]);
                const float4 x0 = xr[0], x1 = xr[1];
                x[0] = x0.x; x[1] = x0.y; x[2] = x0.z; x[3] = x0.w;
                x[4] = x1.x; x[5] = x1.y; x[6] = x1.z; x[7] = x1.w;
#pragma unroll
                for (int kj = 0; kj < 5; ++kj) {
                    const float4* wr = reinterpret_cast<const float4*>(&wg[((ci * 25) + i * 5 + kj) * U3_G]);
                    const float4 wa = wr[0], wb = wr[1];
                    const float2 wv[4] = {make_float2(wa.x, wa.y), make_float2(wa.z, wa.w), make_float2(wb.x, wb.y),
                                          make_float2(wb.z, wb.w)};
#pragma unroll
                    for (int c = 0; c < U3_G / 2; ++c)
#pragma unroll
                        for (int p = 0; p < U3_P; ++p)
                            acc2[c][p] = __ffma2_rn(make_float2(x[p + kj], x[p + kj]), wv[c], acc2[c][p]);
                }
            }
        }
        // bias + tanh, then this group's share of the 1x1 C6 dot products (padded channels
        // have zero C6 weights, so they add exact zeros)
#pragma unroll
        for (int c = 0; c < U3_G; ++c) {
            const float4* k6r = reinterpret_cast<const float4*>(&k6s[(g0 + c) * 12]);
            const float4 ka = k6r[0], kb = k6r[1], kc = k6r[2];
            const float kw[9] = {ka.x, ka.y, ka.z, ka.w, kb.x, kb.y, kb.z, kb.w, kc.x};
#pragma unroll
            for (int p = 0; p < U3_P; ++p) {
                const float av = (c & 1) ? acc2[c >> 1][p].y : acc2[c >> 1][p].x;
                const float t = tanh_f(av + bv[c][p]);
#pragma unroll
                for (int o = 0; o < 9; ++o) c6[o][p] = fmaf(kw[o], t, c6[o][p]);
            }
        }
    }
    if (!row_ok) return;
    float* ob = a.out + img * a.out_img_stride + (R5 - a.out_row0) * a.w5;
#pragma unroll
    for (int o = 0; o < 9; ++o)
#pragma unroll
        for (int p = 0; p < U3_P; ++p) {
            const int64_t c = C5 + p;
            if (c >= a.w5) continue;
            const float b = a.b6_plane ? __ldg(a.b6 + ((int64_t)o * a.b6_rows + (R5 - a.b6_row0)) * a.w5 + c)
                                       : __ldg(a.b6 + o);
            ob[o * a.out_plane_stride + c] = c6[o][p] + b;
        }
}

}  // namespace

cudaError_t launch_cnn_u1(const CnnU1Args& a, cudaStream_t s) {
    if (a.t2_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    U1W w;
    for (int ch = 0; ch < 8; ++ch)
        for (int t = 0; t < 25; ++t) w.k1[t][ch] = a.k1_host[ch * 25 + t];
    std::memcpy(w.p2, a.p2_host, sizeof w.p2);
    // TMA path: 16-byte aligned rows (W % 4 == 0 makes w1, w2 even and w1 % 4 == 0),
    // images at a uniform stride of whole rows
    const int64_t in_rows = a.W > 0 ? a.in_img_stride / a.W : 0;
    const bool tma_ok = (a.W & 3) == 0 && (reinterpret_cast<uintptr_t>(a.in) & 15) == 0 &&
                        in_rows * a.W == a.in_img_stride && (!a.b1_plane || (reinterpret_cast<uintptr_t>(a.b1) & 15) == 0) &&
                        (a.bf16_out || (reinterpret_cast<uintptr_t>(a.t2) & 7) == 0) && in_rows < (1ll << 31) &&
                        a.nimg < (1ll << 31);
    if (tma_ok) {
        CUtensorMap xm, bm;
        bool ok = tma_make_3d(&xm, a.in, (uint64_t)a.W, (uint64_t)in_rows, (uint64_t)a.nimg, (uint64_t)a.W * 4,
                              (uint64_t)a.in_img_stride * 4, U1T_IC, U1T_IR, 1);
        if (ok && a.b1_plane)
            ok = tma_make_3d(&bm, a.b1, (uint64_t)a.w1, (uint64_t)a.b1_rows, 8, (uint64_t)a.w1 * 4,
                             (uint64_t)a.b1_rows * a.w1 * 4, U1T_BC, U1T_BR, 8);
        else
            bm = xm;  // unused
        if (ok) {
            const int tiles_c = (int)((a.w2 + U1T_C - 1) / U1T_C);
            const int tiles_r = (int)((a.t2_rows + U1T_R - 1) / U1T_R);
            const int64_t ntiles = (int64_t)tiles_c * tiles_r * a.nimg;
            if (ntiles >= (1ll << 32)) return cudaErrorInvalidValue;  // 32-bit tile indexing in the kernel
            int dev = 0, sms = 148;
            cudaGetDevice(&dev);
            cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
            // 32 CTAs per SM in the grid (3 resident): the extra CTAs balance the tail of the static
            // tile walk (3 per SM -> 32: U1 0.160 -> 0.148 ms bf16, 0.207 -> 0.191 ms fp32 on cnn3)
            const int64_t grid = std::min<int64_t>(ntiles, 32 * (int64_t)sms);
            const size_t smem = 2 * (size_t)U1T_STAGE + 128;
            auto go = [&](auto kern) -> cudaError_t {
                cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
                if (e != cudaSuccess) return e;
                kern<<<(unsigned)grid, 128, smem, s>>>(xm, bm, a, w, tiles_c, tiles_r, ntiles);
                return cudaGetLastError();
            };
            if (a.bf16_out)
                return a.b1_plane ? go(cnn_u1_tma_kernel<true, true>) : go(cnn_u1_tma_kernel<true, false>);
            return a.b1_plane ? go(cnn_u1_tma_kernel<false, true>) : go(cnn_u1_tma_kernel<false, false>);
        }
    }
    dim3 grid((unsigned)((a.w2 + U1_TC - 1) / U1_TC), (unsigned)((a.t2_rows + U1_TR - 1) / U1_TR), (unsigned)a.nimg);
    if (a.bf16_out)
        cnn_u1_kernel<true><<<grid, 128, 0, s>>>(a, w);
    else
        cnn_u1_kernel<false><<<grid, 128, 0, s>>>(a, w);
    return cudaGetLastError();
}

cudaError_t launch_cnn_u2(const CnnU2Args& a, cudaStream_t s) {
    if (a.t4_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    U2W w;
    for (int co = 0; co < 20; ++co)
        for (int ci = 0; ci < 8; ++ci)
            for (int t = 0; t < 25; ++t) w.k3[ci][t][co] = a.k3_host[(co * 8 + ci) * 25 + t];
    std::memcpy(w.p4, a.p4_host, sizeof w.p4);
    const size_t smem = sizeof(float) * (8 * U2_IR * U2_IC + (a.b3_plane ? 20 * U2_BR * U2_BC : 0));
    static std::atomic<uint32_t> configured{0};  // one bit per device
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(configured.load() & (1u << (dev & 31)))) {
        cudaError_t e = cudaFuncSetAttribute(cnn_u2_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)(sizeof(float) * (8 * U2_IR * U2_IC + 20 * U2_BR * U2_BC)));
        if (e != cudaSuccess) return e;
        configured.fetch_or(1u << (dev & 31));
    }
    dim3 grid((unsigned)((a.w4 + U2_TC - 1) / U2_TC), (unsigned)((a.t4_rows + U2_TR - 1) / U2_TR), (unsigned)a.nimg);
    cnn_u2_kernel<<<grid, 128, smem, s>>>(a, w);
    return cudaGetLastError();
}

cudaError_t launch_cnn_u3(const CnnU3Args& a, cudaStream_t s) {
    if (a.out_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    const int n5p = (a.n5 + U3_G - 1) / U3_G * U3_G;
    // geometry: flattened items when the padded row fits and wastes less than 64-column tiles
    U3Geom gm{};
    const int64_t pitch = (a.w4 + 3) / 4 * 4;
    const int64_t narrow_items = (a.out_rows * pitch + U3_POS - 1) / U3_POS;
    const int64_t tiles_c = (a.w5 + U3W_TC - 1) / U3W_TC;
    const int64_t wide_items = (a.out_rows + U3W_TR - 1) / U3W_TR * tiles_c;
    if (pitch <= U3_NARROW_MAX_PITCH && narrow_items <= wide_items) {
        gm.narrow = 1;
        gm.pitch = (int)pitch;
        gm.stage = (int)(U3_POS + 4 * pitch + 8);
        gm.cs = gm.stage;
        gm.items_per_img = narrow_items;
    } else {
        gm.narrow = 0;
        gm.pitch = U3W_PITCH;
        gm.stage = (U3W_TR + 4) * U3W_PITCH;
        gm.cs = gm.stage;
        gm.tiles_c = (int)tiles_c;
        gm.items_per_img = wide_items;
    }
    const size_t smem = sizeof(float) * ((size_t)20 * gm.cs + 2 * 20 * 25 * U3_G + (size_t)n5p * 12);
    static std::atomic<uint32_t> configured{0};  // one bit per device
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(configured.load() & (1u << (dev & 31)))) {
        cudaError_t e = cudaFuncSetAttribute(cnn_u3_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
        if (e != cudaSuccess) return e;
        configured.fetch_or(1u << (dev & 31));
    }
    if (smem > 227 * 1024) return cudaErrorInvalidValue;
    const int64_t grid = gm.items_per_img * a.nimg;
    if (grid >= (1ll << 31)) return cudaErrorInvalidValue;
    cnn_u3_kernel<<<(unsigned)grid, U3_THREADS, smem, s>>>(a, gm);
    return cudaGetLastError();
}

}  // namespace tg
