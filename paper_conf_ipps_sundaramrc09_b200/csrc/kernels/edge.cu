// edge.cu -- K1, the fused edge-detection offload unit for sm_100a.
//
// Computes the whole 4-orientation edge template of PAPER.md:629 (Fig. 3 graph:
// C1: E1 = Im*K1, C2: E2 = Im*K2, R1: E5 = -E1, R2: E6 = -E2, max: E = max(E1,E2,E5,E6))
// in ONE pass over a chunk, so E1, E2, E5, E6 never leave registers -- the paper's "best
// possible" configuration. The same kernel takes up to 4 convolutions (the
// 8-orientation graph of Fig. 1(b)) and the other combine ops of PAPER.md:621 (addition,
// max absolute value). SAME zero padding with anchor (ks-1)/2
// (R2); a ks x ks kernel (ks <= 16) is embedded in a 16 x 16 frame at offset
// 7 - (ks-1)/2 so one code path serves every size. The tap loops are specialised on the
// frame kF in {4, 8, 16}: a ks <= kF kernel has all its nonzero taps inside the centred
// kF x kF window [8 - kF/2, 8 + kF/2) of the 16 x 16 frame, so only those taps are issued
// (Fig. 2's small kernels cost (kF/16)^2 of the 16 x 16 work instead of all of it).
//
// Roofline: 2 x 256 FMA per output pixel vs 8 HBM bytes -> FP32-ALU
// bound (128 flop/B >> ridge ~11 flop/B). The kernel is organised to keep the FMA pipe busy:
// each thread owns a 1 x 16 strip of outputs; per filter row it loads its 32-wide input
// window with 8 conflict-free LDS.128 and issues 256 FFMA2 (paired FP32 FMA, sm_100) that
// update BOTH filters' accumulators at once: (E1[q], E2[q]) += x[q+j+1] * (K1[i][j], K2[i][j]),
// the x operand broadcast from one register and the weight pair a uniform register loaded
// from the constant bank (__grid_constant__ parameter). Tiles of 64 x 64 outputs, 256
// threads; lanes of a warp own 32 consecutive rows (row pitch 84 floats = 21 x 16 B, odd,
// so the 8 lanes of each LDS.128 phase hit 8 distinct 16-byte bank groups).
//
// Tile staging. Main path (W % 4 == 0): a grid of 32 CTAs per SM (3 resident at a time; the
// rest take the place of CTAs that finish early, which balances the tail) walks the tiles;
// one thread issues a 3-D TMA load (cp.async.bulk.tensor, box 84 x 79 x 1) of the NEXT
// tile into the other shared-memory buffer while the CTA computes the current one, and the
// TMA's out-of-bounds zero fill is exactly the SAME padding at image borders. Fallback
// (any W): each CTA stages its tile with bounds-checked 128-bit loads.
//
// Bit-exactness under splitting: every output pixel is the same sequence of fmaf in the
// same order (filter row i, then column j) whatever tile or chunk it falls in.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <mutex>

#include "kernels.h"
#include "tma_util.cuh"

namespace tg {
namespace {

// Tile geometries kG (Q = outputs per thread, one row of Q columns):
//   kG = 16: 64 x 64 output tiles, 8 warps = 2 row groups x 4 column strips, Q = 16 (the main path);
//   kG = 4:  32 x 32 output tiles, 8 warps = 8 column strips of one 32-row group, Q = 4 -- for images
//            with fewer 64 x 64 tiles than SMs (16 big tiles of a 256 x 256 image would leave 132
//            SMs idle and make each thread's 4096 serial FFMA2 the latency);
//   kG = 5:  16 x 32 output tiles, 4 warps (lanes 0-15 / 16-31 = two column strips of the same 16
//            rows), Q = 4 -- when even the 32 x 32 tiles are fewer than the SMs (configs[0]: 128
//            tiles of 16 x 32 on 148 SMs, one warp per SM sub-partition, instead of 64 of 32 x 32).
// Row pitch in shared memory: an odd number of 16-byte units, so the 8 lanes of each LDS.128
// phase (lanes = consecutive rows) hit 8 distinct bank groups.
template <int kG> struct Geo;
template <> struct Geo<16> {
    static constexpr int R = 64, C = 64, Pitch = 84, Q = 16, Threads = 256;  // 84 / 4 = 21
    __device__ static int lr(int warp, int lane) { return (warp >> 2) * 32 + lane; }
    __device__ static int cb(int warp, int) { return (warp & 3) * 16; }
};
template <> struct Geo<4> {
    static constexpr int R = 32, C = 32, Pitch = 52, Q = 4, Threads = 256;  // 52 / 4 = 13
    __device__ static int lr(int, int lane) { return lane; }
    __device__ static int cb(int warp, int) { return warp * 4; }
};
template <> struct Geo<5> {
    static constexpr int R = 16, C = 32, Pitch = 52, Q = 4, Threads = 128;  // 52 / 4 = 13
    __device__ static int lr(int, int lane) { return lane & 15; }
    __device__ static int cb(int warp, int lane) { return (2 * warp + (lane >> 4)) * 4; }
};
template <int kG> struct GeoT : Geo<kG> {
    static constexpr int SmR = Geo<kG>::R + 15;                  // rows incl. halo
    static constexpr int SmC = Geo<kG>::C + 16;                  // cols used: [c0-8, c0+C+8)
    static constexpr int TileBytes = SmR * Geo<kG>::Pitch * 4;   // one TMA box
    static constexpr int BufStride = (TileBytes + 127) / 128 * 128;
};
constexpr int kThreads = 256;  // the fallback kernel (geometry 16)

// Both filters, embedded in 16 x 16 frames, travel as a __grid_constant__ kernel parameter:
// the weights then sit in the constant bank and every FFMA reads them through a uniform
// register (FFMA R, R, UR, R) -- only two vector-register operands per FFMA, which keeps
// the register-file banks out of the way of the FMA pipe.
struct EdgeWeights {
    float2 w[2][256];  // filter pairs (2p, 2p+1) interleaved per tap: one FFMA2 weight operand
};

// Compute the output tile whose input (+halo) is staged at xs (row pitch Geo<kQ>::Pitch; smem
// (sr, sc) <-> image (tile_r0 - 7 + sr, tile_c0 - 8 + sc)) and store it.
template <int kComb, int kPairs, int kF, int kG>
__device__ __forceinline__ void edge_tile(const float* __restrict__ xs, const EdgeArgs& a, const EdgeWeights& wt,
                                          int64_t img, int64_t tile_r0, int64_t tile_c0) {
    constexpr int kPitch = Geo<kG>::Pitch, kQ = Geo<kG>::Q;
    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int lr = Geo<kG>::lr(warp, lane);     // local output row
    const int cb = Geo<kG>::cb(warp, lane);     // local output column base

    // Paired FP32 FMA (FFMA2, sm_100) over a PAIR OF FILTERS: acc[q] = (E_2p[q], E_2p+1[q]) +=
    // x[q+j+1] (register, broadcast to both lanes) * (K_2p[i][j], K_2p+1[i][j]) (uniform-register
    // pair from the constant bank). Each lane rounds exactly like fmaf, in the same (i, j) order
    // as a scalar loop. Filter pairs run one after the other over the same staged tile, and the
    // combine op folds each pair into e[] (8 orientations = 4 convolutions = 2 pairs).
    float e[kQ];
#pragma unroll
    for (int q = 0; q < kQ; ++q) e[q] = 0.f;
#pragma unroll
    for (int fp = 0; fp < kPairs; ++fp) {  // compile-time: constant-bank weight offsets
        float2 acc[kQ];
#pragma unroll
        for (int q = 0; q < kQ; ++q) acc[q] = make_float2(0.f, 0.f);
        constexpr int kOff = 8 - kF / 2;  // first tap row/column of the kF x kF window
#pragma unroll 1
        for (int i = kOff; i < kOff + kF; ++i) {
            // input window: smem cols [cb, cb+kQ+16) <-> image cols [c0+cb-8, c0+cb+kQ+8);
            // output column c0+cb+q, tap j reads image col c0+cb+q+j-7 = smem col cb+q+j+1
            float x[kQ + 16];
            const float4* xr = reinterpret_cast<const float4*>(&xs[(lr + i) * kPitch + cb]);
#pragma unroll
            for (int v = 0; v < (kQ + 16) / 4; ++v) {
                const float4 t = xr[v];
                x[4 * v + 0] = t.x;
                x[4 * v + 1] = t.y;
                x[4 * v + 2] = t.z;
                x[4 * v + 3] = t.w;
            }
#pragma unroll
            for (int j = kOff; j < kOff + kF; ++j) {
                const float2 w = wt.w[fp][i * 16 + j];
#pragma unroll
                for (int q = 0; q < kQ; ++q)
                    acc[q] = __ffma2_rn(make_float2(x[q + j + 1], x[q + j + 1]), w, acc[q]);
            }
        }
        // combine (x > m) ? x : m folds; sum = left fold of fp32 adds
        const bool has2 = 2 * fp + 1 < a.nf;
#pragma unroll
        for (int q = 0; q < kQ; ++q) {
            const float e1 = acc[q].x, e2 = acc[q].y;
            float m = e[q];
            switch (kComb) {
                case 1:  // SUM
                    m = fp == 0 ? e1 : m + e1;
                    if (has2) m = m + e2;
                    break;
                case 2:  // MAXABS
                    m = fp == 0 ? fabsf(e1) : ((fabsf(e1) > m) ? fabsf(e1) : m);
                    if (has2) m = (fabsf(e2) > m) ? fabsf(e2) : m;
                    break;
                case 3:  // plain max of the responses
                    m = fp == 0 ? e1 : ((e1 > m) ? e1 : m);
                    if (has2) m = (e2 > m) ? e2 : m;
                    break;
                default:  // MAX over the responses and their remaps (negations): E1, E2, -E1, -E2
                    m = fp == 0 ? e1 : ((e1 > m) ? e1 : m);
                    if (has2) m = (e2 > m) ? e2 : m;
                    m = (-e1 > m) ? -e1 : m;
                    if (has2) m = (-e2 > m) ? -e2 : m;
            }
            e[q] = m;
        }
    }

    const int64_t row = tile_r0 + lr;
    if (row >= a.out_row0 + a.out_rows) return;
    float* orow = a.out + img * a.out_img_stride + (row - a.out_row0) * a.W;
    const int64_t c0 = tile_c0 + cb;
    const bool ovec = (a.W & 3) == 0 && ((reinterpret_cast<uintptr_t>(a.out) & 15) == 0) &&
                      (a.out_img_stride & 3) == 0;
    if (ovec && c0 + kQ - 1 < a.W) {
#pragma unroll
        for (int v = 0; v < kQ / 4; ++v)
            *reinterpret_cast<float4*>(orow + c0 + 4 * v) =
                make_float4(e[4 * v], e[4 * v + 1], e[4 * v + 2], e[4 * v + 3]);
    } else {
#pragma unroll
        for (int q = 0; q < kQ; ++q)
            if (c0 + q < a.W) orow[c0 + q] = e[q];
    }
}

// ---------------------------------------------------------------------------- fallback
template <int kComb, int kPairs, int kF>
__global__ void __launch_bounds__(kThreads, 2)
    edge_fused_kernel(const EdgeArgs a, const __grid_constant__ EdgeWeights wt) {
    using G = GeoT<16>;
    constexpr int kTileR = G::R, kTileC = G::C, kSmR = G::SmR, kSmC = G::SmC, kPitch = G::Pitch;
    __shared__ __align__(16) float xs[kSmR * kPitch];
    const int tid = threadIdx.x;
    const int64_t img = blockIdx.z;
    const int64_t tile_r0 = a.out_row0 + (int64_t)blockIdx.y * kTileR;  // global output row
    const int64_t tile_c0 = (int64_t)blockIdx.x * kTileC;
    const float* __restrict__ inb = a.in + img * a.in_img_stride;
    const bool vec = (a.W & 3) == 0 && ((reinterpret_cast<uintptr_t>(a.in) & 15) == 0) &&
                     (a.in_img_stride & 3) == 0;
    for (int idx = tid; idx < kSmR * (kSmC / 4); idx += kThreads) {
        const int sr = idx / (kSmC / 4);
        const int q = idx - sr * (kSmC / 4);
        const int64_t g = tile_r0 - 7 + sr;
        const int64_t gc = tile_c0 - 8 + 4 * q;
        float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
        if (g >= 0 && g < a.H && g >= a.in_row0 && g < a.in_row0 + a.in_rows) {
            const float* row = inb + (g - a.in_row0) * a.W;
            if (vec && gc >= 0 && gc + 3 < a.W) {
                v = __ldg(reinterpret_cast<const float4*>(row + gc));
            } else {
                v.x = (gc + 0 >= 0 && gc + 0 < a.W) ? __ldg(row + gc + 0) : 0.f;
                v.y = (gc + 1 >= 0 && gc + 1 < a.W) ? __ldg(row + gc + 1) : 0.f;
                v.z = (gc + 2 >= 0 && gc + 2 < a.W) ? __ldg(row + gc + 2) : 0.f;
                v.w = (gc + 3 >= 0 && gc + 3 < a.W) ? __ldg(row + gc + 3) : 0.f;
            }
        }
        *reinterpret_cast<float4*>(&xs[sr * kPitch + 4 * q]) = v;
    }
    __syncthreads();
    edge_tile<kComb, kPairs, kF, 16>(xs, a, wt, img, tile_r0, tile_c0);
}

// ---------------------------------------------------------------------------- TMA path
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

template <int kComb, int kPairs, int kF, int kG>
__global__ void __launch_bounds__(Geo<kG>::Threads, 2)
    edge_fused_tma_kernel(const __grid_constant__ CUtensorMap tmap, const EdgeArgs a,
                          const __grid_constant__ EdgeWeights wt, const int tiles_c, const int tiles_r,
                          const int64_t ntiles) {
    using G = GeoT<kG>;
    constexpr int kTileR = G::R, kTileC = G::C, kTileBytes = G::TileBytes, kBufStride = G::BufStride;
    // (the tensor map must sit in the first 4 KB of the parameter space, hence first)
    extern __shared__ __align__(128) uint8_t smraw[];
    // two tile buffers at 128-byte aligned shared-memory addresses
    uint8_t* base = smraw + ((128 - (smem_u32(smraw) & 127)) & 127);
    float* buf0 = reinterpret_cast<float*>(base);                   // TMA stage 0
    float* buf1 = reinterpret_cast<float*>(base + kBufStride);      // TMA stage 1
    __shared__ __align__(8) uint64_t full[2];
    const int tid = threadIdx.x;
    if (tid == 0) {
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&tmap)) : "memory");
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(smem_u32(&full[0])) : "memory");
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(smem_u32(&full[1])) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    __syncthreads();
    // tile -> (image, first row, first column) in 32-bit arithmetic (the launcher checks that the
    // tile count fits; 64-bit division is a long software sequence)
    const uint32_t per_img = (uint32_t)tiles_c * (uint32_t)tiles_r;
    auto coords = [&](int64_t t, int64_t& img, int64_t& tr0, int64_t& tc0) {
        const uint32_t tu = (uint32_t)t, im = tu / per_img, rem = tu - im * per_img, ty = rem / (uint32_t)tiles_c;
        img = im;
        tr0 = a.out_row0 + (int64_t)ty * kTileR;
        tc0 = (int64_t)(rem - ty * (uint32_t)tiles_c) * kTileC;
    };
    auto issue = [&](int64_t t, int b) {
        int64_t img, tr0, tc0;
        coords(t, img, tr0, tc0);
        // box origin: image col tc0 - 8, buffer row (tr0 - 7) - in_row0 (out-of-range -> zeros)
        const int x = (int)(tc0 - 8), y = (int)(tr0 - 7 - a.in_row0), z = (int)img;
        float* dst = b ? buf1 : buf0;
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(&full[b])),
                     "r"(kTileBytes)
                     : "memory");
        // (TMA box origins must be 16-byte aligned, so the one-column shift for the FFMA2
        // pairs is made in shared memory after the tile lands)
        for (int h = 0; h < 1; ++h)
            asm volatile(
                "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
                "%4}], [%5];\n" ::"r"(smem_u32(dst) + (uint32_t)(h * kBufStride)),
                "l"(reinterpret_cast<uint64_t>(&tmap)), "r"(x), "r"(y), "r"(z), "r"(smem_u32(&full[b]))
                : "memory");
    };
    int64_t t = blockIdx.x;
    if (tid == 0 && t < ntiles) issue(t, 0);
    for (int k = 0; t < ntiles; ++k, t += gridDim.x) {
        const int b = k & 1;
        if (tid == 0 && t + gridDim.x < ntiles) issue(t + gridDim.x, b ^ 1);  // prefetch the next tile
        const uint32_t parity = (uint32_t)((k >> 1) & 1);
        asm volatile(
            "{\n\t.reg .pred done;\n\t"
            "WAIT_%=:\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 done, [%0], %1;\n\t"
            "@!done bra WAIT_%=;\n\t}\n" ::"r"(smem_u32(&full[b])),
            "r"(parity)
            : "memory");
        int64_t img, tr0, tc0;
        coords(t, img, tr0, tc0);
        const float* tb = b ? buf1 : buf0;
        edge_tile<kComb, kPairs, kF, kG>(tb, a, wt, img, tr0, tc0);
        __syncthreads();  // buffer b is free for the prefetch issued in iteration k+1
    }
}

}  // namespace

PFN_cuTensorMapEncodeTiled_v12000 tma_encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    });
    return fn;
}

template <int kComb, int kPairs, int kF>
cudaError_t launch_edge_t(const EdgeArgs& a, cudaStream_t s);

template <int kPairs, int kF>
cudaError_t launch_edge_p(const EdgeArgs& a, cudaStream_t s) {
    switch (a.combine) {
        case 0: return launch_edge_t<0, kPairs, kF>(a, s);
        case 1: return launch_edge_t<1, kPairs, kF>(a, s);
        case 2: return launch_edge_t<2, kPairs, kF>(a, s);
        case 3: return launch_edge_t<3, kPairs, kF>(a, s);
        default: return cudaErrorInvalidValue;
    }
}

template <int kF>
cudaError_t launch_edge_f(const EdgeArgs& a, cudaStream_t s) {
    return a.nf <= 2 ? launch_edge_p<1, kF>(a, s) : launch_edge_p<2, kF>(a, s);
}

cudaError_t launch_edge(const EdgeArgs& a, cudaStream_t s) {
    if (a.nf < 1 || a.nf > 4 || a.ks < 1 || a.ks > 16) return cudaErrorInvalidValue;
    if (a.ks <= 4) return launch_edge_f<4>(a, s);
    if (a.ks <= 8) return launch_edge_f<8>(a, s);
    return launch_edge_f<16>(a, s);
}

// The TMA path in tile geometry kG; cudaErrorNotSupported when the tensor map cannot be encoded
// (the caller then takes the bounds-checked fallback kernel).
template <int kComb, int kPairs, int kF, int kG>
cudaError_t launch_edge_tma(const EdgeArgs& a, const EdgeWeights& wt, PFN_cuTensorMapEncodeTiled_v12000 enc, int dev,
                            int sms, cudaStream_t s) {
    using G = GeoT<kG>;
    const int tiles_c = (int)((a.W + G::C - 1) / G::C);
    const int tiles_r = (int)((a.out_rows + G::R - 1) / G::R);
    CUtensorMap tmap;
    const cuuint64_t gdim[3] = {(cuuint64_t)a.W, (cuuint64_t)a.in_rows, (cuuint64_t)a.nimg};
    const cuuint64_t gstride[2] = {(cuuint64_t)a.W * 4, (cuuint64_t)a.in_rows * a.W * 4};
    const cuuint32_t box[3] = {(cuuint32_t)G::Pitch, (cuuint32_t)G::SmR, 1};
    const cuuint32_t estride[3] = {1, 1, 1};
    CUresult r = enc(&tmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<float*>(a.in), gdim, gstride, box, estride,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return cudaErrorNotSupported;
    static std::atomic<uint32_t> configured{0};
    const size_t smem = 2 * (size_t)G::BufStride + 128;
    if (!(configured.load() & (1u << (dev & 31)))) {
        cudaError_t e = cudaFuncSetAttribute(edge_fused_tma_kernel<kComb, kPairs, kF, kG>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        configured.fetch_or(1u << (dev & 31));
    }
    const int64_t ntiles = (int64_t)tiles_c * tiles_r * a.nimg;
    if (ntiles >= (1ll << 32)) return cudaErrorInvalidValue;  // 32-bit tile indexing in the kernel
    // 32 CTAs per SM in the grid (3 are resident at a time): CTAs that finish early pick up
    // the remaining ones, which balances the tail of the static tile walk -- 2 per SM
    // (exactly resident) ran at 0.918 of the FP32 peak, 8 at 0.936, 32 at 0.941
    const int64_t grid = std::min<int64_t>(ntiles, 32 * (int64_t)sms);
    edge_fused_tma_kernel<kComb, kPairs, kF, kG><<<(unsigned)grid, G::Threads, smem, s>>>(tmap, a, wt, tiles_c, tiles_r, ntiles);
    return cudaGetLastError();
}

template <int kComb, int kPairs, int kF>
cudaError_t launch_edge_t(const EdgeArgs& a, cudaStream_t s) {
    if (a.out_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    // filters embedded in a 16 x 16 frame at offset 7 - (ks-1)/2 (zeros elsewhere)
    if (a.nf < 1 || a.nf > 4) return cudaErrorInvalidValue;
    EdgeWeights wt{};
    const int off = 7 - (a.ks - 1) / 2;
    for (int f = 0; f < a.nf; ++f)
        for (int r = 0; r < a.ks; ++r)
            for (int c = 0; c < a.ks; ++c) {
                float2& w = wt.w[f >> 1][(r + off) * 16 + c + off];
                (f & 1 ? w.y : w.x) = a.k_host[f][r * a.ks + c];
            }
    PFN_cuTensorMapEncodeTiled_v12000 enc = tma_encode_fn();
    const bool tma_ok = enc && (a.W & 3) == 0 && (reinterpret_cast<uintptr_t>(a.in) & 15) == 0 &&
                        a.in_img_stride == a.in_rows * a.W && a.in_rows < (1ll << 31) && a.W < (1ll << 31);
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t big_tiles = ((a.W + 63) / 64) * ((a.out_rows + 63) / 64) * a.nimg;
    const int64_t mid_tiles = ((a.W + 31) / 32) * ((a.out_rows + 31) / 32) * a.nimg;
    if (tma_ok) {
        // smaller tiles when the big ones cannot occupy every SM
        cudaError_t e = big_tiles >= sms   ? launch_edge_tma<kComb, kPairs, kF, 16>(a, wt, enc, dev, sms, s)
                        : mid_tiles >= sms ? launch_edge_tma<kComb, kPairs, kF, 4>(a, wt, enc, dev, sms, s)
                                           : launch_edge_tma<kComb, kPairs, kF, 5>(a, wt, enc, dev, sms, s);
        if (e != cudaErrorNotSupported) return e;
    }
    using G = GeoT<16>;
    const int tiles_c = (int)((a.W + G::C - 1) / G::C);
    const int tiles_r = (int)((a.out_rows + G::R - 1) / G::R);
    dim3 grid((unsigned)tiles_c, (unsigned)tiles_r, (unsigned)a.nimg);
    if (grid.y > 65535 || grid.z > 65535) return cudaErrorInvalidConfiguration;
    edge_fused_kernel<kComb, kPairs, kF><<<grid, kThreads, 0, s>>>(a, wt);
    return cudaGetLastError();
}

}  // namespace tg
