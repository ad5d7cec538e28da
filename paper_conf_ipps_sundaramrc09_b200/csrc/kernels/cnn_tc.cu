// cnn_tc.cu -- CNN units U2 (C3 T S4 T) and U3 (C5 T C6) as tcgen05 implicit GEMMs (sm_100a).
//
// The multi-channel layers of the CNN are dense contractions:
// C3: per output pixel 8 input planes x 25 taps -> 20 maps; C5: 20 x 25 -> n5 maps. Here the
// pixels of a band are the MMA's M dimension (two M=128 tiles), output maps the N dimension,
// and (input plane, tap) the K dimension, accumulated in TMEM (fp32) from bf16 operands.
//
// Implicit GEMM without an im2col buffer: the band's input window is staged ONCE in shared
// memory as K-major core matrices with one pixel per 16-byte row ([channel-block][row][col][8
// channels], bf16). A tap (i, j) is then the same matrix shifted by i*pitch + j rows, i.e. just
// another descriptor start address. Channel blocks that are not full (C3: 8 channels; C5: the
// last 4 of 20) are paired ACROSS taps: a K=16 step whose second half has LBO = 16 bytes reads
// the next pixel's channels, i.e. tap (i, j+1) -- so C3 needs 15 K-steps (not 25 x 16-wide)
// and C5 40 (not 50 with a 12-channel zero pad).
//
// Both kernels are persistent and warp-specialised: one thread issues the bulk copies (TMA
// engine) and the MMAs, epilogue warps drain TMEM (tcgen05.ld 32x32b): bias plane + tanh, then
//   U2: the 2x2 subsample pairs row 2R (tile 0) with row 2R+1 (tile 1) in the same thread and
//       columns c, c+1 across neighbouring lanes (shfl), + tanh -> T4 (bf16 channel blocks);
//   U3: the 1x1 C6 layer as a dot product over n5 in registers, + bias -> output (fp32).
// Precision: bf16 operands, fp32 accumulation; parity bound 2e-2 normwise (R16).
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstring>
#include <vector>

#include "kernels.h"
#include "tc_sm100.cuh"

#ifndef U2_EXP
#define U2_EXP 0
#endif
#ifndef U3_EXP
#define U3_EXP 0
#endif
namespace tg {
namespace {

// MUFU tanh (max relative error ~2^-11): used on the bf16 tensor-core path only, whose parity
// bound is 2e-2 normwise (the fp32 path keeps the < 3e-7 formula above)
__device__ __forceinline__ float tanh_approx(float x) {
    float y;
    asm("tanh.approx.f32 %0, %1;\n" : "=f"(y) : "f"(x));
    return y;
}

constexpr int kTileM = 128;

// ============================================================================ U2 (C3)
// Segment = T4 row R (C3 rows 2R, 2R+1) x 128 C3 columns [c0, c0+128): tile 0 = C3 row 2R,
// tile 1 = row 2R+1 (M = 128 each, N = 32: 20 maps padded). Window: T2 rows [2R, 2R+6) x
// cols [c0, c0+134), 8 channels per pixel (one 16-byte row each).
// Warp-specialised and persistent (one CTA per SM, 9 warps):
//   warp 8, one thread   producer + MMA issuer: the C3 B operand (15 K-steps) once per CTA by a
//                        bulk copy; per segment six 1-D bulk copies (TMA engine) of the window's
//                        T2 rows into one of U2_NA buffers (prefetched U2_NA-1 segments ahead);
//                        2 tiles x 15 tcgen05.mma into one of 4 TMEM slots; tcgen05.commit frees
//                        the window buffer and hands the slot to the epilogue
//   warps 0-3 / 4-7      epilogue groups for even / odd segments: bias plane (prefetched one
//                        segment ahead), tanh, the 2x2 subsample (rows in the same thread,
//                        columns across neighbouring lanes), tanh -> T4 bf16 channel blocks
constexpr int U2_WR = 6, U2_WP = kTileM + 6;  // +4 taps, +1 for the (4,5) tap pair, +1 spare
constexpr int U2_N = 32;                      // 20 maps padded to 32
constexpr int U2_KS = 15;                     // 5 rows x pairs (0,1) (2,3) (4,5)
constexpr int U2_NA = 8;                      // window buffers
constexpr int U2_NT = 4;                      // TMEM slots (2 per epilogue group)
constexpr int kThreadsU2 = 9 * 32;

struct U2P {
    float p4[20][4];  // S4 weights (constant bank)
};

struct U2Smem {
    uint4 a[U2_NA][U2_WR * U2_WP];  // [row][col] -> 8 bf16 channels
    uint4 b[U2_KS * 2 * U2_N];      // [ks][half][n] -> 8 bf16
    uint64_t b_full, a_full[U2_NA], a_empty[U2_NA], t_full[U2_NT], t_empty[U2_NT];
    uint32_t tmem;
};

__global__ void __launch_bounds__(kThreadsU2, 1)
    cnn_u2_tc_kernel(const CnnU2Args a, const __grid_constant__ U2P pw, const int64_t nseg) {
    extern __shared__ __align__(128) uint8_t smraw[];
    U2Smem& S = *reinterpret_cast<U2Smem*>(smraw + ((128 - (tc::smem_u32(smraw) & 127)) & 127));
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t segs_per_row = (a.w3 + kTileM - 1) / kTileM;
    const int64_t per_img = a.t4_rows * segs_per_row;
    auto seg_coords = [&](int64_t sg, int64_t& img, int64_t& R, int64_t& c0) {
        img = sg / per_img;
        const int64_t rem = sg - img * per_img;
        const int64_t rr = rem / segs_per_row;
        R = a.t4_row0 + rr;
        c0 = (rem - rr * segs_per_row) * kTileM;
    };

    if (warp == 0) tc::tmem_alloc<256>(&S.tmem);
    if (tid == 0) {
        tc::mbar_init(&S.b_full, 1);
        for (int i = 0; i < U2_NA; ++i) {
            tc::mbar_init(&S.a_full[i], 1);
            tc::mbar_init(&S.a_empty[i], 1);
        }
        for (int i = 0; i < U2_NT; ++i) {
            tc::mbar_init(&S.t_full[i], 1);
            tc::mbar_init(&S.t_empty[i], 4);
        }
        tc::mbar_fence_init();
    }
    // windows start zeroed: pixels a copy does not cover (beyond the image) then only ever
    // hold finite T2 values
    for (int idx = tid; idx < U2_NA * U2_WR * U2_WP; idx += kThreadsU2) (&S.a[0][0])[idx] = make_uint4(0u, 0u, 0u, 0u);
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    const uint32_t tmem = S.tmem;
    const int64_t my = nseg > blockIdx.x ? (nseg - 1 - blockIdx.x) / gridDim.x + 1 : 0;

    if (warp == 8) {
        // -------------------------------------------------------------------- producer + MMA
        // (the whole warp runs the loop, so descriptors stay in uniform registers; one elected
        // lane issues the copies, MMAs and commits)
        const uint4* t2all = reinterpret_cast<const uint4*>(a.t2);
        auto load_a = [&](int64_t k) {
            int64_t img, R, c0;
            seg_coords(blockIdx.x + k * gridDim.x, img, R, c0);
            const int buf = (int)(k % U2_NA);
            const int64_t r0 = 2 * R - a.t2_row0;
            const int64_t rows = min((int64_t)U2_WR, a.t2_rows - r0);
            const int64_t cols = min((int64_t)U2_WP, a.w2 - c0);
            if (tc::elect_one()) {
                tc::mbar_expect_tx(&S.a_full[buf], (uint32_t)(rows * cols * 16));
                const uint4* src = t2all + (img * a.t2_rows + r0) * a.w2 + c0;
                for (int r = 0; r < rows; ++r)
                    tc::bulk_g2s(&S.a[buf][r * U2_WP], src + r * a.w2, (uint32_t)(cols * 16), &S.a_full[buf]);
            }
            __syncwarp();
        };
        const uint32_t bbytes = (uint32_t)(U2_KS * 2 * U2_N * 16);
        if (tc::elect_one()) {
            tc::mbar_expect_tx(&S.b_full, bbytes);
            tc::bulk_g2s(S.b, a.k3_tc, bbytes, &S.b_full);
        }
        __syncwarp();
        for (int64_t k = 0; k < U2_NA - 1 && k < my; ++k) load_a(k);
        tc::mbar_wait(&S.b_full, 0);
        const uint32_t idesc = tc::make_idesc_bf16(kTileM, U2_N);
        // descriptors: the start address is the low 14 bits (16-byte units), advanced by adding
        const uint64_t bdesc0 = tc::make_desc(tc::smem_u32(S.b), U2_N * 16, 128);
        const uint64_t adesc0 = tc::make_desc(tc::smem_u32(S.a[0]), 16, 128);  // 2nd K-half = next pixel
        for (int64_t k = 0; k < my; ++k) {
            const int buf = (int)(k % U2_NA), ts = (int)(k % U2_NT);
            tc::mbar_wait(&S.a_full[buf], (uint32_t)((k / U2_NA) & 1));
            if (k >= U2_NT) tc::mbar_wait(&S.t_empty[ts], (uint32_t)(((k - U2_NT) / U2_NT) & 1));
            tc::fence_after_sync();
            const uint64_t abuf = adesc0 + (uint64_t)(buf * (U2_WR * U2_WP));
            const uint32_t d0 = tmem + (uint32_t)(ts * 2 * U2_N);
#if U2_EXP == 2
            if (0)
#endif
            if (tc::elect_one()) {
#pragma unroll
                for (int t = 0; t < 2; ++t) {  // tile t = C3 row 2R + t
#pragma unroll
                    for (int ks = 0; ks < U2_KS; ++ks) {
                        const int i = ks / 3, j = 2 * (ks % 3);
                        tc::mma_bf16(d0 + (uint32_t)(t * U2_N), abuf + (uint64_t)((t + i) * U2_WP + j),
                                     bdesc0 + (uint64_t)(ks * 2 * U2_N), idesc, ks > 0 ? 1u : 0u);
                    }
                }
            }
            __syncwarp();
            if (tc::elect_one()) {
                tc::commit(&S.a_empty[buf]);
                tc::commit(&S.t_full[ts]);
            }
            __syncwarp();
            // keep U2_NA-1 windows in flight: refill the buffer segment k-1 used (its MMAs
            // are done or about to be: segment k's MMAs are queued behind them)
            if (k + U2_NA - 1 < my) {
                if (k >= 1) tc::mbar_wait(&S.a_empty[(k - 1) % U2_NA], (uint32_t)(((k - 1) / U2_NA) & 1));
                load_a(k + U2_NA - 1);
            }
        }
    } else {
        // -------------------------------------------------------------------- epilogue groups
        const int grp = warp >> 2, wq = warp & 3;
        const uint32_t lane_base = (uint32_t)(32 * wq) << 16;
        const int64_t bplane = a.t4_rows * a.w4;
        // Bias of both C3 rows of a segment, software-pipelined across segments: the loads for
        // this group's NEXT segment are issued as soon as the current values are consumed, so
        // they are in flight during the stores and the wait for the next accumulator.
        float b0v[20], b1v[20];
        auto load_bias = [&](int64_t kk) {
            int64_t img_, R_, c0_;
            seg_coords(blockIdx.x + kk * gridDim.x, img_, R_, c0_);
            const int64_t cc = min(c0_ + 32 * wq + lane, a.w3 - 1);
#pragma unroll
            for (int co = 0; co < 20; ++co) {
                if (a.b3_plane) {
                    b0v[co] = __ldg(a.b3 + ((int64_t)co * a.b3_rows + (2 * R_ - a.b3_row0)) * a.w3 + cc);
                    b1v[co] = __ldg(a.b3 + ((int64_t)co * a.b3_rows + (2 * R_ + 1 - a.b3_row0)) * a.w3 + cc);
                } else {
                    b0v[co] = b1v[co] = __ldg(a.b3 + co);
                }
            }
        };
        if (grp < my) load_bias(grp);
        for (int64_t k = grp; k < my; k += 2) {
            const int ts = (int)(k % U2_NT);
            int64_t img, R, c0;
            seg_coords(blockIdx.x + k * gridDim.x, img, R, c0);
            const int64_t c = c0 + 32 * wq + lane;  // C3 column
            const int64_t C = c >> 1;               // T4 column
            tc::mbar_wait(&S.t_full[ts], (uint32_t)((k / U2_NT) & 1));
            tc::fence_after_sync();
#if U2_EXP >= 1
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&S.t_empty[ts]);
            continue;
#endif
            float v0[32], v1[32];
            tc::tmem_ld32_async(tmem + lane_base + (uint32_t)(ts * 2 * U2_N), v0);
            tc::tmem_ld32_async(tmem + lane_base + (uint32_t)(ts * 2 * U2_N + U2_N), v1);
            tc::tmem_wait_ld();
            tc::fence_before_sync();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&S.t_empty[ts]);
            const bool out_ok = !(lane & 1) && C < a.w4;
            float tv[20];
#pragma unroll
            for (int co = 0; co < 20; ++co) {
                const float t0 = tanh_approx(v0[co] + b0v[co]);
                const float t1 = tanh_approx(v1[co] + b1v[co]);
                // odd lanes hold column c+1 of the even lane's 2x2 window
                const float t01 = __shfl_down_sync(0xffffffffu, t0, 1);
                const float t11 = __shfl_down_sync(0xffffffffu, t1, 1);
                float s4 = pw.p4[co][0] * t0;
                s4 = fmaf(pw.p4[co][1], t01, s4);
                s4 = fmaf(pw.p4[co][2], t1, s4);
                s4 = fmaf(pw.p4[co][3], t11, s4);
                tv[co] = tanh_approx(s4);
            }
            if (k + 2 < my) load_bias(k + 2);
            if (out_ok) {
                // T4 as bf16 channel blocks [3][rows][w4][8] (U3's tensor-core operand rows)
                uint4* t4 = reinterpret_cast<uint4*>(a.t4) + img * 3 * bplane + (R - a.t4_row0) * a.w4 + C;
                t4[0] = make_uint4(tc::pack_bf16(tv[0], tv[1]), tc::pack_bf16(tv[2], tv[3]),
                                   tc::pack_bf16(tv[4], tv[5]), tc::pack_bf16(tv[6], tv[7]));
                t4[bplane] = make_uint4(tc::pack_bf16(tv[8], tv[9]), tc::pack_bf16(tv[10], tv[11]),
                                        tc::pack_bf16(tv[12], tv[13]), tc::pack_bf16(tv[14], tv[15]));
                t4[2 * bplane] = make_uint4(tc::pack_bf16(tv[16], tv[17]), tc::pack_bf16(tv[18], tv[19]), 0u, 0u);
            }
        }
    }
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<256>(tmem);
}

// ============================================================================ U3 (C5 + C6)
// Warp-specialised and persistent (one CTA per SM, 9 warps):
//   warp 8, one thread   producer + MMA issuer: per band, 1-D bulk copies (TMA engine) of the
//                        input window into one of two A buffers; the 40 K-steps of the C5 B
//                        operand stream through a 4-slot ring of bulk copies (the weights are the
//                        same for every band); tcgen05.mma into one of two TMEM accumulators
//                        (2 tiles x NP columns each); tcgen05.commit releases the ring slot, the
//                        A buffer and hands the accumulator to the epilogue
//   warps 0-7            epilogue: TMEM -> registers, bias plane + tanh, the 1x1 C6 layer as a
//                        dot product over n5 (weights in the constant bank), + bias -> output
// so the epilogue of band k overlaps the MMAs of band k+1 and the copies of band k+2.
// Bands are 256 output positions (two M=128 tiles): narrow images (w4 <= kFlatMax) use the
// flattened (row, col) index with the window pitch = w4 (columns >= w5 discarded; a window is
// a run of whole T4 rows = one contiguous copy per channel block); wide images use 256-column
// segments of one output row (window pitch 262, 5 row copies per block).
constexpr int kFlatMax = 180;
constexpr int U3_KS = 40, U3_KS_STAGE = 4, U3_STAGES = U3_KS / U3_KS_STAGE, U3_BRING = 6;
constexpr int U3_NMAX = 128;
constexpr int U3_WP_COL = 2 * kTileM + 6;
constexpr int U3_APX = 1320;  // window pixels per block: flat <= 7*180+8, column 5*262+8
constexpr int kEpiWarps = 8;
constexpr int kThreadsU3 = (kEpiWarps + 1) * 32;

struct U3K6 {
    float k6[U3_NMAX][12];  // [ch][o] (9 used): C6 weights, broadcast from the constant bank
};

struct U3Smem {
    uint4 a[2][3][U3_APX];                         // double-buffered window, 3 channel blocks
    uint4 b[U3_BRING][U3_KS_STAGE * 2 * U3_NMAX];  // B ring (4 K-steps per slot)
    uint64_t a_full[2], a_empty[2], b_full[U3_BRING], b_empty[U3_BRING], t_full[2], t_empty[2];
    uint32_t tmem;
};

struct U3Band {
    int64_t img, q0, wr0, wc0;
    int WP, WR, base;
};

__device__ __forceinline__ U3Band u3_band(const CnnU3Args& a, int64_t band, int64_t per_img, bool flat) {
    U3Band g;
    g.img = band / per_img;
    const int64_t bi = band - g.img * per_img;
    if (flat) {
        g.q0 = bi * 2 * kTileM;
        const int64_t r_first = g.q0 / a.w4;
        g.wr0 = a.out_row0 + r_first;
        g.wc0 = 0;
        g.WP = (int)a.w4;
        g.base = (int)(g.q0 - r_first * a.w4);
        g.WR = (g.base + 2 * kTileM - 1) / g.WP + 1 + 4;
    } else {
        const int64_t bpr = (a.w5 + 2 * kTileM - 1) / (2 * kTileM);
        const int64_t row = bi / bpr;
        g.q0 = (bi - row * bpr) * 2 * kTileM;
        g.wr0 = a.out_row0 + row;
        g.wc0 = g.q0;
        g.WP = U3_WP_COL;
        g.WR = 5;
        g.base = 0;
    }
    return g;
}

__global__ void __launch_bounds__(kThreadsU3, 1)
    cnn_u3_tc_kernel(const CnnU3Args a, const __grid_constant__ U3K6 k6w, const int64_t nbands) {
    extern __shared__ __align__(128) uint8_t smraw[];
    U3Smem& S = *reinterpret_cast<U3Smem*>(smraw + ((128 - (tc::smem_u32(smraw) & 127)) & 127));
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int NP = a.n_pad;
    const bool flat = a.w4 <= kFlatMax;
    const int64_t per_img = flat ? (a.out_rows * a.w4 + 2 * kTileM - 1) / (2 * kTileM)
                                 : a.out_rows * ((a.w5 + 2 * kTileM - 1) / (2 * kTileM));
    const int64_t bplane = a.t4_rows * a.w4;

    if (warp == 0) tc::tmem_alloc<512>(&S.tmem);
    if (tid == 0) {
        for (int i = 0; i < 2; ++i) {
            tc::mbar_init(&S.a_full[i], 1);
            tc::mbar_init(&S.a_empty[i], 1);
            tc::mbar_init(&S.t_full[i], 1);
            tc::mbar_init(&S.t_empty[i], kEpiWarps);
        }
        for (int i = 0; i < U3_BRING; ++i) {
            tc::mbar_init(&S.b_full[i], 1);
            tc::mbar_init(&S.b_empty[i], 1);
        }
        tc::mbar_fence_init();
    }
    // windows start zeroed: pixels a copy does not cover (beyond the image, the spare pixels of
    // tap pair (4,5)) then only ever hold finite T4 values
    for (int idx = tid; idx < 2 * 3 * U3_APX; idx += kThreadsU3) (&S.a[0][0][0])[idx] = make_uint4(0u, 0u, 0u, 0u);
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    const uint32_t tmem = S.tmem;

    if (warp == kEpiWarps) {
        if (lane == 0) {
            // ------------------------------------------------------------ producer + MMA
            const uint4* t4b_all = reinterpret_cast<const uint4*>(a.t4);
            const uint4* kb = reinterpret_cast<const uint4*>(a.k5_tc);
            const uint32_t stage_bytes = (uint32_t)(U3_KS_STAGE * 2 * NP * 16);
            const int64_t my_bands = nbands > blockIdx.x ? (nbands - 1 - blockIdx.x) / gridDim.x + 1 : 0;
            const int64_t total_stages = my_bands * U3_STAGES;
            auto load_b = [&](int64_t gs) {
                const int slot = (int)(gs % U3_BRING);
                tc::mbar_expect_tx(&S.b_full[slot], stage_bytes);
                tc::bulk_g2s(S.b[slot], kb + (size_t)(gs % U3_STAGES) * (stage_bytes / 16), stage_bytes, &S.b_full[slot]);
            };
            auto load_a = [&](int64_t band, int buf) {
                const U3Band g = u3_band(a, band, per_img, flat);
                const uint4* t4b = t4b_all + g.img * 3 * bplane;
                const int64_t r0 = g.wr0 - a.t4_row0;
                uint32_t bytes = 0;
                if (flat) {
                    const int64_t rows = min((int64_t)g.WR, a.t4_rows - r0);
                    bytes = (uint32_t)(3 * rows * a.w4 * 16);
                    tc::mbar_expect_tx(&S.a_full[buf], bytes);
                    for (int blk = 0; blk < 3; ++blk)
                        tc::bulk_g2s(S.a[buf][blk], t4b + blk * bplane + r0 * a.w4, (uint32_t)(rows * a.w4 * 16),
                                     &S.a_full[buf]);
                } else {
                    const int64_t cols = min((int64_t)U3_WP_COL, a.w4 - g.wc0);
                    bytes = (uint32_t)(3 * 5 * cols * 16);
                    tc::mbar_expect_tx(&S.a_full[buf], bytes);
                    for (int blk = 0; blk < 3; ++blk)
                        for (int r = 0; r < 5; ++r)
                            tc::bulk_g2s(&S.a[buf][blk][r * U3_WP_COL], t4b + blk * bplane + (r0 + r) * a.w4 + g.wc0,
                                         (uint32_t)(cols * 16), &S.a_full[buf]);
                }
            };
            const uint32_t idesc = tc::make_idesc_bf16(kTileM, NP);
            for (int64_t gs = 0; gs < (int64_t)(U3_BRING - 1) && gs < total_stages; ++gs) load_b(gs);
            if (my_bands > 0) load_a(blockIdx.x, 0);
            int64_t gs = 0;
            for (int64_t k = 0; k < my_bands; ++k) {
                const int buf = (int)(k & 1);
                const U3Band g = u3_band(a, blockIdx.x + k * gridDim.x, per_img, flat);
                tc::mbar_wait(&S.a_full[buf], (uint32_t)((k >> 1) & 1));
                if (k >= 2) tc::mbar_wait(&S.t_empty[buf], (uint32_t)(((k - 2) >> 1) & 1));
                tc::fence_after_sync();
                const uint32_t a_base = tc::smem_u32(S.a[buf][0]);
                const uint32_t plane_bytes = (uint32_t)(U3_APX * 16);
                const uint32_t d_base = tmem + (uint32_t)(buf * 256);
                for (int st = 0; st < U3_STAGES; ++st, ++gs) {
                    const int slot = (int)(gs % U3_BRING);
                    tc::mbar_wait(&S.b_full[slot], (uint32_t)((gs / U3_BRING) & 1));
                    tc::fence_after_sync();
                    const uint32_t b_base = tc::smem_u32(S.b[slot]);
                    for (int u = 0; u < U3_KS_STAGE; ++u) {
                        const int ks = st * U3_KS_STAGE + u;
                        const int i = ks / 8, r8 = ks % 8;
                        uint32_t a_addr, lbo;
                        if (r8 < 5) {  // channels 0-15 of tap (i, r8): blocks 0 and 1
                            a_addr = a_base + (uint32_t)((g.base + i * g.WP + r8) * 16);
                            lbo = plane_bytes;
                        } else {       // channels 16-19 of taps (i, j), (i, j+1): block 2, next pixel
                            a_addr = a_base + 2 * plane_bytes + (uint32_t)((g.base + i * g.WP + 2 * (r8 - 5)) * 16);
                            lbo = 16;
                        }
                        const uint64_t bd = tc::make_desc(b_base + (uint32_t)(u * 2 * NP * 16), (uint32_t)(NP * 16), 128);
#if U3_EXP == 2
                        if (0)
#endif
                        for (int t = 0; t < 2; ++t) {
                            const uint64_t ad = tc::make_desc(a_addr + (uint32_t)(t * kTileM * 16), lbo, 128);
                            tc::mma_bf16(d_base + (uint32_t)(t * NP), ad, bd, idesc, ks > 0 ? 1u : 0u);
                        }
                    }
                    tc::commit(&S.b_empty[slot]);
                    // refill the slot of stage gs-1 with stage gs+BRING-1 (it has BRING-1 stages to land)
                    if (gs + U3_BRING - 1 < total_stages) {
                        if (gs >= 1) tc::mbar_wait(&S.b_empty[(gs - 1) % U3_BRING], (uint32_t)(((gs - 1) / U3_BRING) & 1));
                        load_b(gs + U3_BRING - 1);
                    }
                }
                tc::commit(&S.a_empty[buf]);
                tc::commit(&S.t_full[buf]);
                // prefetch the next band's window into the other buffer (freed by band k-1's MMAs)
                if (k + 1 < my_bands) {
                    if (k >= 1) tc::mbar_wait(&S.a_empty[buf ^ 1], (uint32_t)(((k - 1) >> 1) & 1));
                    load_a(blockIdx.x + (k + 1) * gridDim.x, buf ^ 1);
                }
            }
        }
    } else {
        // ---------------------------------------------------------------- epilogue warps
        const int t = warp >> 2;  // tile
        const uint32_t lane_base = (uint32_t)(32 * (warp & 3)) << 16;
        int64_t k = 0;
        for (int64_t band = blockIdx.x; band < nbands; band += gridDim.x, ++k) {
            const int buf = (int)(k & 1);
            const U3Band g = u3_band(a, band, per_img, flat);
            tc::mbar_wait(&S.t_full[buf], (uint32_t)((k >> 1) & 1));
            tc::fence_after_sync();
#if U3_EXP >= 1
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&S.t_empty[buf]);
            continue;
#endif
            const int m = t * kTileM + 32 * (warp & 3) + lane;
            int64_t orow, ocol;
            if (flat) {
                const int64_t q = g.q0 + m;
                orow = a.out_row0 + q / a.w4;
                ocol = q - (q / a.w4) * a.w4;
            } else {
                orow = g.wr0;
                ocol = g.q0 + m;
            }
            const bool ok = orow < a.out_row0 + a.out_rows && ocol < a.w5;
            float c6[9];
#pragma unroll
            for (int o = 0; o < 9; ++o) c6[o] = 0.f;
            // software-pipelined drain: TMEM columns and bias values of chunk c+1 are in flight
            // while chunk c is computed (up to 4 chunks of 32 columns; NP <= 128)
            const int nch = (NP + 31) / 32;
            float v[2][32], bv[2][32];
            auto issue = [&](int c, int s) {
                tc::tmem_ld32_async(tmem + lane_base + (uint32_t)(buf * 256 + t * NP + 32 * c), v[s]);
                if (ok) {
#pragma unroll
                    for (int u = 0; u < 32; ++u) {
                        const int ch = min(32 * c + u, a.n5 - 1);
                        bv[s][u] = a.b5_plane
                                       ? __ldg(a.b5 + ((int64_t)ch * a.b5_rows + (orow - a.b5_row0)) * a.w5 + ocol)
                                       : __ldg(a.b5 + ch);
                    }
                }
            };
            issue(0, 0);
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                if (c < nch) {
                    tc::tmem_wait_ld();
                    if (c + 1 < nch) issue(c + 1, (c + 1) & 1);
                    if (ok) {
                        // branch-free over the chunk (C6 weights of the padding channels
                        // n5..NP-1 are zero and their accumulators finite), so the tanh of
                        // several channels are in flight at once
#pragma unroll
                        for (int u = 0; u < 32; ++u) {
                            const int ch = 32 * c + u;
                            const float th = tanh_approx(v[c & 1][u] + bv[c & 1][u]);
#pragma unroll
                            for (int o = 0; o < 9; ++o) c6[o] = fmaf(k6w.k6[ch][o], th, c6[o]);
                        }
                    }
                }
            }
            tc::fence_before_sync();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&S.t_empty[buf]);  // the accumulator can be reused
            if (ok) {
                float* ob = a.out + g.img * a.out_img_stride + (orow - a.out_row0) * a.w5 + ocol;
#pragma unroll
                for (int o = 0; o < 9; ++o) {
                    const float b = a.b6_plane
                                        ? __ldg(a.b6 + ((int64_t)o * a.b6_rows + (orow - a.b6_row0)) * a.w5 + ocol)
                                        : __ldg(a.b6 + o);
                    ob[o * a.out_plane_stride] = c6[o] + b;
                }
            }
        }
    }
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<512>(tmem);
}

uint16_t to_bf16(float f) {  // round to nearest even (host)
    uint32_t u;
    std::memcpy(&u, &f, 4);
    if ((u & 0x7fffffffu) > 0x7f800000u) return 0x7fc0;
    u += 0x7fffu + ((u >> 16) & 1u);
    return (uint16_t)(u >> 16);
}

bool set_smem_attr(const void* fn, size_t bytes, std::atomic<uint32_t>& flags) {
    int dev = 0;
    cudaGetDevice(&dev);
    const uint32_t bit = 1u << (dev & 31);
    if (flags.load() & bit) return true;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) != cudaSuccess) return false;
    flags.fetch_or(bit);
    return true;
}

}  // namespace

// B operand of C3 for the 15 K-steps: [ks][half][n<32][8 ci]; half h of K-step (i, j-pair)
// holds tap (i, j + h) (zero for j + h == 5), output maps >= 20 are zero.
size_t cnn_k3_tc_bytes() { return (size_t)U2_KS * 2 * U2_N * 8 * 2; }
void cnn_prepare_k3_tc(const float* k3, uint16_t* dst) {
    for (int ks = 0; ks < U2_KS; ++ks) {
        const int i = ks / 3, j0 = 2 * (ks % 3);
        for (int h = 0; h < 2; ++h)
            for (int n = 0; n < U2_N; ++n)
                for (int e = 0; e < 8; ++e) {
                    const int j = j0 + h;
                    const float v = (n < 20 && j < 5) ? k3[(n * 8 + e) * 25 + i * 5 + j] : 0.f;
                    dst[((ks * 2 + h) * U2_N + n) * 8 + e] = to_bf16(v);
                }
    }
}

// B operand of C5 for the 40 K-steps: per filter row i, steps 0-4 = tap (i, j) channels 0-15
// (half h = channels 8h..8h+7), steps 5-7 = channels 16-19 of taps (i, j) and (i, j+1).
int cnn_n5_pad(int n5) { return (n5 + 15) / 16 * 16; }
size_t cnn_k5_tc_bytes(int n5) { return (size_t)U3_KS * 2 * cnn_n5_pad(n5) * 8 * 2; }
void cnn_prepare_k5_tc(const float* k5, int n5, uint16_t* dst) {
    const int NP = cnn_n5_pad(n5);
    for (int ks = 0; ks < U3_KS; ++ks) {
        const int i = ks / 8, r8 = ks % 8;
        for (int h = 0; h < 2; ++h)
            for (int n = 0; n < NP; ++n)
                for (int e = 0; e < 8; ++e) {
                    int ci, j;
                    if (r8 < 5) {
                        ci = 8 * h + e;
                        j = r8;
                    } else {
                        ci = 16 + e;
                        j = 2 * (r8 - 5) + h;
                    }
                    const float v = (n < n5 && ci < 20 && j < 5) ? k5[((size_t)n * 20 + ci) * 25 + i * 5 + j] : 0.f;
                    dst[((size_t)(ks * 2 + h) * NP + n) * 8 + e] = to_bf16(v);
                }
    }
}

cudaError_t launch_cnn_u2_tc(const CnnU2Args& a, cudaStream_t s) {
    if (a.t4_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    static std::atomic<uint32_t> flags{0};
    const size_t smem = sizeof(U2Smem) + 128;
    if (!set_smem_attr((const void*)cnn_u2_tc_kernel, smem, flags)) return cudaErrorInvalidValue;
    U2P pw;
    std::memcpy(pw.p4, a.p4_host, sizeof pw.p4);
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t nseg = a.t4_rows * ((a.w3 + kTileM - 1) / kTileM) * a.nimg;
    const unsigned grid = (unsigned)std::min<int64_t>(nseg, sms);
    cnn_u2_tc_kernel<<<grid, kThreadsU2, smem, s>>>(a, pw, nseg);
    return cudaGetLastError();
}

cudaError_t launch_cnn_u3_tc(const CnnU3Args& a, cudaStream_t s) {
    if (a.out_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    if (a.n_pad > U3_NMAX || a.n_pad % 16 || a.n5 > U3_NMAX) return cudaErrorInvalidValue;
    static std::atomic<uint32_t> flags{0};
    const size_t smem = sizeof(U3Smem) + 128;
    if (!set_smem_attr((const void*)cnn_u3_tc_kernel, smem, flags)) return cudaErrorInvalidValue;
    const bool flat = a.w4 <= kFlatMax;
    const int64_t per_img = flat ? (a.out_rows * a.w4 + 2 * kTileM - 1) / (2 * kTileM)
                                 : a.out_rows * ((a.w5 + 2 * kTileM - 1) / (2 * kTileM));
    U3K6 k6w{};
    for (int ch = 0; ch < a.n5; ++ch)
        for (int o = 0; o < 9; ++o) k6w.k6[ch][o] = a.k6_host[o * a.n5 + ch];
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t nbands = per_img * a.nimg;
    const unsigned grid = (unsigned)std::min<int64_t>(nbands, sms);
    cnn_u3_tc_kernel<<<grid, kThreadsU3, smem, s>>>(a, k6w, nbands);
    return cudaGetLastError();
}

}  // namespace tg
