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
//   U3: bias plane + tanh -> T5 packed to bf16 and written back into TMEM (tcgen05.st); the
//       1x1 C6 layer is a second tcgen05.mma whose A operand is read from TMEM (N = 16: 9
//       maps padded), + the C6 bias plane -> output (fp32).
// Precision: bf16 operands, fp32 accumulation; parity bound 2e-2 normwise (R16).
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstring>
#include <vector>

#include "kernels.h"
#include "tc_sm100.cuh"

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
// Segment = T4 row R (C3 rows 2R, 2R+1) x 128 C3 columns [c0, c0+128): ONE M = 128 tile whose N
// holds BOTH C3 rows: columns [0, 20) = row 2R, [24, 44) = row 2R+1 (N = 48). Window: T2 rows
// [2R, 2R+6) x cols [c0, c0+134), 8 channels per pixel (one 16-byte row each).
// Window row y feeds C3 row 2R with filter row y and row 2R+1 with filter row y - 1, so ONE
// MMA per (window row, tap pair) serves both output rows: its B operand (one of 6 row variants)
// holds filter row y in columns [0, 20) and filter row y - 1 in [24, 44) (zero where the filter
// row does not exist). 6 rows x 3 tap pairs = 18 MMAs of N = 48 per segment instead of
// 2 tiles x 15 of N = 32: the A operand -- the shared-memory read that bounds these small-N
// MMAs -- is read 18 times instead of 30.
// Warp-specialised and persistent (one CTA per SM, 4 U2_G + 2 warps; single-lane issue under
// elect.sync):
//   warp 4 U2_G + 1      copy producer: the C3 B operand (6 x 3 K-steps) once per CTA by a bulk
//                        copy; per segment six 1-D bulk copies (TMA engine) of the window's T2
//                        rows into one of U2_NA buffers, as soon as the buffer is free
//   warp 4 U2_G          MMA issuer: 18 tcgen05.mma into one of U2_NT TMEM slots; tcgen05.commit
//                        frees the window buffer and hands the slot to the epilogue (copy issue
//                        -- ~150 cycles per bulk copy -- does not serialise with MMA issue)
//   warps 0 .. 4 U2_G-1  U2_G epilogue groups of 4 warps taking segments in turn: bias plane
//                        (prefetched one segment of the group ahead), tanh, the 2x2 subsample
//                        (rows in the same thread, columns across neighbouring lanes), tanh -> T4
//                        bf16 channel blocks. Three groups rather than two: U2 0.193 -> 0.159 ms
//                        on the single 6400x4800 image (bias planes from HBM), +1 % on cnn3
constexpr int U2_WR = 6, U2_WP = kTileM + 6;  // +4 taps, +1 for the (4,5) tap pair, +1 spare
constexpr int U2_N = 48;                      // [0,20) row 2R, [24,44) row 2R+1, rest zero
constexpr int U2_ROW1 = 24;                   // first column of C3 row 2R+1
constexpr int U2_KS = 18;                     // 6 window rows x tap pairs (0,1) (2,3) (4,5)
constexpr int U2_NA = 8;                      // window buffers
constexpr int U2_G = 3;                       // epilogue groups (4 warps each), taking segments in turn
constexpr int U2_NT = 4;                      // TMEM slots, 64 columns apart
constexpr int U2_TCOLS = U2_NT * 64;          // TMEM columns allocated (a power of two)
constexpr int kThreadsU2 = (4 * U2_G + 2) * 32;

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
    // segment -> (image, T4 row, first C3 column) in 32-bit arithmetic (the launcher checks that
    // segment counts fit; 64-bit division is a ~100-instruction software sequence)
    const uint32_t per_img_u = (uint32_t)per_img, spr_u = (uint32_t)segs_per_row;
    auto seg_coords = [&](int64_t sg, int64_t& img, int64_t& R, int64_t& c0) {
        const uint32_t s = (uint32_t)sg, im = s / per_img_u, rem = s - im * per_img_u, rr = rem / spr_u;
        img = im;
        R = a.t4_row0 + rr;
        c0 = (int64_t)(rem - rr * spr_u) * kTileM;
    };

    if (warp == 0) tc::tmem_alloc<U2_TCOLS>(&S.tmem);
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

    if (warp == 4 * U2_G + 1) {
        // -------------------------------------------------------------------- copy producer
        // (the whole warp runs the loop; the window rows are issued by one lane each)
        const uint4* t2all = reinterpret_cast<const uint4*>(a.t2);
        const uint32_t bbytes = (uint32_t)(U2_KS * 2 * U2_N * 16);
        if (tc::elect_one()) {
            tc::mbar_expect_tx(&S.b_full, bbytes);
            tc::bulk_g2s(S.b, a.k3_tc, bbytes, &S.b_full);
        }
        __syncwarp();
        for (int64_t k = 0; k < my; ++k) {
            const int buf = (int)(k % U2_NA);
            if (k >= U2_NA) tc::mbar_wait(&S.a_empty[buf], (uint32_t)(((k - U2_NA) / U2_NA) & 1));
            int64_t img, R, c0;
            seg_coords(blockIdx.x + k * gridDim.x, img, R, c0);
            const int64_t r0 = 2 * R - a.t2_row0;
            const int64_t rows = min((int64_t)U2_WR, a.t2_rows - r0);
            const int64_t cols = min((int64_t)U2_WP, a.w2 - c0);
            // one window row per lane, all issued in ONE warp instruction (a single thread
            // serialises ~150 cycles per bulk copy)
            if (lane == 0) tc::mbar_expect_tx(&S.a_full[buf], (uint32_t)(rows * cols * 16));
            __syncwarp();
            if (lane < rows) {
                const uint4* src = t2all + (img * a.t2_rows + r0 + lane) * a.w2 + c0;
                tc::bulk_g2s(&S.a[buf][lane * U2_WP], src, (uint32_t)(cols * 16), &S.a_full[buf]);
            }
            __syncwarp();
        }
    } else if (warp == 4 * U2_G) {
        // -------------------------------------------------------------------- MMA issuer
        // ONE elected lane runs the whole loop (barrier waits, MMAs, commits): warp-level
        // hand-offs per segment left the tensor pipe idle (tools/micro/umma_probe.cu)
        if (tc::elect_one()) {
            tc::mbar_wait(&S.b_full, 0);
            const uint32_t idesc = tc::make_idesc_bf16(kTileM, U2_N);
            // descriptors: the start address is the low 14 bits (16-byte units), advanced by adding
            const uint64_t bdesc0 = tc::make_desc(tc::smem_u32(S.b), U2_N * 16, 128);
            const uint64_t adesc0 = tc::make_desc(tc::smem_u32(S.a[0]), 16, 128);  // 2nd K-half = next pixel
            // the barriers of the NEXT segment are probed (mbarrier.test_wait) before the last MMAs
            // of the current one: a barrier access waits ~150 cycles for the shared-memory port the
            // MMA operand reads saturate, and overlaps the queued MMAs this way instead of stalling
            // the issue between segments (blocking waits only after a failed probe;
            // tools/micro/umma_probe.cu)
            bool a_ready = false, t_ready = false;
            for (int64_t k = 0; k < my; ++k) {
                const int buf = (int)(k % U2_NA), ts = (int)(k % U2_NT);
                if (!a_ready) tc::mbar_wait(&S.a_full[buf], (uint32_t)((k / U2_NA) & 1));
                if (k >= U2_NT && !t_ready) tc::mbar_wait(&S.t_empty[ts], (uint32_t)(((k - U2_NT) / U2_NT) & 1));
                tc::fence_after_sync();
                const uint64_t abuf = adesc0 + (uint64_t)(buf * (U2_WR * U2_WP));
                const uint32_t d0 = tmem + (uint32_t)(ts * 64);
                const int64_t kn = k + 1;
#pragma unroll
                for (int ks = 0; ks < U2_KS; ++ks) {  // window row y = ks / 3, tap pair (j, j+1)
                    if (ks == U2_KS - 4) {
                        a_ready = kn < my && tc::mbar_test(&S.a_full[kn % U2_NA], (uint32_t)((kn / U2_NA) & 1));
                        t_ready = kn >= U2_NT && kn < my &&
                                  tc::mbar_test(&S.t_empty[kn % U2_NT], (uint32_t)(((kn - U2_NT) / U2_NT) & 1));
                    }
                    const int y = ks / 3, j = 2 * (ks % 3);
                    tc::mma_bf16(d0, abuf + (uint64_t)(y * U2_WP + j), bdesc0 + (uint64_t)(ks * 2 * U2_N), idesc,
                                 ks > 0 ? 1u : 0u);
                }
                tc::commit(&S.a_empty[buf]);
                tc::commit(&S.t_full[ts]);
            }
        }
        __syncwarp();
    } else {
        // -------------------------------------------------------------------- epilogue groups
        const int grp = warp >> 2, wq = warp & 3;
        const uint32_t lane_base = (uint32_t)(32 * wq) << 16;
        const int64_t bplane = a.t4_rows * a.w4;
        // Bias of both C3 rows of a segment, software-pipelined across segments: the loads for
        // this group's NEXT segment are issued as soon as the current values are consumed, so
        // they are in flight during the stores and the wait for the next accumulator.
        float b0v[20], b1v[20];
        const uint32_t bcs = a.b3_plane ? (uint32_t)(a.b3_rows * a.w3) : 1u;  // channel stride of the bias
        const uint32_t brs = a.b3_plane ? (uint32_t)a.w3 : 0u;                 // row stride
        auto load_bias = [&](int64_t kk) {
            int64_t img_, R_, c0_;
            seg_coords(blockIdx.x + kk * gridDim.x, img_, R_, c0_);
            const int64_t cc = min(c0_ + 32 * wq + lane, a.w3 - 1);
            const float* p0 = a.b3_plane ? a.b3 + (2 * R_ - a.b3_row0) * a.w3 + cc : a.b3;
#pragma unroll
            for (int co = 0; co < 20; ++co) {
                b0v[co] = __ldg(p0 + co * bcs);
                b1v[co] = __ldg(p0 + co * bcs + brs);
            }
        };
        if (grp < my) load_bias(grp);
        for (int64_t k = grp; k < my; k += U2_G) {
            const int ts = (int)(k % U2_NT);
            int64_t img, R, c0;
            seg_coords(blockIdx.x + k * gridDim.x, img, R, c0);
            const int64_t c = c0 + 32 * wq + lane;  // C3 column
            const int64_t C = c >> 1;               // T4 column
            tc::mbar_wait(&S.t_full[ts], (uint32_t)((k / U2_NT) & 1));
            tc::fence_after_sync();
            float va[32], vb[16], v1[20];
            tc::tmem_ld32_async(tmem + lane_base + (uint32_t)(ts * 64), va);       // columns [0, 32)
            tc::tmem_ld16_async(tmem + lane_base + (uint32_t)(ts * 64 + 32), vb);  // columns [32, 48)
            tc::tmem_wait_ld();
            const float* v0 = va;  // C3 row 2R: columns [0, 20)
#pragma unroll
            for (int co = 0; co < 20; ++co) v1[co] = co < 8 ? va[U2_ROW1 + co] : vb[U2_ROW1 + co - 32];
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
            if (k + U2_G < my) load_bias(k + U2_G);
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
    if (warp == 0) tc::tmem_dealloc<U2_TCOLS>(tmem);
}

// ============================================================================ U3 (C5 + C6)
// Band = U3_BT x 128 consecutive output positions in the FLATTENED (row, col) index of the chunk
// with pitch w4 (U3_BT M=128 tiles; the w4 - w5 = 4 positions past each row's end are computed
// and dropped). For any width, filter row i of a band reads one contiguous run of T4: flat pixels
// [q0 + i*w4, q0 + i*w4 + 128 U3_BT + 6) -- the band's "slice" i (+4 taps, +1 for the (4,5) tap
// pair, +1 spare).
// Both layers run on the tensor cores:
//   C5  D5[px][n] = sum_k A5[px][k] B5[k][n]  (A5: the slices in smem, B5: resident in smem)
//   C6  D6[px][o] = sum_n T5[px][n] B6[n][o]  with T5 = tanh(D5 + bias plane) written back by
//       the epilogue into the drained TMEM columns as bf16 pairs, and the MMA reading its A
//       operand straight from TMEM (M = 128 lanes, K = NP channels, N = 16: 9 maps padded)
// TMEM (512 columns): U3_NB accumulator buffers; buffer b, tile t: the 128-column region at
// 128 (U3_BT b + t), holding D5 in [0, NP), then T5 in [0, NP/2) and D6 in [64, 80).
// Warp-specialised and persistent (one CTA per SM, 18 warps; single-lane issue under elect.sync):
//   warp 17              copy producer: the whole C5 B operand (40 K-steps x NP maps, up to
//                        160 KB) ONCE per CTA (it stays resident), then the slices through a ring
//                        of U3_NA buffers (three 1-D bulk copies each, one per channel block)
//   warp 16              MMA issuer: per slice 8 K-steps x U3_BT tiles of tcgen05.mma; after the
//                        5th slice the accumulator goes to the epilogue. The C6 MMAs of earlier
//                        bands are slotted in between slices as soon as their T5 is in TMEM.
//   warps 0-15           U3_NB epilogue groups; group g owns buffer g and takes bands k = g mod
//                        U3_NB: TMEM -> registers, + bias plane, tanh -> bf16 T5 -> TMEM; then
//                        D6 -> registers, + C6 bias -> output (fp32)
// so the MMAs run up to U3_NB - 1 bands ahead of the epilogue. With one tile per band (U3_BT = 1,
// four buffers) a band's epilogue latency -- drain, C6 round trip, D6 -- may take three MMA band
// times; with two tiles per band (two buffers) it had one, and the MMAs waited for it (DESIGN.md
// §5.3). (Earlier versions re-streamed B5 for every band, and computed C6 as 9 x n5 FFMA per
// position on the CUDA cores.)
constexpr int U3_KS = 40;
constexpr int U3_NMAX = 128;
constexpr int U3_BT = 2;                // M = 128 tiles per band
constexpr int U3_NB = 4 / U3_BT;        // TMEM accumulator buffers (512 columns, 128 per tile)
constexpr int U3_SPX = U3_BT * kTileM + 8;  // pixels per slice buffer (U3_BT * 128 + 6 used)
constexpr int U3_NA = 8 / U3_BT;        // slice buffers
constexpr int U3_C6K = U3_NMAX / 16;    // C6 K-steps (max)
constexpr int U3_C6N = 16;              // C6 N: 9 maps padded
constexpr int U3_C6COL = 64;            // D6 column within a tile region
constexpr int kEpiGroups = U3_NB;             // epilogue groups: group g takes bands k = g mod U3_NB
constexpr int kEpiWarps = 4 * U3_BT * kEpiGroups;
constexpr int kThreadsU3 = (kEpiWarps + 2) * 32;

struct U3P {
    uint4 b6[U3_C6K * 2 * U3_C6N];  // C6 B operand, bf16 [ks][half][o][8 ch] (4 KB)
};

struct U3Smem {
    uint4 b[U3_KS * 2 * U3_NMAX];     // resident C5 B operand: [ks][half][n] -> 8 bf16
    uint4 b6[U3_C6K * 2 * U3_C6N];    // C6 B operand
    uint4 a[U3_NA][3][U3_SPX];        // slice ring: [channel block][pixel] -> 8 bf16
    uint64_t b_full, a_full[U3_NA], a_empty[U3_NA], t_full[U3_NB], t_empty[U3_NB], t5_full[U3_NB], c6_full[U3_NB];
    uint32_t tmem;
};

// NCH: TMEM chunks of 32 columns (NP = n5 padded to 16, NCH = ceil(NP / 32)); BQ: the C5 bias
// layout (CnnU3Args::b5_q4: 0 planes, 1 channel quads), a compile-time choice so the drain carries
// no branch
template <int NCH, int BQ>
__global__ void __launch_bounds__(kThreadsU3, 1)
    cnn_u3_tc_kernel(const CnnU3Args a, const __grid_constant__ U3P pw, const int64_t nbands) {
    extern __shared__ __align__(128) uint8_t smraw[];
    U3Smem& S = *reinterpret_cast<U3Smem*>(smraw + ((128 - (tc::smem_u32(smraw) & 127)) & 127));
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int NP = a.n_pad;
    const int64_t per_img = (a.out_rows * a.w4 + U3_BT * kTileM - 1) / (U3_BT * kTileM);
    const int64_t bplane = a.t4_rows * a.w4;                 // pixels per channel block of one image
    const int64_t flat0 = (a.out_row0 - a.t4_row0) * a.w4;  // flat index of output row 0 in the T4 buffer

    if (warp == 0) tc::tmem_alloc<512>(&S.tmem);
    if (tid == 0) {
        tc::mbar_init(&S.b_full, 1);
        for (int i = 0; i < U3_NA; ++i) {
            tc::mbar_init(&S.a_full[i], 1);
            tc::mbar_init(&S.a_empty[i], 1);
        }
        for (int i = 0; i < U3_NB; ++i) {
            tc::mbar_init(&S.t_full[i], 1);
            tc::mbar_init(&S.t_empty[i], 4 * U3_BT);   // the warps of the group that owns buffer i
            tc::mbar_init(&S.t5_full[i], 4 * U3_BT);
            tc::mbar_init(&S.c6_full[i], 1);
        }
        tc::mbar_fence_init();
    }
    // slice buffers start zeroed: pixels a copy does not cover (past the chunk's last T4 row)
    // then only ever hold finite T4 values; they feed positions that are not stored
    for (int idx = tid; idx < U3_NA * 3 * U3_SPX; idx += kThreadsU3) (&S.a[0][0][0])[idx] = make_uint4(0u, 0u, 0u, 0u);
    for (int idx = tid; idx < U3_C6K * 2 * U3_C6N; idx += kThreadsU3) S.b6[idx] = pw.b6[idx];
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    const uint32_t tmem = S.tmem;

    const int64_t my_bands = nbands > blockIdx.x ? (nbands - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    const int64_t total = my_bands * 5;  // slices
    if (warp == kEpiWarps + 1) {
        // ---------------------------------------------------------------- copy producer
        // (warp-uniform loop, one elected lane issues): B5 once, then every slice as soon as
        // its ring buffer is free
        const uint4* t4all = reinterpret_cast<const uint4*>(a.t4);
        if (my_bands > 0) {
            const uint32_t bbytes = (uint32_t)(U3_KS * 2 * NP * 16);
            if (tc::elect_one()) {
                tc::mbar_expect_tx(&S.b_full, bbytes);
                const uint8_t* kb = reinterpret_cast<const uint8_t*>(a.k5_tc);
                for (uint32_t off = 0; off < bbytes; off += 16384u)
                    tc::bulk_g2s(reinterpret_cast<uint8_t*>(S.b) + off, kb + off, min(16384u, bbytes - off), &S.b_full);
            }
            __syncwarp();
        }
        for (int64_t s = 0; s < total; ++s) {
            const int slot = (int)(s % U3_NA);
            if (s >= U3_NA) tc::mbar_wait(&S.a_empty[slot], (uint32_t)(((s - U3_NA) / U3_NA) & 1));
            const int64_t band = blockIdx.x + (s / 5) * gridDim.x;
            const int i = (int)(s % 5);
            const int64_t img = (uint32_t)band / (uint32_t)per_img;
            const int64_t q0 = (band - img * per_img) * U3_BT * kTileM;
            const int64_t e = flat0 + q0 + (int64_t)i * a.w4;
            const int64_t n = max((int64_t)0, min((int64_t)U3_SPX, bplane - e));
            if (lane == 0) tc::mbar_expect_tx(&S.a_full[slot], (uint32_t)(3 * n * 16));
            __syncwarp();
            if (n > 0 && lane < 3)  // one channel block per lane, in one warp instruction
                tc::bulk_g2s(S.a[slot][lane], t4all + (img * 3 + lane) * bplane + e, (uint32_t)(n * 16), &S.a_full[slot]);
            __syncwarp();
        }
    } else if (warp == kEpiWarps) {
        // ---------------------------------------------------------------- MMA issuer
        // (warp-uniform loop so descriptors live in uniform registers; one elected lane issues)
        if (my_bands > 0) tc::mbar_wait(&S.b_full, 0);
        const uint32_t idesc = tc::make_idesc_bf16(kTileM, NP);
        const uint32_t idesc6 = tc::make_idesc_bf16(kTileM, U3_C6N);
        const uint64_t bdesc0 = tc::make_desc(tc::smem_u32(S.b), (uint32_t)(NP * 16), 128);
        const uint64_t b6desc0 = tc::make_desc(tc::smem_u32(S.b6), (uint32_t)(U3_C6N * 16), 128);
        const uint32_t plane_bytes = (uint32_t)(U3_SPX * 16);
        // ONE elected lane runs the whole issue loop: tcgen05.mma issue blocks once a few MMAs are
        // queued, so warp-level hand-offs between slices (elect / __syncwarp, ~170 cycles per slice
        // measured by tools/micro/umma_probe.cu) left the tensor pipe idle; a single lane's barrier
        // waits cost less and the queue stays fed.
        if (tc::elect_one()) {
            // C6 of local band kb (its T5 is in TMEM): 2 tiles x NP/16 K-steps, A from TMEM
            int64_t c6_next = 0;
            auto issue_c6 = [&](int64_t kb) {
                const uint32_t base = tmem + (uint32_t)((kb % U3_NB) * U3_BT * 128);
                for (int t = 0; t < U3_BT; ++t)
                    for (int kk = 0; kk < NP / 16; ++kk)
                        tc::mma_bf16_ts(base + (uint32_t)(t * 128 + U3_C6COL), base + (uint32_t)(t * 128 + kk * 8),
                                        b6desc0 + (uint64_t)(kk * 2 * U3_C6N), idesc6, kk > 0 ? 1u : 0u);
                tc::commit(&S.c6_full[kb % U3_NB]);
            };
            // The barrier probes for the NEXT slice (and for a pending C6) are issued before the
            // last MMAs of the current slice (mbarrier.test_wait, non-blocking): a barrier access
            // waits ~150 cycles for the shared-memory port the MMAs' operand reads saturate, and
            // so overlaps the queued MMAs instead of stalling the issue between slices (a blocking
            // wait only follows when a probe failed; tools/micro/umma_probe.cu).
            bool a_ready = false, t5_ready = false;
            const int64_t total_s = my_bands * 5;
            for (int64_t k = 0; k < my_bands; ++k) {
                const int buf = (int)(k % U3_NB);
                if (k >= U3_NB) {
                    // band k-NB shares this accumulator: its C6 must be issued before its epilogue
                    // can release the buffer
                    while (c6_next <= k - U3_NB) {
                        tc::mbar_wait(&S.t5_full[c6_next % U3_NB], (uint32_t)((c6_next / U3_NB) & 1));
                        tc::fence_after_sync();
                        issue_c6(c6_next++);
                        t5_ready = false;
                    }
                    tc::mbar_wait(&S.t_empty[buf], (uint32_t)(((k - U3_NB) / U3_NB) & 1));
                    tc::fence_after_sync();
                }
                const uint32_t d_base = tmem + (uint32_t)(buf * U3_BT * 128);
                for (int i = 0; i < 5; ++i) {
                    const int64_t s = k * 5 + i;
                    const int slot = (int)(s % U3_NA);
                    if (!a_ready) tc::mbar_wait(&S.a_full[slot], (uint32_t)((s / U3_NA) & 1));
                    tc::fence_after_sync();
                    // descriptors once per slice; the 16 MMAs add constant offsets (16-byte units)
                    const uint32_t a_base = tc::smem_u32(S.a[slot][0]);
                    const uint64_t ad_lo = tc::make_desc(a_base, plane_bytes, 128);            // blocks 0, 1
                    const uint64_t ad_hi = tc::make_desc(a_base + 2 * plane_bytes, 16u, 128);  // block 2, next pixel
                    const uint64_t bd_i = bdesc0 + (uint64_t)(i * 8 * 2 * NP);
#pragma unroll
                    for (int r8 = 0; r8 < 8; ++r8) {
                        if (r8 == 6) {
                            a_ready = s + 1 < total_s &&
                                      tc::mbar_test(&S.a_full[(s + 1) % U3_NA], (uint32_t)(((s + 1) / U3_NA) & 1));
                            if (c6_next < k && !t5_ready)
                                t5_ready = tc::mbar_test(&S.t5_full[c6_next % U3_NB], (uint32_t)((c6_next / U3_NB) & 1));
                        }
                        // r8 < 5: channels 0-15 of tap (i, r8) (blocks 0 and 1); r8 >= 5: channels
                        // 16-19 of taps (i, j) and (i, j+1), j = 2(r8-5) (block 2, next pixel)
                        const uint64_t ad = r8 < 5 ? ad_lo + (uint64_t)r8 : ad_hi + (uint64_t)(2 * (r8 - 5));
                        const uint64_t bd = bd_i + (uint64_t)(r8 * 2 * NP);
#pragma unroll
                        for (int t = 0; t < U3_BT; ++t)
                            tc::mma_bf16(d_base + (uint32_t)(t * 128), ad + (uint64_t)(t * kTileM), bd, idesc,
                                         (i | r8) > 0 ? 1u : 0u);
                    }
                    tc::commit(&S.a_empty[slot]);
                    if (i == 4) tc::commit(&S.t_full[buf]);
                    // the previous band's C6 as soon as its T5 is ready (between slices)
                    if (t5_ready) {
                        tc::fence_after_sync();
                        issue_c6(c6_next++);
                        t5_ready = false;
                    }
                }
            }
            while (c6_next < my_bands) {
                tc::mbar_wait(&S.t5_full[c6_next % U3_NB], (uint32_t)((c6_next / U3_NB) & 1));
                tc::fence_after_sync();
                issue_c6(c6_next++);
            }
        }
        __syncwarp();
    } else {
        // ---------------------------------------------------------------- epilogue groups
        // Two groups of 8 warps take alternate bands (group g: bands k = g, g+2, ..., always TMEM
        // buffer g), so one group's wait for its C6 result overlaps the other group's drain.
        // Thread = one output position of the band (tile t, TMEM lane group warp % 4), all NP
        // channels in chunks of 16 TMEM columns. Bias-plane values are loaded RING chunks ahead
        // (across band boundaries), so their L2 latency hides behind the chunk compute.
        const int grp = warp / (4 * U3_BT);
        const int t = (warp >> 2) % U3_BT;  // tile
        const uint32_t lane_base = (uint32_t)(32 * (warp & 3)) << 16;
        const int m = t * kTileM + 32 * (warp & 3) + lane;
        constexpr int NC = 2 * NCH;     // 16-column chunks (NP = 16 NC or 16 NC - 16)
        const int nc = NP / 16;
        struct Pos {
            int img, orow, ocol;  // image, global output row, column (32-bit: per-chunk extents)
            bool ok;
            const float* pb;      // bias-plane address of channel 0 at this position
        };
        const uint32_t bcs = a.b5_plane ? (uint32_t)(a.b5_rows * a.w5) : 1u;  // channel stride of the bias
        const int w4 = (int)a.w4, w5 = (int)a.w5, orow_end = (int)(a.out_row0 + a.out_rows);
        auto pos_of = [&](int64_t band) {
            Pos q;
            const int64_t img = (uint32_t)band / (uint32_t)per_img;
            const int qq = (int)(band - img * per_img) * U3_BT * kTileM + m;
            q.img = (int)img;
            const int r = qq / w4;
            q.orow = (int)a.out_row0 + r;
            q.ocol = qq - r * w4;
            q.ok = q.orow < orow_end && q.ocol < w5;
            // positions past the chunk's last row / the row's last column compute on clamped
            // (in-bounds) bias addresses and are not stored: the drain stays branch-free
            const int orow_c = min(q.orow, orow_end - 1), ocol_c = min(q.ocol, w5 - 1);
            const int64_t pix = (int64_t)(orow_c - a.b5_row0) * w5 + ocol_c;
            q.pb = a.b5_plane ? a.b5 + (BQ == 1 ? 4 * pix : pix) : a.b5;
            return q;
        };
        // bias ring of 2 chunk buffers loaded 2 chunks ahead (nc is even or 1 ... the ring index
        // of chunk c is c % 2 in every band when nc is even; for odd nc the ring degenerates to
        // one buffer loaded one chunk ahead)
        float bv[2][16];
        auto load_bias = [&](const float* pb, int c, int r) {
            if (BQ == 1) {              // channel quads (or a scalar bias): 4 x 128-bit loads
                const float4* p4 = reinterpret_cast<const float4*>(pb) + (size_t)(4 * c) * bcs;
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const float4 f = (16 * c + 4 * u < a.n5) ? __ldg(p4 + (size_t)u * bcs) : make_float4(0.f, 0.f, 0.f, 0.f);
                    bv[r][4 * u] = f.x;
                    bv[r][4 * u + 1] = f.y;
                    bv[r][4 * u + 2] = f.z;
                    bv[r][4 * u + 3] = f.w;
                }
                return;
            }
            const float* p = pb + (size_t)(16 * c) * bcs;
            if (16 * c + 16 <= a.n5) {  // a full chunk of real channels (uniform)
#pragma unroll
                for (int u = 0; u < 16; ++u, p += bcs) bv[r][u] = __ldg(p);
            } else {                    // padding channels: accumulator 0, C6 weight 0
#pragma unroll
                for (int u = 0; u < 16; ++u, p += bcs) bv[r][u] = (16 * c + u < a.n5) ? __ldg(p) : 0.f;
            }
        };
        // channel quads: one chunk ahead (a ring of two loaded two chunks ahead -- 32 registers
        // instead of 16 at the 96-register budget of 576 threads -- measured 2-3 % slower, DESIGN.md
        // §5.3); scalar loads (planes): two chunks ahead (one spills)
        const int ring = (BQ == 1 || nc % 2) ? 1 : 2;
        const int64_t first = blockIdx.x + (int64_t)grp * gridDim.x;
        Pos cur = pos_of(first);
        if (first < nbands) {
            load_bias(cur.pb, 0, 0);
            if (ring == 2) load_bias(cur.pb, 1, 1);
        }
        int64_t k = grp;
        for (int64_t band = first; band < nbands; band += kEpiGroups * gridDim.x, k += kEpiGroups) {
            const int buf = (int)(k % U3_NB);
            const uint32_t region = tmem + lane_base + (uint32_t)((buf * U3_BT + t) * 128);
            const bool has_next = band + kEpiGroups * gridDim.x < nbands;
            const float* nxt_pb = pos_of(has_next ? band + kEpiGroups * gridDim.x : band).pb;
            tc::mbar_wait(&S.t_full[buf], (uint32_t)((k / U3_NB) & 1));
            tc::fence_after_sync();
#pragma unroll
            for (int c = 0; c < NC; ++c) {
                if (c < nc) {
                    float v[16];
                    tc::tmem_ld16_async(region + (uint32_t)(16 * c), v);
                    tc::tmem_wait_ld();
                    const int rb = ring == 2 ? (c & 1) : 0;
                    if (rb == 0) {
#pragma unroll
                        for (int u = 0; u < 16; ++u) v[u] = tanh_approx(v[u] + bv[0][u]);
                    } else {
#pragma unroll
                        for (int u = 0; u < 16; ++u) v[u] = tanh_approx(v[u] + bv[1][u]);
                    }
                    uint32_t r[8];
#pragma unroll
                    for (int u = 0; u < 8; ++u) r[u] = tc::pack_bf16(v[2 * u], v[2 * u + 1]);
                    // refill the consumed buffer with the chunk `ring` steps ahead
                    const int cn = c + ring;
                    if (rb == 0) {
                        if (cn < nc) load_bias(cur.pb, cn, 0);
                        else if (has_next) load_bias(nxt_pb, cn - nc, 0);
                    } else {
                        if (cn < nc) load_bias(cur.pb, cn, 1);
                        else if (has_next) load_bias(nxt_pb, cn - nc, 1);
                    }
                    // T5 chunk c -> TMEM columns [8c, 8c+8) (already drained), bf16 pairs
                    tc::tmem_st8(region + (uint32_t)(8 * c), r);
                }
            }
            tc::tmem_wait_st();
            tc::fence_before_sync();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&S.t5_full[buf]);  // T5 ready for the C6 MMA
            float d6[16];
            tc::mbar_wait(&S.c6_full[buf], (uint32_t)((k / U3_NB) & 1));
            tc::fence_after_sync();
            tc::tmem_ld16_async(region + (uint32_t)U3_C6COL, d6);
            tc::tmem_wait_ld();
            tc::fence_before_sync();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&S.t_empty[buf]);  // the accumulator can be reused
            if (cur.ok) {
                float* ob = a.out + cur.img * a.out_img_stride + (int64_t)(cur.orow - a.out_row0) * w5 + cur.ocol;
#pragma unroll
                for (int o = 0; o < 9; ++o) {
                    const float b = a.b6_plane
                                        ? __ldg(a.b6 + ((int64_t)o * a.b6_rows + (cur.orow - a.b6_row0)) * w5 + cur.ocol)
                                        : __ldg(a.b6 + o);
                    ob[o * a.out_plane_stride] = d6[o] + b;
                }
            }
            if (has_next) cur = pos_of(band + kEpiGroups * gridDim.x);
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

// B operand of C3 for the 18 K-steps (window row y, tap pair (j, j+1)): [ks][half][n<48][8 ci];
// half h holds tap j + h (zero for j + h == 5); columns n < 20 = map n with filter row y (C3 row
// 2R), 24 <= n < 44 = map n - 24 with filter row y - 1 (C3 row 2R+1), zero where the filter row
// is outside 0..4 and in the padding columns.
size_t cnn_k3_tc_bytes() { return (size_t)U2_KS * 2 * U2_N * 8 * 2; }
void cnn_prepare_k3_tc(const float* k3, uint16_t* dst) {
    for (int ks = 0; ks < U2_KS; ++ks) {
        const int y = ks / 3, j0 = 2 * (ks % 3);
        for (int h = 0; h < 2; ++h)
            for (int n = 0; n < U2_N; ++n)
                for (int e = 0; e < 8; ++e) {
                    const int j = j0 + h;
                    const int t = n >= U2_ROW1 ? 1 : 0, map = n - t * U2_ROW1, i = y - t;
                    const bool ok = map < 20 && j < 5 && i >= 0 && i < 5;
                    const float v = ok ? k3[(map * 8 + e) * 25 + i * 5 + j] : 0.f;
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
    // the epilogue addresses bias channels with 32-bit offsets
    if (a.b3_plane && 20 * a.b3_rows * a.w3 >= (1ll << 32)) return cudaErrorInvalidValue;
    if (!set_smem_attr((const void*)cnn_u2_tc_kernel, smem, flags)) return cudaErrorInvalidValue;
    U2P pw;
    std::memcpy(pw.p4, a.p4_host, sizeof pw.p4);
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t nseg = a.t4_rows * ((a.w3 + kTileM - 1) / kTileM) * a.nimg;
    if (nseg >= (1ll << 32)) return cudaErrorInvalidValue;  // 32-bit segment indexing in the kernel
    const unsigned grid = (unsigned)std::min<int64_t>(nseg, sms);
    cnn_u2_tc_kernel<<<grid, kThreadsU2, smem, s>>>(a, pw, nseg);
    return cudaGetLastError();
}

cudaError_t launch_cnn_u3_tc(const CnnU3Args& a, cudaStream_t s) {
    if (a.out_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    if (a.n_pad > U3_NMAX || a.n_pad % 16 || a.n5 > U3_NMAX) return cudaErrorInvalidValue;
    const size_t smem = sizeof(U3Smem) + 128;
    const int nch = (a.n_pad + 31) / 32;
    // a scalar bias ([n5], 16-byte aligned in the arena) is read like one position of channel quads
    const int q4 = (a.b5_plane ? a.b5_q4 != 0 : a.n5 % 4 == 0) ? 1 : 0;
    const void* fns[2][4] = {{(const void*)cnn_u3_tc_kernel<1, 0>, (const void*)cnn_u3_tc_kernel<2, 0>,
                              (const void*)cnn_u3_tc_kernel<3, 0>, (const void*)cnn_u3_tc_kernel<4, 0>},
                             {(const void*)cnn_u3_tc_kernel<1, 1>, (const void*)cnn_u3_tc_kernel<2, 1>,
                              (const void*)cnn_u3_tc_kernel<3, 1>, (const void*)cnn_u3_tc_kernel<4, 1>}};
    static std::atomic<uint32_t> flag_n[2][4];
    if (!set_smem_attr(fns[q4][nch - 1], smem, flag_n[q4][nch - 1])) return cudaErrorInvalidValue;
    const int64_t per_img = (a.out_rows * a.w4 + U3_BT * kTileM - 1) / (U3_BT * kTileM);
    // the epilogue addresses bias channels with 32-bit offsets
    if (a.b5_plane && (int64_t)a.n5 * a.b5_rows * a.w5 >= (1ll << 32)) return cudaErrorInvalidValue;
    // C6 B operand: bf16 [ks][half][o][8 ch], value K6[o][16 ks + 8 half + e] (zero padding)
    U3P pw{};
    uint16_t* b6 = reinterpret_cast<uint16_t*>(pw.b6);
    for (int ks = 0; ks < U3_C6K; ++ks)
        for (int h = 0; h < 2; ++h)
            for (int o = 0; o < U3_C6N; ++o)
                for (int e = 0; e < 8; ++e) {
                    const int ch = 16 * ks + 8 * h + e;
                    b6[((ks * 2 + h) * U3_C6N + o) * 8 + e] = to_bf16(o < 9 && ch < a.n5 ? a.k6_host[o * a.n5 + ch] : 0.f);
                }
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t nbands = per_img * a.nimg;
    if (nbands >= (1ll << 32)) return cudaErrorInvalidValue;  // 32-bit band indexing in the kernel
    const unsigned grid = (unsigned)std::min<int64_t>(nbands, sms);
    void* args[] = {(void*)&a, (void*)&pw, (void*)&nbands};
    return cudaLaunchKernel(fns[q4][nch - 1], dim3(grid), dim3(kThreadsU3), args, smem, s);
}

}  // namespace tg
