// cnn_h3.cu -- U2 (C3 T S4 T) and U3 (C5 T C6) with fp32 accuracy on the tcgen05 tensor cores
// from fp16 operands: "3xFP16" (precision TG_FP32_TC, sm_100a).
//
// Every operand is scaled by a power of two and split into two fp16 numbers,
//   x' = x * 2^s,  hi = fp16_rn(x'),  lo = fp16_rn(x' - hi),   |x' - hi - lo| <= 2^-22 |x'|
// (activations T2/T4 in [-1, 1]: s = 4; weights: s chosen per layer on the host so that max |w| x 2^s
// lies in [2^13, 2^14) -- both keep hi and lo in the fp16 normal range for every value that
// matters, for any weight magnitude; a lo that falls into the subnormals errs by at most 2^-25
// of the scaled range). A product is accumulated from three MMAs, hi.hi + hi.lo + lo.hi, in fp32
// in TMEM (lo.lo < 2^-22 of the product is dropped), and the result is scaled back by the exact
// power of two w_unscale. fp16 carries as many mantissa bits as TF32 (11) at half the bytes, and kind::f16 MMAs
// take K = 16 at twice the TF32 rate: the same fp32 accuracy as the 3xTF32 kernels (cnn_t32.cu)
// for half the shared-memory operand traffic per K element and half the MMA time (this replaced a
// 3xTF32 implementation of the same layers: U2 0.43 -> 0.32 ms, U3 0.88 -> 0.55 ms on cnn3).
//
// Data between units (written by the producing unit's epilogue, pixel-blocked like the bf16 path):
//   T2 [part][rows][w2][8 ch]          part 0 = hi, 1 = lo (16 B per pixel per part)
//   T4 [part][block][rows][w4][8 ch]   blocks: channels 0-7, 8-15, 16-19 + 4 zeros
// The implicit GEMMs are those of the bf16 kernels (cnn_tc.cu): U2 pairs taps (j, j+1) in one
// K = 16 step (18 K-steps per segment: 6 window rows x 3 tap pairs, both C3 rows in N), U3 runs
// 8 K-steps per filter row (taps 0-4 over blocks 0-1, then block 2 of tap pairs), 40 per tile.
//   U2: as the bf16 U2, ONE M = 128 tile per segment serves both C3 rows (window row y feeds row
//       2R with filter row y and row 2R+1 with filter row y - 1: N = 48, 18 K-steps of 6 window
//       rows x 3 tap pairs), and A_hi is read ONCE for both of its products: A_hi x [B_hi | B_lo]
//       (N = 96) and A_lo x B_hi (N = 48) accumulated onto the hi.hi columns; the epilogue adds
//       the two 48-column halves. (Earlier: two tiles of 15 K-steps at N = 64 + 32, 2640 vs 1800
//       shared-memory operand cycles per segment.)
//   U3: three MMAs per K-step into one accumulator (N = n5 padded to 16), or for NP <= 64 the
//       same read-once fusion as U2; the B operand (40 K-steps x 2 parts, up to 320 KB) streams
//       through a ring of 32 KB stages.
// Both kernels are persistent and warp-specialised (copy producer warp, MMA issuer warp, epilogue
// warps), like their bf16 and 3xTF32 counterparts.
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstring>
#include <vector>

#include "kernels.h"
#include "tanh_fp32.cuh"
#include "tc_sm100.cuh"

namespace tg {
namespace {

// tanh of the fp32 paths (tanh_fp32.cuh): a few ulps relative, also near 0
__device__ __forceinline__ float tanh_acc(float x) { return tanh_fp32(x); }

constexpr float kActScale = 16.f;          // 2^4: activations (T2, T4: tanh outputs, |x| <= 1)

// hi/lo fp16 pairs of two consecutive channels (element 0 in the low half, as the MMA reads K)
__device__ __forceinline__ void split2(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    const __half2 h = __floats2half2_rn(x0, x1);
    const float2 hf = __half22float2(h);
    const __half2 l = __floats2half2_rn(x0 - hf.x, x1 - hf.y);
    hi = *reinterpret_cast<const uint32_t*>(&h);
    lo = *reinterpret_cast<const uint32_t*>(&l);
}

// instruction descriptor, kind::f16 with fp16 A and B (format 0), D F32, both K-major
__host__ __device__ constexpr uint32_t idesc_f16(int M, int N) {
    return (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

constexpr int kTileM = 128;

bool set_smem_attr_h3(const void* fn, size_t bytes, std::atomic<uint32_t>& flags) {
    int dev = 0;
    cudaGetDevice(&dev);
    const uint32_t bit = 1u << (dev & 31);
    if (flags.load() & bit) return true;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) != cudaSuccess) return false;
    flags.fetch_or(bit);
    return true;
}

uint16_t to_f16(float f) {
    const __half h = __float2half_rn(f);
    return *reinterpret_cast<const uint16_t*>(&h);
}
float from_f16(uint16_t u) {
    __half h;
    std::memcpy(&h, &u, 2);
    return __half2float(h);
}

// ============================================================================ U2 (C3)
// Segment = T4 row R (C3 rows 2R, 2R+1) x 128 C3 columns, one M = 128 tile. Window: T2 rows
// [2R, 2R+6) x cols [c0, c0+134) of both parts, [part][row][col] -> 8 fp16 channels.
constexpr int U2H_WR = 6, U2H_WP = kTileM + 6;
constexpr int U2H_N = 48;                  // [0,20) row 2R, [24,44) row 2R+1; B rows per K half = 2 x U2H_N
constexpr int U2H_ROW1 = 24;               // first column of C3 row 2R+1
constexpr int U2H_KS = 18;                 // 6 window rows x tap pairs (0,1) (2,3) (4,5)
constexpr int U2H_NA = 6;                  // window buffers
constexpr int U2H_NT = 4;                  // TMEM slots (128 columns apart, 2 x U2H_N used)
constexpr int U2H_PLANE = U2H_WR * U2H_WP;
constexpr int kThreads = 10 * 32;
constexpr int U2H_G = 3;                    // U2 epilogue groups (4 warps each), taking segments in turn
constexpr int kThreadsU2H = (4 * U2H_G + 2) * 32;

struct U2HP {
    float p4[20][4];  // S4 weights (constant bank)
};

struct U2HSmem {
    uint4 a[U2H_NA][2][U2H_PLANE];           // [buf][part][row*WP + col] -> 8 fp16
    uint4 b[U2H_KS * 2 * 2 * U2H_N];         // [ks][half][row < 96: hi columns, then lo] -> 8 fp16
    uint64_t b_full, a_full[U2H_NA], a_empty[U2H_NA], t_full[U2H_NT], t_empty[U2H_NT];
    uint32_t tmem;
};

__global__ void __launch_bounds__(kThreadsU2H, 1)
    cnn_u2_h3_kernel(const CnnU2Args a, const __grid_constant__ U2HP pw, const int64_t nseg) {
    extern __shared__ __align__(128) uint8_t smraw[];
    U2HSmem& S = *reinterpret_cast<U2HSmem*>(smraw + ((128 - (tc::smem_u32(smraw) & 127)) & 127));
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

    if (warp == 0) tc::tmem_alloc<512>(&S.tmem);
    if (tid == 0) {
        tc::mbar_init(&S.b_full, 1);
        for (int i = 0; i < U2H_NA; ++i) {
            tc::mbar_init(&S.a_full[i], 1);
            tc::mbar_init(&S.a_empty[i], 1);
        }
        for (int i = 0; i < U2H_NT; ++i) {
            tc::mbar_init(&S.t_full[i], 1);
            tc::mbar_init(&S.t_empty[i], 4);
        }
        tc::mbar_fence_init();
    }
    // windows start zeroed: pixels a copy does not cover (beyond the image) only ever hold
    // finite T2 values; they feed C3 columns that are not stored
    for (int idx = tid; idx < U2H_NA * 2 * U2H_PLANE; idx += kThreadsU2H) (&S.a[0][0][0])[idx] = make_uint4(0u, 0u, 0u, 0u);
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    const uint32_t tmem = S.tmem;
    const int64_t my = nseg > blockIdx.x ? (nseg - 1 - blockIdx.x) / gridDim.x + 1 : 0;

    if (warp == 4 * U2H_G + 1) {
        // ---------------------------------------------------------------- copy producer
        const uint4* t2all = reinterpret_cast<const uint4*>(a.t2);
        const int64_t tplane = a.t2_rows * a.w2;  // pixels per part plane of one image's T2
        const uint32_t bbytes = (uint32_t)(U2H_KS * 2 * 2 * U2H_N * 16);
        if (tc::elect_one()) {
            tc::mbar_expect_tx(&S.b_full, bbytes);
            tc::bulk_g2s(S.b, a.k3_h3, bbytes, &S.b_full);
        }
        __syncwarp();
        for (int64_t k = 0; k < my; ++k) {
            const int buf = (int)(k % U2H_NA);
            if (k >= U2H_NA) tc::mbar_wait(&S.a_empty[buf], (uint32_t)(((k - U2H_NA) / U2H_NA) & 1));
            int64_t img, R, c0;
            seg_coords(blockIdx.x + k * gridDim.x, img, R, c0);
            const int64_t r0 = 2 * R - a.t2_row0;
            const int64_t rows = min((int64_t)U2H_WR, a.t2_rows - r0);
            const int64_t cols = min((int64_t)U2H_WP, a.w2 - c0);
            // 2 parts x `rows` window rows, one bulk copy per lane in one warp instruction
            if (lane == 0) tc::mbar_expect_tx(&S.a_full[buf], (uint32_t)(2 * rows * cols * 16));
            __syncwarp();
            if (lane < 2 * rows) {
                const int part = lane / (int)rows, r = lane - part * (int)rows;
                const uint4* src = t2all + (img * 2 + part) * tplane + (r0 + r) * a.w2 + c0;
                tc::bulk_g2s(&S.a[buf][part][r * U2H_WP], src, (uint32_t)(cols * 16), &S.a_full[buf]);
            }
            __syncwarp();
        }
    } else if (warp == 4 * U2H_G) {
        // ---------------------------------------------------------------- MMA issuer
        // ONE elected lane runs the whole loop (warp-level hand-offs per segment left the tensor
        // pipe idle, tools/micro/umma_probe.cu)
        if (tc::elect_one()) {
            tc::mbar_wait(&S.b_full, 0);
            const uint32_t idesc2n = idesc_f16(kTileM, 2 * U2H_N), idesc1n = idesc_f16(kTileM, U2H_N);
            // descriptors: the start address is the low 14 bits (16-byte units), advanced by adding;
            // A: the second K half is the next pixel (tap j+1, LBO = 16 B); B: LBO = one K half
            const uint64_t a_desc0 = tc::make_desc(tc::smem_u32(S.a[0][0]), 16, 128);
            const uint64_t b_desc0 = tc::make_desc(tc::smem_u32(S.b), 2 * U2H_N * 16, 128);
            for (int64_t k = 0; k < my; ++k) {
                const int buf = (int)(k % U2H_NA), ts = (int)(k % U2H_NT);
                tc::mbar_wait(&S.a_full[buf], (uint32_t)((k / U2H_NA) & 1));
                if (k >= U2H_NT) tc::mbar_wait(&S.t_empty[ts], (uint32_t)(((k - U2H_NT) / U2H_NT) & 1));
                tc::fence_after_sync();
                const uint64_t abuf = a_desc0 + (uint64_t)(buf * (2 * U2H_PLANE));
                const uint32_t d = tmem + (uint32_t)(ts * 128);
#pragma unroll
                for (int ks = 0; ks < U2H_KS; ++ks) {  // window row y = ks / 3, tap pair (j, j+1)
                    const int y = ks / 3, j = 2 * (ks % 3);
                    const uint64_t a_hi = abuf + (uint64_t)(y * U2H_WP + j);
                    const uint64_t a_lo = a_hi + (uint64_t)U2H_PLANE;
                    const uint64_t b_ks = b_desc0 + (uint64_t)(ks * 2 * 2 * U2H_N);  // rows 0..47 = B_hi
                    // hi.hi -> [0, 48), hi.lo -> [48, 96); lo.hi accumulates onto hi.hi
                    tc::mma_bf16(d, a_hi, b_ks, idesc2n, ks > 0 ? 1u : 0u);
                    tc::mma_bf16(d, a_lo, b_ks, idesc1n, 1u);
                }
                tc::commit(&S.a_empty[buf]);
                tc::commit(&S.t_full[ts]);
            }
        }
        __syncwarp();
    } else {
        // ---------------------------------------------------------------- epilogue groups
        const int grp = warp >> 2, wq = warp & 3;
        const uint32_t lane_base = (uint32_t)(32 * wq) << 16;
        const int64_t bplane = a.t4_rows * a.w4;
        float b0v[20], b1v[20];
        const uint32_t bcs = a.b3_plane ? (uint32_t)(a.b3_rows * a.w3) : 1u;
        const uint32_t brs = a.b3_plane ? (uint32_t)a.w3 : 0u;
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
        for (int64_t k = grp; k < my; k += U2H_G) {
            const int ts = (int)(k % U2H_NT);
            int64_t img, R, c0;
            seg_coords(blockIdx.x + k * gridDim.x, img, R, c0);
            const int64_t c = c0 + 32 * wq + lane;  // C3 column
            const int64_t C = c >> 1;               // T4 column
            tc::mbar_wait(&S.t_full[ts], (uint32_t)((k / U2H_NT) & 1));
            tc::fence_after_sync();
            float v0[20], v1[20];
            {
                // columns [0, 48) hi.hi + lo.hi, [48, 96) hi.lo; C3 row 2R at column co, row 2R+1
                // at U2H_ROW1 + co (20 maps each)
                const uint32_t tb = tmem + lane_base + (uint32_t)(ts * 128);
                float p[32], q[32];
                tc::tmem_ld32_async(tb, p);           // [0, 32)
                tc::tmem_ld32_async(tb + U2H_N, q);   // [48, 80)
                tc::tmem_wait_ld();
#pragma unroll
                for (int co = 0; co < 20; ++co) v0[co] = (p[co] + q[co]) * a.w_unscale;
#pragma unroll
                for (int co = 0; co < 8; ++co) v1[co] = (p[U2H_ROW1 + co] + q[U2H_ROW1 + co]) * a.w_unscale;
                float p2[16], q2[16];
                tc::tmem_ld16_async(tb + 32, p2);           // [32, 48)
                tc::tmem_ld16_async(tb + U2H_N + 32, q2);   // [80, 96)
                tc::tmem_wait_ld();
#pragma unroll
                for (int co = 8; co < 20; ++co) v1[co] = (p2[U2H_ROW1 + co - 32] + q2[U2H_ROW1 + co - 32]) * a.w_unscale;
            }
            tc::fence_before_sync();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&S.t_empty[ts]);
            const bool out_ok = !(lane & 1) && C < a.w4;
            // the two C3 rows' tanh as one pair (tanh_fp32x2: paired FP32 arithmetic, bit-identical
            // to the scalar form), then the S4 tanh of channels (co, co+1) as one pair
            float tv[24];
#pragma unroll
            for (int co = 0; co < 20; co += 2) {
                float s4[2];
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    const float2 t = tanh_fp32x2(__fadd2_rn(make_float2(v0[co + e], v1[co + e]),
                                                            make_float2(b0v[co + e], b1v[co + e])));
                    const float t01 = __shfl_down_sync(0xffffffffu, t.x, 1);  // column c+1
                    const float t11 = __shfl_down_sync(0xffffffffu, t.y, 1);
                    float s = 0.f;
                    s = fmaf(pw.p4[co + e][0], t.x, s);
                    s = fmaf(pw.p4[co + e][1], t01, s);
                    s = fmaf(pw.p4[co + e][2], t.y, s);
                    s4[e] = fmaf(pw.p4[co + e][3], t11, s);
                }
                const float2 t4 = tanh_fp32x2(make_float2(s4[0], s4[1]));
                tv[co] = t4.x * kActScale;
                tv[co + 1] = t4.y * kActScale;
            }
#pragma unroll
            for (int co = 20; co < 24; ++co) tv[co] = 0.f;
            if (k + U2H_G < my) load_bias(k + U2H_G);
            if (out_ok) {
                uint4* t4 = reinterpret_cast<uint4*>(a.t4) + img * 6 * bplane + (R - a.t4_row0) * a.w4 + C;
#pragma unroll
                for (int blk = 0; blk < 3; ++blk) {
                    uint32_t hi[4], lo[4];
#pragma unroll
                    for (int m = 0; m < 4; ++m) split2(tv[8 * blk + 2 * m], tv[8 * blk + 2 * m + 1], hi[m], lo[m]);
                    t4[blk * bplane] = make_uint4(hi[0], hi[1], hi[2], hi[3]);
                    t4[(3 + blk) * bplane] = make_uint4(lo[0], lo[1], lo[2], lo[3]);
                }
            }
        }
    }
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<512>(tmem);
}

// ============================================================================ U3 (C5 + C6)
// Band = 256 consecutive output positions in the flat (row, col) index with pitch w4 (two M=128
// tiles); filter row i reads slice i = flat T4 pixels [q0 + i*w4, +262) of both parts and all 3
// blocks. 8 K-steps per filter row (as the bf16 U3): r8 < 5 = channels 0-15 of tap (i, r8)
// (blocks 0, 1; LBO = one block plane), r8 >= 5 = channels 16-19 of taps (i, j), (i, j+1) with
// j = 2 (r8 - 5) (block 2, next pixel: LBO = 16 B); 40 K-steps x 3 MMAs per tile.
//   warp 9   copy producer: slices through a ring of 3 buffers (6 bulk copies each, by 6 lanes),
//            B stages of 4 K-steps (32 KB at NP = 128) through a ring of 3
//   warp 8   MMA issuer: per K-step 3 MMAs x 2 tiles into one of two TMEM accumulators
//   0-7      epilogue: TMEM -> registers, x 2^-12, + bias plane, tanh, the 1x1 C6 as fp32 FMAs
//            over n5 (weights in the constant bank), + C6 bias -> output
constexpr int U3H_KS = 40;
constexpr int U3H_KST = 4;                   // K-steps per B stage
constexpr int U3H_NST = U3H_KS / U3H_KST;    // 10 stages per band
constexpr int U3H_BRING = 3;
constexpr int U3H_NMAX = 128;
constexpr int U3H_SPX = 2 * kTileM + 8;      // pixels per slice block (262 used)
constexpr int U3H_NA = 3;                    // slice buffers
constexpr int kEpiWarps = 8;

struct U3HK6 {
    float k6[U3H_NMAX][12];  // [ch][o] (9 used): C6 weights, broadcast from the constant bank
};

struct U3HSmem {
    uint4 b[U3H_BRING][U3H_KST * 2 * 2 * U3H_NMAX];  // [stage][u][part][half][n] -> 8 fp16
    uint4 a[U3H_NA][2][3][U3H_SPX];                  // [slot][part][block][pixel] -> 8 fp16
    uint64_t a_full[U3H_NA], a_empty[U3H_NA], b_full[U3H_BRING], b_empty[U3H_BRING], t_full[2], t_empty[2];
    uint32_t tmem;
};

// NCH <= 2 (NP <= 64, the small net): like U2, A_hi is read once for both of its products --
// [B_hi | B_lo] at N = 2 NP, A_lo x B_hi onto the cross-term columns -- and a tile's accumulator is
// 2 NP columns (2 tiles x 2 buffers fit the 512 TMEM columns); larger NP: three MMAs into NP columns.
template <int NCH>  // TMEM chunks of 32 columns: NP = n5 padded to 16, NCH = ceil(NP / 32)
__global__ void __launch_bounds__(kThreads, 1)
    cnn_u3_h3_kernel(const CnnU3Args a, const __grid_constant__ U3HK6 k6w, const int64_t nbands) {
    extern __shared__ __align__(128) uint8_t smraw[];
    U3HSmem& S = *reinterpret_cast<U3HSmem*>(smraw + ((128 - (tc::smem_u32(smraw) & 127)) & 127));
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    constexpr bool kFuse = NCH <= 2;
    const int NP = a.n_pad;
    const int64_t per_img = (a.out_rows * a.w4 + 2 * kTileM - 1) / (2 * kTileM);
    const int64_t bplane = a.t4_rows * a.w4;                 // pixels per block plane of one image
    const int64_t flat0 = (a.out_row0 - a.t4_row0) * a.w4;  // flat index of output row 0 in the T4 buffer

    if (warp == 0) tc::tmem_alloc<512>(&S.tmem);
    if (tid == 0) {
        for (int i = 0; i < U3H_NA; ++i) {
            tc::mbar_init(&S.a_full[i], 1);
            tc::mbar_init(&S.a_empty[i], 1);
        }
        for (int i = 0; i < U3H_BRING; ++i) {
            tc::mbar_init(&S.b_full[i], 1);
            tc::mbar_init(&S.b_empty[i], 1);
        }
        for (int i = 0; i < 2; ++i) {
            tc::mbar_init(&S.t_full[i], 1);
            tc::mbar_init(&S.t_empty[i], kEpiWarps);
        }
        tc::mbar_fence_init();
    }
    // slice buffers start zeroed: pixels a copy does not cover (past the chunk's last T4 row)
    // then only ever hold finite values; they feed positions that are not stored
    for (int idx = tid; idx < U3H_NA * 2 * 3 * U3H_SPX; idx += kThreads) (&S.a[0][0][0][0])[idx] = make_uint4(0u, 0u, 0u, 0u);
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    const uint32_t tmem = S.tmem;
    const int64_t my_bands = nbands > blockIdx.x ? (nbands - 1 - blockIdx.x) / gridDim.x + 1 : 0;

    if (warp == kEpiWarps + 1) {
        // ---------------------------------------------------------------- copy producer
        const uint4* t4all = reinterpret_cast<const uint4*>(a.t4);
        const uint8_t* kb = reinterpret_cast<const uint8_t*>(a.k5_tc);
        const uint32_t stage_bytes = (uint32_t)(U3H_KST * 2 * 2 * NP * 16);
        int64_t si = 0, gi = 0;  // slices and B stages issued so far
        for (int64_t k = 0; k < my_bands; ++k) {
            const int64_t band = blockIdx.x + k * gridDim.x;
            const int64_t img = (uint32_t)band / (uint32_t)per_img;
            const int64_t q0 = (band - img * per_img) * 2 * kTileM;
            for (int ks = 0; ks < U3H_KS; ++ks) {
                if (ks % 8 == 0) {  // slice i = ks / 8
                    const int slot = (int)(si % U3H_NA);
                    if (si >= U3H_NA) tc::mbar_wait(&S.a_empty[slot], (uint32_t)(((si - U3H_NA) / U3H_NA) & 1));
                    const int64_t e = flat0 + q0 + (int64_t)(ks / 8) * a.w4;
                    const int64_t n = max((int64_t)0, min((int64_t)U3H_SPX, bplane - e));
                    if (lane == 0) tc::mbar_expect_tx(&S.a_full[slot], (uint32_t)(6 * n * 16));
                    __syncwarp();
                    if (n > 0 && lane < 6) {
                        const int part = lane / 3, blk = lane - 3 * part;
                        tc::bulk_g2s(S.a[slot][part][blk], t4all + ((img * 2 + part) * 3 + blk) * bplane + e,
                                     (uint32_t)(n * 16), &S.a_full[slot]);
                    }
                    __syncwarp();
                    ++si;
                }
                if (ks % U3H_KST == 0) {  // B stage ks / 4
                    const int slot = (int)(gi % U3H_BRING);
                    if (gi >= U3H_BRING) tc::mbar_wait(&S.b_empty[slot], (uint32_t)(((gi - U3H_BRING) / U3H_BRING) & 1));
                    if (tc::elect_one()) {
                        tc::mbar_expect_tx(&S.b_full[slot], stage_bytes);
                        tc::bulk_g2s(S.b[slot], kb + (size_t)(ks / U3H_KST) * stage_bytes, stage_bytes, &S.b_full[slot]);
                    }
                    __syncwarp();
                    ++gi;
                }
            }
        }
    } else if (warp == kEpiWarps) {
        // ---------------------------------------------------------------- MMA issuer
        // ONE elected lane runs the whole loop: a warp-level hand-off after every K-step (6 MMAs)
        // left the tensor pipe idle (tools/micro/umma_probe.cu)
        if (tc::elect_one()) {
            const uint32_t idesc = idesc_f16(kTileM, NP), idesc2 = idesc_f16(kTileM, 2 * NP);
            const uint32_t plane_bytes = (uint32_t)(U3H_SPX * 16), part_bytes = 3 * plane_bytes;
            // Descriptors are built once per slice / B stage and advanced by constant offsets (the
            // start address is the descriptor's low field, in 16-byte units): with the K-step loop
            // unrolled per stage, the issuing thread spends a few uniform adds per MMA instead of
            // rebuilding four descriptors per tile and K-step (which left it barely ahead of the pipe)
            static_assert(U3H_KST == 4 && 8 % U3H_KST == 0, "two B stages per slice");
            const uint64_t b_step = (uint64_t)(2 * 2 * NP);       // one K-step of B, 16-byte units
            const uint64_t b_part = (uint64_t)(2 * NP);           // B_lo after B_hi (NP > 64 layout)
            const uint64_t a_part = (uint64_t)(part_bytes >> 4);  // A_lo after A_hi
            int64_t si = 0, gi = 0;
            for (int64_t k = 0; k < my_bands; ++k) {
                const int buf = (int)(k & 1);
                if (k >= 2) tc::mbar_wait(&S.t_empty[buf], (uint32_t)(((k - 2) >> 1) & 1));
                const uint32_t d_base = tmem + (uint32_t)(buf * 256);
                for (int i = 0; i < 5; ++i) {
                    const int aslot = (int)(si % U3H_NA);
                    tc::mbar_wait(&S.a_full[aslot], (uint32_t)((si / U3H_NA) & 1));
                    ++si;
                    const uint32_t a_base = tc::smem_u32(S.a[aslot][0][0]);
                    // r8 < 5: channels 0-15 of tap (i, r8) (blocks 0, 1; LBO = one block plane);
                    // r8 >= 5: channels 16-19 of taps (i, j), (i, j+1), j = 2 (r8 - 5) (block 2, next pixel)
                    const uint64_t ad_lo = tc::make_desc(a_base, plane_bytes, 128);
                    const uint64_t ad_hi = tc::make_desc(a_base + 2 * plane_bytes, 16u, 128);
#pragma unroll
                    for (int hs = 0; hs < 2; ++hs) {
                        const int bslot = (int)(gi % U3H_BRING);
                        tc::mbar_wait(&S.b_full[bslot], (uint32_t)((gi / U3H_BRING) & 1));
                        ++gi;
                        tc::fence_after_sync();
                        const uint64_t bd0 = kFuse ? tc::make_desc(tc::smem_u32(S.b[bslot]), (uint32_t)(2 * NP * 16), 128)
                                                   : tc::make_desc(tc::smem_u32(S.b[bslot]), (uint32_t)(NP * 16), 128);
#pragma unroll
                        for (int u = 0; u < U3H_KST; ++u) {
                            const int r8 = 4 * hs + u;
                            const uint64_t ad = r8 < 5 ? ad_lo + (uint64_t)r8 : ad_hi + (uint64_t)(2 * (r8 - 5));
                            const uint64_t bd = bd0 + (uint64_t)u * b_step;
                            const uint32_t acc0 = (i | r8) > 0 ? 1u : 0u;
#pragma unroll
                            for (int t = 0; t < 2; ++t) {
                                const uint64_t a_hi = ad + (uint64_t)(t * kTileM), a_lo = a_hi + a_part;
                                if (kFuse) {  // A_hi read once: [B_hi | B_lo] at N = 2 NP, then A_lo x B_hi
                                    const uint32_t d = d_base + (uint32_t)(t * 2 * NP);
                                    tc::mma_bf16(d, a_hi, bd, idesc2, acc0);
                                    tc::mma_bf16(d + (uint32_t)NP, a_lo, bd, idesc, 1u);
                                } else {
                                    const uint32_t d = d_base + (uint32_t)(t * NP);
                                    tc::mma_bf16(d, a_hi, bd, idesc, acc0);
                                    tc::mma_bf16(d, a_hi, bd + b_part, idesc, 1u);
                                    tc::mma_bf16(d, a_lo, bd, idesc, 1u);
                                }
                            }
                        }
                        tc::commit(&S.b_empty[bslot]);
                    }
                    tc::commit(&S.a_empty[aslot]);
                }
                tc::commit(&S.t_full[buf]);
            }
        }
        __syncwarp();
    } else {
        // ---------------------------------------------------------------- epilogue warps
        // Thread = one output position of the band (tile t = warp / 4, TMEM lane group warp % 4),
        // all NP channels in chunks of 32 TMEM columns; bias-plane values loaded one chunk ahead.
        const int t = warp >> 2;
        const uint32_t lane_base = (uint32_t)(32 * (warp & 3)) << 16;
        const int m = t * kTileM + 32 * (warp & 3) + lane;
        const uint32_t bcs = a.b5_plane ? (uint32_t)(a.b5_rows * a.w5) : 1u;
        const int w4 = (int)a.w4, w5 = (int)a.w5, orow_end = (int)(a.out_row0 + a.out_rows);
        struct Pos {
            int img, orow, ocol;
            bool ok;
            const float* pb;
        };
        auto pos_of = [&](int64_t band) {
            Pos q;
            const int64_t img = (uint32_t)band / (uint32_t)per_img;
            const int qq = (int)(band - img * per_img) * 2 * kTileM + m;
            q.img = (int)img;
            const int r = qq / w4;
            q.orow = (int)a.out_row0 + r;
            q.ocol = qq - r * w4;
            q.ok = q.orow < orow_end && q.ocol < w5;
            const int orow_c = min(q.orow, orow_end - 1), ocol_c = min(q.ocol, w5 - 1);
            const int64_t pix = (int64_t)(orow_c - a.b5_row0) * w5 + ocol_c;
            q.pb = a.b5_plane ? a.b5 + (a.b5_q4 ? 4 * pix : pix) : a.b5;
            return q;
        };
        float bv[32];
        auto load_bias = [&](const float* pb, int c) {
            if (a.b5_q4) {  // channel-quad bias: 8 x 128-bit loads (n5 % 4 == 0)
                const float4* p4 = reinterpret_cast<const float4*>(pb) + (size_t)(8 * c) * bcs;
#pragma unroll
                for (int u = 0; u < 8; ++u) {
                    const float4 f = (32 * c + 4 * u < a.n5) ? __ldg(p4 + (size_t)u * bcs) : make_float4(0.f, 0.f, 0.f, 0.f);
                    bv[4 * u] = f.x;
                    bv[4 * u + 1] = f.y;
                    bv[4 * u + 2] = f.z;
                    bv[4 * u + 3] = f.w;
                }
                return;
            }
            const float* p = pb + (size_t)(32 * c) * bcs;
            if (c < NCH - 1) {
#pragma unroll
                for (int u = 0; u < 32; ++u, p += bcs) bv[u] = __ldg(p);
            } else {  // padding channels: accumulator 0, C6 weight 0
#pragma unroll
                for (int u = 0; u < 32; ++u, p += bcs) bv[u] = (32 * c + u < a.n5) ? __ldg(p) : 0.f;
            }
        };
        Pos cur = pos_of(blockIdx.x);
        if (blockIdx.x < nbands) load_bias(cur.pb, 0);
        int64_t k = 0;
        for (int64_t band = blockIdx.x; band < nbands; band += gridDim.x, ++k) {
            const int buf = (int)(k & 1);
            const bool has_next = band + gridDim.x < nbands;
            const float* nxt_pb = pos_of(has_next ? band + gridDim.x : band).pb;
            tc::mbar_wait(&S.t_full[buf], (uint32_t)((k >> 1) & 1));
            tc::fence_after_sync();
            float2 c6[5];  // C6 maps (2j, 2j+1) as pairs for FFMA2; map 9 is padding (weight 0)
#pragma unroll
            for (int o = 0; o < 5; ++o) c6[o] = make_float2(0.f, 0.f);
#pragma unroll
            for (int c = 0; c < NCH; ++c) {
                float v[32];
                const uint32_t col = (uint32_t)(buf * 256 + t * (kFuse ? 2 * NP : NP) + 32 * c);
                tc::tmem_ld32_async(tmem + lane_base + col, v);
                if (kFuse) {  // + the cross terms hi.lo + lo.hi, NP columns further
                    float x[32];
                    tc::tmem_ld32_async(tmem + lane_base + col + (uint32_t)NP, x);
                    tc::tmem_wait_ld();
#pragma unroll
                    for (int u = 0; u < 32; ++u) v[u] += x[u];
                } else {
                    tc::tmem_wait_ld();
                }
#pragma unroll
                for (int u = 0; u < 32; u += 2) {
                    const float2 x = __ffma2_rn(make_float2(v[u], v[u + 1]), make_float2(a.w_unscale, a.w_unscale),
                                                make_float2(bv[u], bv[u + 1]));
                    const float2 y = tanh_fp32x2(x);
                    v[u] = y.x;
                    v[u + 1] = y.y;
                }
                if (c + 1 < NCH)
                    load_bias(cur.pb, c + 1);
                else if (has_next)
                    load_bias(nxt_pb, 0);
#pragma unroll
                for (int u = 0; u < 32; ++u) {
                    const int ch = 32 * c + u;
#pragma unroll
                    for (int o = 0; o < 5; ++o)
                        c6[o] = __ffma2_rn(make_float2(k6w.k6[ch][2 * o], k6w.k6[ch][2 * o + 1]), make_float2(v[u], v[u]),
                                           c6[o]);
                }
            }
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
                    ob[o * a.out_plane_stride] = ((o & 1) ? c6[o >> 1].y : c6[o >> 1].x) + b;
                }
            }
            if (has_next) cur = pos_of(band + gridDim.x);
        }
    }
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<512>(tmem);
}

}  // namespace

// B operand of the 3xFP16 C3: [ks < 18][half][row < 96][8] fp16, K-step ks = window row y = ks / 3,
// taps j = 2 (ks % 3) + half (tap 5 = zero); column n < 48 as the bf16 C3 (cnn_prepare_k3_tc: n < 20
// = map n with filter row y, 24 <= n < 44 = map n - 24 with filter row y - 1, zero where the filter
// row is outside 0..4) holds the hi part, row 48 + n the lo part, of w * scale.
size_t cnn_k3_h3_bytes() { return (size_t)U2H_KS * 2 * 2 * U2H_N * 8 * 2; }
float cnn_h3_act_scale() { return kActScale; }
float cnn_h3_weight_scale(const float* w, size_t n) {
    float m = 0.f;
    for (size_t i = 0; i < n; ++i) m = std::max(m, std::fabs(w[i]));
    if (!(m > 0.f) || !std::isfinite(m)) return 1.f;
    int e = 0;
    std::frexp(m, &e);             // m = f 2^e, f in [0.5, 1)
    return std::ldexp(1.f, 14 - e);  // m x scale in [2^13, 2^14)
}

void cnn_prepare_k3_h3(const float* k3, float scale, uint16_t* dst) {
    std::memset(dst, 0, cnn_k3_h3_bytes());
    for (int ks = 0; ks < U2H_KS; ++ks) {
        const int y = ks / 3, j0 = 2 * (ks % 3);
        for (int h = 0; h < 2; ++h)
            for (int n = 0; n < U2H_N; ++n)
                for (int e = 0; e < 8; ++e) {
                    const int j = j0 + h;
                    const int t = n >= U2H_ROW1 ? 1 : 0, map = n - t * U2H_ROW1, i = y - t;
                    const bool ok = map < 20 && j < 5 && i >= 0 && i < 5;
                    const float w = ok ? k3[(map * 8 + e) * 25 + i * 5 + j] * scale : 0.f;
                    const uint16_t hi = to_f16(w);
                    dst[(((size_t)ks * 2 + h) * 2 * U2H_N + n) * 8 + e] = hi;
                    dst[(((size_t)ks * 2 + h) * 2 * U2H_N + U2H_N + n) * 8 + e] = to_f16(w - from_f16(hi));
                }
    }
}

// B operand of the 3xFP16 C5, 40 K-steps (stages of 4 are contiguous); K-step ks = 8 i + r8 of
// filter row i as the bf16 C5 (cnn_prepare_k5_tc); part 0 = hi, 1 = lo of w * 2^8. NP > 64:
// [ks][part][half][n < NP][8] fp16; NP <= 64 (the fused MMAs): [ks][half][part][n < NP][8], i.e.
// each K half is the 2 NP rows [B_hi | B_lo].
size_t cnn_k5_h3_bytes(int n5) { return (size_t)U3H_KS * 2 * 2 * cnn_n5_pad(n5) * 8 * 2; }
void cnn_prepare_k5_h3(const float* k5, int n5, float scale, uint16_t* dst) {
    const int NP = cnn_n5_pad(n5);
    std::memset(dst, 0, cnn_k5_h3_bytes(n5));
    for (int ks = 0; ks < U3H_KS; ++ks) {
        const int i = ks / 8, r8 = ks % 8;
        for (int h = 0; h < 2; ++h)
            for (int n = 0; n < n5; ++n)
                for (int e = 0; e < 8; ++e) {
                    int ci, j;
                    if (r8 < 5) {
                        ci = 8 * h + e;
                        j = r8;
                    } else {
                        ci = 16 + e;
                        j = 2 * (r8 - 5) + h;
                    }
                    const float w = (ci < 20 && j < 5) ? k5[((size_t)n * 20 + ci) * 25 + i * 5 + j] * scale : 0.f;
                    const uint16_t hi = to_f16(w), lo = to_f16(w - from_f16(hi));
                    if (NP <= 64) {
                        dst[(((size_t)(ks * 2 + h) * 2 + 0) * NP + n) * 8 + e] = hi;
                        dst[(((size_t)(ks * 2 + h) * 2 + 1) * NP + n) * 8 + e] = lo;
                    } else {
                        dst[(((size_t)(ks * 2 + 0) * 2 + h) * NP + n) * 8 + e] = hi;
                        dst[(((size_t)(ks * 2 + 1) * 2 + h) * NP + n) * 8 + e] = lo;
                    }
                }
    }
}

cudaError_t launch_cnn_u2_h3(const CnnU2Args& a, cudaStream_t s) {
    if (a.t4_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    if (!a.k3_h3) return cudaErrorInvalidValue;
    if (a.b3_plane && 20 * a.b3_rows * a.w3 >= (1ll << 32)) return cudaErrorInvalidValue;
    static std::atomic<uint32_t> flags{0};
    const size_t smem = sizeof(U2HSmem) + 128;
    if (!set_smem_attr_h3((const void*)cnn_u2_h3_kernel, smem, flags)) return cudaErrorInvalidValue;
    U2HP pw;
    std::memcpy(pw.p4, a.p4_host, sizeof pw.p4);
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t nseg = a.t4_rows * ((a.w3 + kTileM - 1) / kTileM) * a.nimg;
    if (nseg >= (1ll << 32)) return cudaErrorInvalidValue;  // 32-bit segment indexing in the kernel
    const unsigned grid = (unsigned)std::min<int64_t>(nseg, sms);
    cnn_u2_h3_kernel<<<grid, kThreadsU2H, smem, s>>>(a, pw, nseg);
    return cudaGetLastError();
}

cudaError_t launch_cnn_u3_h3(const CnnU3Args& a, cudaStream_t s) {
    if (a.out_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    if (a.n_pad > U3H_NMAX || a.n_pad % 16 || a.n5 > U3H_NMAX) return cudaErrorInvalidValue;
    if (a.b5_plane && (int64_t)a.n5 * a.b5_rows * a.w5 >= (1ll << 32)) return cudaErrorInvalidValue;
    const size_t smem = sizeof(U3HSmem) + 128;
    const int nch = (a.n_pad + 31) / 32;
    const void* fns[4] = {(const void*)cnn_u3_h3_kernel<1>, (const void*)cnn_u3_h3_kernel<2>,
                          (const void*)cnn_u3_h3_kernel<3>, (const void*)cnn_u3_h3_kernel<4>};
    static std::atomic<uint32_t> flag_n[4];
    if (!set_smem_attr_h3(fns[nch - 1], smem, flag_n[nch - 1])) return cudaErrorInvalidValue;
    const int64_t per_img = (a.out_rows * a.w4 + 2 * kTileM - 1) / (2 * kTileM);
    U3HK6 k6w{};
    for (int ch = 0; ch < a.n5; ++ch)
        for (int o = 0; o < 9; ++o) k6w.k6[ch][o] = a.k6_host[o * a.n5 + ch];
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t nbands = per_img * a.nimg;
    if (nbands >= (1ll << 32)) return cudaErrorInvalidValue;  // 32-bit band indexing in the kernel
    const unsigned grid = (unsigned)std::min<int64_t>(nbands, sms);
    switch (nch) {
        case 1: cnn_u3_h3_kernel<1><<<grid, kThreads, smem, s>>>(a, k6w, nbands); break;
        case 2: cnn_u3_h3_kernel<2><<<grid, kThreads, smem, s>>>(a, k6w, nbands); break;
        case 3: cnn_u3_h3_kernel<3><<<grid, kThreads, smem, s>>>(a, k6w, nbands); break;
        default: cnn_u3_h3_kernel<4><<<grid, kThreads, smem, s>>>(a, k6w, nbands); break;
    }
    return cudaGetLastError();
}

}  // namespace tg
