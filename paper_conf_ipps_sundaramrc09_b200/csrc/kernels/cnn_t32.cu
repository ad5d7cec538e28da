// cnn_t32.cu -- U3 (C5 T C6) of the CNN with fp32 accuracy on the tcgen05 tensor cores
// (precision TG_FP32_TC, sm_100a).
//
// C5 (20 x 25 -> n5) is a dense contraction. TF32 alone (10-bit
// mantissa) misses the fp32 parity bound (1e-5 normwise, R16) by two orders of
// magnitude, so every operand is split into two TF32 numbers, x = big + small with
// big = tf32_rn(x), small = tf32_rn(x - big) (|x - big - small| <= 2^-22 |x|), and the product is
// accumulated from three TF32 MMAs, big.big + big.small + small.big, in fp32 (the dropped
// small.small term is < 2^-21 of the product). Error on a 500-term C5 dot product: ~5e-7
// normwise, the same as an fp32 FMA chain.
//
// Implicit GEMM as in the bf16 U3 (cnn_tc.cu): band = 256 consecutive output positions in the
// flat (row, col) index with pitch w4; filter row i reads the contiguous slice [q0 + i*w4, +262)
// of T4. T4 comes from U2 in TF32-split, pixel-blocked form [part][block][rows][w4][4 ch]
// (part 0 = big, 1 = small; 5 blocks of 4 channels; one pixel's 4 channels = one 16-byte core
// matrix row). A K=8 step is two 4-channel halves: blocks (0,1) or (2,3) of one tap (LBO = one
// block plane), or block 4 of taps (j, j+1) (LBO = 16 B: the next pixel) -- 13 K-steps per filter
// row, 65 per tile (K = 520, 500 useful).
// B (65 K-steps x 2 parts x NP maps x 8 tf32 = up to 532 KB) streams through a ring of stages
// of 4 K-steps (32 KB bulk copies); slices through a ring of 2 buffers (10 bulk copies each).
// Warp-specialised and persistent (one CTA per SM, 10 warps):
//   warp 9   copy producer (slices and B stages, in consumption order)
//   warp 8   MMA issuer (elect.sync): per K-step 3 MMAs x 2 tiles into one of two TMEM
//            accumulators (2 tiles x NP columns)
//   0-7      epilogue: TMEM -> registers, + bias plane, tanh (fp32 formula), the 1x1 C6 as
//            fp32 FMAs over n5 (weights in the constant bank), + C6 bias -> output
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstring>
#include <vector>

#include "kernels.h"
#include "tc_sm100.cuh"

namespace tg {
namespace {

// tanh = 1 - 2/(1+e^{2x}) with MUFU ex2/rcp (|x| clamped to 15): absolute error < 3e-7 (the
// fp32 path's formula, cnn_fp32.cu)
__device__ __forceinline__ float tanh_acc(float x) {
    x = fminf(fmaxf(x, -15.f), 15.f);
    const float e = __expf(2.f * x);
    return 1.f - __fdividef(2.f, 1.f + e);
}

// round to TF32 (10-bit mantissa; nearest, ties away): the "big" part of a 3xTF32 split (the
// same rounding as U1 and the FFMA U2 in cnn_fp32.cu)
__device__ __forceinline__ float tf32_rn_dev(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return __uint_as_float(r);
}

constexpr int kTileM = 128;
constexpr int T3_KS = 65;                        // K-steps (K = 8) per tile
constexpr int T3_KST = 4;                        // K-steps per B stage
constexpr int T3_NST = (T3_KS + T3_KST - 1) / T3_KST;  // 17 stages per band (B padded to 68 K-steps)
constexpr int T3_BRING = 3;                      // B stage buffers
constexpr int T3_NMAX = 128;
constexpr int T3_SPX = 2 * kTileM + 8;           // pixels per slice block (262 used)
constexpr int T3_NA = 2;                         // slice buffers
constexpr int kEpiWarps = 8;
constexpr int kThreads = (kEpiWarps + 2) * 32;

struct T3K6 {
    float k6[T3_NMAX][12];  // [ch][o] (9 used): C6 weights, broadcast from the constant bank
};

struct T3Smem {
    uint4 b[T3_BRING][T3_KST * 2 * 2 * T3_NMAX];  // [stage][u][part][half][n] -> 4 tf32
    uint4 a[T3_NA][2][5][T3_SPX];                 // [slot][part][block][pixel] -> 4 tf32
    uint64_t a_full[T3_NA], a_empty[T3_NA], b_full[T3_BRING], b_empty[T3_BRING], t_full[2], t_empty[2];
    uint32_t tmem;
};

// instruction descriptor, kind::tf32: D F32, A and B TF32 (format 2), both K-major
__host__ __device__ constexpr uint32_t idesc_tf32(int M, int N) {
    return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void mma_tf32(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                         uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(d_tmem),
        "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate));
}

template <int NCH>  // TMEM chunks of 32 columns: NP = n5 padded to 16, NCH = ceil(NP / 32)
__global__ void __launch_bounds__(kThreads, 1)
    cnn_u3_t32_kernel(const CnnU3Args a, const __grid_constant__ T3K6 k6w, const int64_t nbands) {
    extern __shared__ __align__(128) uint8_t smraw[];
    T3Smem& S = *reinterpret_cast<T3Smem*>(smraw + ((128 - (tc::smem_u32(smraw) & 127)) & 127));
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int NP = a.n_pad;
    const int64_t per_img = (a.out_rows * a.w4 + 2 * kTileM - 1) / (2 * kTileM);
    const int64_t bplane = a.t4_rows * a.w4;                 // pixels per block plane of one image
    const int64_t flat0 = (a.out_row0 - a.t4_row0) * a.w4;  // flat index of output row 0 in the T4 buffer

    if (warp == 0) tc::tmem_alloc<512>(&S.tmem);
    if (tid == 0) {
        for (int i = 0; i < T3_NA; ++i) {
            tc::mbar_init(&S.a_full[i], 1);
            tc::mbar_init(&S.a_empty[i], 1);
        }
        for (int i = 0; i < T3_BRING; ++i) {
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
    for (int idx = tid; idx < T3_NA * 2 * 5 * T3_SPX; idx += kThreads) (&S.a[0][0][0][0])[idx] = make_uint4(0u, 0u, 0u, 0u);
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
        const uint32_t stage_bytes = (uint32_t)(T3_KST * 2 * 2 * NP * 16);
        int64_t si = 0, gi = 0;  // slices and B stages issued so far
        for (int64_t k = 0; k < my_bands; ++k) {
            const int64_t band = blockIdx.x + k * gridDim.x;
            const int64_t img = band / per_img;
            const int64_t q0 = (band - img * per_img) * 2 * kTileM;
            for (int ks = 0; ks < T3_KS; ++ks) {
                if (ks % 13 == 0) {  // slice i = ks / 13
                    const int slot = (int)(si % T3_NA);
                    if (si >= T3_NA) tc::mbar_wait(&S.a_empty[slot], (uint32_t)(((si - T3_NA) / T3_NA) & 1));
                    const int64_t e = flat0 + q0 + (int64_t)(ks / 13) * a.w4;
                    const int64_t n = max((int64_t)0, min((int64_t)T3_SPX, bplane - e));
                    if (tc::elect_one()) {
                        tc::mbar_expect_tx(&S.a_full[slot], (uint32_t)(10 * n * 16));
                        if (n > 0) {
                            for (int part = 0; part < 2; ++part)
                                for (int blk = 0; blk < 5; ++blk)
                                    tc::bulk_g2s(S.a[slot][part][blk], t4all + ((img * 2 + part) * 5 + blk) * bplane + e,
                                                 (uint32_t)(n * 16), &S.a_full[slot]);
                        }
                    }
                    __syncwarp();
                    ++si;
                }
                if (ks % T3_KST == 0) {  // B stage ks / 4
                    const int slot = (int)(gi % T3_BRING);
                    if (gi >= T3_BRING) tc::mbar_wait(&S.b_empty[slot], (uint32_t)(((gi - T3_BRING) / T3_BRING) & 1));
                    if (tc::elect_one()) {
                        tc::mbar_expect_tx(&S.b_full[slot], stage_bytes);
                        tc::bulk_g2s(S.b[slot], kb + (size_t)(ks / T3_KST) * stage_bytes, stage_bytes, &S.b_full[slot]);
                    }
                    __syncwarp();
                    ++gi;
                }
            }
        }
    } else if (warp == kEpiWarps) {
        // ---------------------------------------------------------------- MMA issuer
        const uint32_t idesc = idesc_tf32(kTileM, NP);
        const uint32_t plane_bytes = (uint32_t)(T3_SPX * 16), part_bytes = 5 * plane_bytes;
        int64_t si = 0, gi = 0;
        for (int64_t k = 0; k < my_bands; ++k) {
            const int buf = (int)(k & 1);
            if (k >= 2) tc::mbar_wait(&S.t_empty[buf], (uint32_t)(((k - 2) >> 1) & 1));
            const uint32_t d_base = tmem + (uint32_t)(buf * 256);
            uint32_t a_base = 0, b_base = 0;
            int aslot = 0, bslot = 0;
            for (int ks = 0; ks < T3_KS; ++ks) {
                if (ks % 13 == 0) {
                    aslot = (int)(si % T3_NA);
                    tc::mbar_wait(&S.a_full[aslot], (uint32_t)((si / T3_NA) & 1));
                    a_base = tc::smem_u32(S.a[aslot][0][0]);
                    ++si;
                }
                if (ks % T3_KST == 0) {
                    bslot = (int)(gi % T3_BRING);
                    tc::mbar_wait(&S.b_full[bslot], (uint32_t)((gi / T3_BRING) & 1));
                    b_base = tc::smem_u32(S.b[bslot]);
                    ++gi;
                }
                tc::fence_after_sync();
                const int s = ks % 13, u = ks % T3_KST;
                // s < 10: blocks (2p, 2p+1) of tap (i, s/2); s >= 10: block 4 of taps (i, j), (i, j+1)
                const uint32_t a_off = s < 10 ? (uint32_t)(2 * (s & 1)) * plane_bytes + (uint32_t)((s >> 1) * 16)
                                              : 4 * plane_bytes + (uint32_t)(2 * (s - 10) * 16);
                const uint32_t lbo = s < 10 ? plane_bytes : 16u;
                if (tc::elect_one()) {
#pragma unroll
                    for (int t = 0; t < 2; ++t) {
                        const uint32_t ab = a_base + a_off + (uint32_t)(t * kTileM * 16);
                        const uint64_t a_big = tc::make_desc(ab, lbo, 128);
                        const uint64_t a_small = tc::make_desc(ab + part_bytes, lbo, 128);
                        const uint32_t bb = b_base + (uint32_t)(u * 2 * 2 * NP * 16);
                        const uint64_t b_big = tc::make_desc(bb, (uint32_t)(NP * 16), 128);
                        const uint64_t b_small = tc::make_desc(bb + (uint32_t)(2 * NP * 16), (uint32_t)(NP * 16), 128);
                        const uint32_t d = d_base + (uint32_t)(t * NP);
                        mma_tf32(d, a_big, b_big, idesc, ks > 0 ? 1u : 0u);
                        mma_tf32(d, a_big, b_small, idesc, 1u);
                        mma_tf32(d, a_small, b_big, idesc, 1u);
#ifdef T32_FOUR
                        mma_tf32(d, a_small, b_small, idesc, 1u);
#endif
                    }
                    if (u == T3_KST - 1 || ks == T3_KS - 1) tc::commit(&S.b_empty[bslot]);
                    if (s == 12) tc::commit(&S.a_empty[aslot]);
                    if (ks == T3_KS - 1) tc::commit(&S.t_full[buf]);
                }
                __syncwarp();
            }
        }
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
            const int64_t img = band / per_img;
            const int qq = (int)(band - img * per_img) * 2 * kTileM + m;
            q.img = (int)img;
            const int r = qq / w4;
            q.orow = (int)a.out_row0 + r;
            q.ocol = qq - r * w4;
            q.ok = q.orow < orow_end && q.ocol < w5;
            const int orow_c = min(q.orow, orow_end - 1), ocol_c = min(q.ocol, w5 - 1);
            q.pb = a.b5_plane ? a.b5 + ((int64_t)(orow_c - a.b5_row0) * w5 + ocol_c) : a.b5;
            return q;
        };
        float bv[32];
        auto load_bias = [&](const float* pb, int c) {
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
            float c6[9];
#pragma unroll
            for (int o = 0; o < 9; ++o) c6[o] = 0.f;
#pragma unroll
            for (int c = 0; c < NCH; ++c) {
                float v[32];
                tc::tmem_ld32_async(tmem + lane_base + (uint32_t)(buf * 256 + t * NP + 32 * c), v);
                tc::tmem_wait_ld();
#pragma unroll
                for (int u = 0; u < 32; ++u) v[u] = tanh_acc(v[u] + bv[u]);
                if (c + 1 < NCH)
                    load_bias(cur.pb, c + 1);
                else if (has_next)
                    load_bias(nxt_pb, 0);
#pragma unroll
                for (int u = 0; u < 32; ++u) {
                    const int ch = 32 * c + u;
#pragma unroll
                    for (int o = 0; o < 9; ++o) c6[o] = fmaf(k6w.k6[ch][o], v[u], c6[o]);
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
                    ob[o * a.out_plane_stride] = c6[o] + b;
                }
            }
            if (has_next) cur = pos_of(band + gridDim.x);
        }
    }
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<512>(tmem);
}

// ============================================================================ U2 (C3, 3xTF32)
// C3 (8 x 25 -> 20) with fp32 accuracy: the bf16 U2's implicit GEMM (cnn_tc.cu) with TF32-split
// operands. Segment = T4 row R (C3 rows 2R, 2R+1) x 128 C3 columns: tile t = C3 row 2R + t
// (M = 128), one K = 8 step per tap (the pixel's 8 channels: block 0 = channels 0-3, block 1 =
// 4-7, LBO = one block plane of the window). With N = 20 maps (padded to 32) an MMA is bound by
// reading its A operand from shared memory (4 KB per 128 x 8 tf32 slice), so the big part of
// A is read ONCE for both of its products: per tap and tile
//   MMA 1  A_big   x [B_big | B_small]  (N = 64)  -> columns [0, 32) big.big, [32, 64) big.small
//   MMA 2  A_small x  B_big             (N = 32)  -> accumulates onto columns [32, 64)
// and the epilogue adds the two halves (2 A reads per tap instead of 3). Window: T2 rows
// [2R, 2R+6) x cols [c0, c0+134) of both parts and both blocks, [part][block][row][col] -> 4 tf32.
// Warp-specialised and persistent (one CTA per SM, 10 warps), as the bf16 U2:
//   warp 9   copy producer: the B operand once per CTA, per segment 24 row copies
//   warp 8   MMA issuer: 2 tiles x 25 K-steps x 2 MMAs into one of 4 TMEM slots (128 columns)
//   0-3/4-7  epilogue groups (even / odd segments): bias plane, tanh (fp32 formula), the 2x2
//            subsample (rows in the thread, columns across lanes), tanh -> T4 TF32-split
//            [part][block][rows][w4][4] for the 3xTF32 U3 above
constexpr int U2T_WR = 6, U2T_WP = kTileM + 6;
constexpr int U2T_N = 32;                      // 20 maps padded; B rows per K half = 2 x U2T_N
constexpr int U2T_KS = 25;
constexpr int U2T_NA = 3;
constexpr int U2T_NT = 4;
constexpr int U2T_PLANE = U2T_WR * U2T_WP;     // pixels per block plane of one window

struct U2TP {
    float p4[20][4];  // S4 weights (constant bank)
};

struct U2TSmem {
    uint4 a[U2T_NA][2][2][U2T_PLANE];          // [buf][part][block][row*WP + col] -> 4 tf32
    uint4 b[U2T_KS * 2 * 2 * U2T_N];           // [ks][half][row < 64: big maps, then small] -> 4 tf32
    uint64_t b_full, a_full[U2T_NA], a_empty[U2T_NA], t_full[U2T_NT], t_empty[U2T_NT];
    uint32_t tmem;
};

__global__ void __launch_bounds__(kThreads, 1)
    cnn_u2_t32_kernel(const CnnU2Args a, const __grid_constant__ U2TP pw, const int64_t nseg) {
    extern __shared__ __align__(128) uint8_t smraw[];
    U2TSmem& S = *reinterpret_cast<U2TSmem*>(smraw + ((128 - (tc::smem_u32(smraw) & 127)) & 127));
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

    if (warp == 0) tc::tmem_alloc<512>(&S.tmem);
    if (tid == 0) {
        tc::mbar_init(&S.b_full, 1);
        for (int i = 0; i < U2T_NA; ++i) {
            tc::mbar_init(&S.a_full[i], 1);
            tc::mbar_init(&S.a_empty[i], 1);
        }
        for (int i = 0; i < U2T_NT; ++i) {
            tc::mbar_init(&S.t_full[i], 1);
            tc::mbar_init(&S.t_empty[i], 4);
        }
        tc::mbar_fence_init();
    }
    // windows start zeroed: pixels a copy does not cover (beyond the image) only ever hold
    // finite T2 values; they feed C3 columns that are not stored
    for (int idx = tid; idx < U2T_NA * 4 * U2T_PLANE; idx += kThreads) (&S.a[0][0][0][0])[idx] = make_uint4(0u, 0u, 0u, 0u);
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    const uint32_t tmem = S.tmem;
    const int64_t my = nseg > blockIdx.x ? (nseg - 1 - blockIdx.x) / gridDim.x + 1 : 0;

    if (warp == kEpiWarps + 1) {
        // ---------------------------------------------------------------- copy producer
        const uint4* t2all = reinterpret_cast<const uint4*>(a.t2);
        const int64_t tplane = a.t2_rows * a.w2;  // pixels per block plane of one image's T2
        const uint32_t bbytes = (uint32_t)(U2T_KS * 2 * 2 * U2T_N * 16);
        if (tc::elect_one()) {
            tc::mbar_expect_tx(&S.b_full, bbytes);
            tc::bulk_g2s(S.b, a.k3_t32, bbytes, &S.b_full);
        }
        __syncwarp();
        for (int64_t k = 0; k < my; ++k) {
            const int buf = (int)(k % U2T_NA);
            if (k >= U2T_NA) tc::mbar_wait(&S.a_empty[buf], (uint32_t)(((k - U2T_NA) / U2T_NA) & 1));
            int64_t img, R, c0;
            seg_coords(blockIdx.x + k * gridDim.x, img, R, c0);
            const int64_t r0 = 2 * R - a.t2_row0;
            const int64_t rows = min((int64_t)U2T_WR, a.t2_rows - r0);
            const int64_t cols = min((int64_t)U2T_WP, a.w2 - c0);
            // the 4 planes x `rows` window rows are issued by as many lanes in ONE warp
            // instruction (a single thread would serialise ~150 cycles per bulk copy)
            if (lane == 0) tc::mbar_expect_tx(&S.a_full[buf], (uint32_t)(4 * rows * cols * 16));
            __syncwarp();
            if (lane < 4 * rows) {
                const int pb = lane / (int)rows, r = lane - pb * (int)rows;  // plane = part * 2 + block
                const uint4* src = t2all + (img * 4 + pb) * tplane + (r0 + r) * a.w2 + c0;
                tc::bulk_g2s(&S.a[buf][pb >> 1][pb & 1][r * U2T_WP], src, (uint32_t)(cols * 16), &S.a_full[buf]);
            }
            __syncwarp();
        }
    } else if (warp == kEpiWarps) {
        // ---------------------------------------------------------------- MMA issuer
        tc::mbar_wait(&S.b_full, 0);
        const uint32_t idesc64 = idesc_tf32(kTileM, 2 * U2T_N), idesc32 = idesc_tf32(kTileM, U2T_N);
        const uint32_t blk_bytes = (uint32_t)(U2T_PLANE * 16);
        const uint64_t a_desc0 = tc::make_desc(tc::smem_u32(S.a[0][0][0]), blk_bytes, 128);  // K half 2 = block 1
        const uint64_t b_desc0 = tc::make_desc(tc::smem_u32(S.b), 2 * U2T_N * 16, 128);
        for (int64_t k = 0; k < my; ++k) {
            const int buf = (int)(k % U2T_NA), ts = (int)(k % U2T_NT);
            tc::mbar_wait(&S.a_full[buf], (uint32_t)((k / U2T_NA) & 1));
            if (k >= U2T_NT) tc::mbar_wait(&S.t_empty[ts], (uint32_t)(((k - U2T_NT) / U2T_NT) & 1));
            tc::fence_after_sync();
            // descriptors: the start address is the low 14 bits (16-byte units), advanced by adding
            const uint64_t abuf = a_desc0 + (uint64_t)(buf * (4 * U2T_PLANE));
            const uint32_t d0 = tmem + (uint32_t)(ts * 4 * U2T_N);
            if (tc::elect_one()) {
#pragma unroll
                for (int t = 0; t < 2; ++t) {  // tile t = C3 row 2R + t
#pragma unroll
                    for (int ks = 0; ks < U2T_KS; ++ks) {
                        const int i = ks / 5, j = ks % 5;
                        const uint64_t a_big = abuf + (uint64_t)((t + i) * U2T_WP + j);
                        const uint64_t a_small = a_big + (uint64_t)(2 * U2T_PLANE);
                        const uint64_t b_ks = b_desc0 + (uint64_t)(ks * 2 * 2 * U2T_N);  // rows 0..31 = B_big
                        const uint32_t d = d0 + (uint32_t)(t * 2 * U2T_N);
                        mma_tf32(d, a_big, b_ks, idesc64, ks > 0 ? 1u : 0u);
                        mma_tf32(d + U2T_N, a_small, b_ks, idesc32, 1u);
                    }
                }
                tc::commit(&S.a_empty[buf]);
                tc::commit(&S.t_full[ts]);
            }
            __syncwarp();
        }
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
        for (int64_t k = grp; k < my; k += 2) {
            const int ts = (int)(k % U2T_NT);
            int64_t img, R, c0;
            seg_coords(blockIdx.x + k * gridDim.x, img, R, c0);
            const int64_t c = c0 + 32 * wq + lane;  // C3 column
            const int64_t C = c >> 1;               // T4 column
            tc::mbar_wait(&S.t_full[ts], (uint32_t)((k / U2T_NT) & 1));
            tc::fence_after_sync();
            float v0[32], v1[32];
            {
                float x0[32], x1[32];
                const uint32_t tb = tmem + lane_base + (uint32_t)(ts * 4 * U2T_N);
                tc::tmem_ld32_async(tb, v0);                     // tile 0: big.big
                tc::tmem_ld32_async(tb + U2T_N, x0);             //         big.small + small.big
                tc::tmem_ld32_async(tb + 2 * U2T_N, v1);         // tile 1
                tc::tmem_ld32_async(tb + 3 * U2T_N, x1);
                tc::tmem_wait_ld();
#pragma unroll
                for (int co = 0; co < 20; ++co) {
                    v0[co] += x0[co];
                    v1[co] += x1[co];
                }
            }
            tc::fence_before_sync();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&S.t_empty[ts]);
            const bool out_ok = !(lane & 1) && C < a.w4;
            float tv[20];
#pragma unroll
            for (int co = 0; co < 20; ++co) {
                const float t0 = tanh_acc(v0[co] + b0v[co]);
                const float t1 = tanh_acc(v1[co] + b1v[co]);
                const float t01 = __shfl_down_sync(0xffffffffu, t0, 1);  // column c+1
                const float t11 = __shfl_down_sync(0xffffffffu, t1, 1);
                float s4 = 0.f;
                s4 = fmaf(pw.p4[co][0], t0, s4);
                s4 = fmaf(pw.p4[co][1], t01, s4);
                s4 = fmaf(pw.p4[co][2], t1, s4);
                s4 = fmaf(pw.p4[co][3], t11, s4);
                tv[co] = tanh_acc(s4);
            }
            if (k + 2 < my) load_bias(k + 2);
            if (out_ok) {
                float4* t4 = reinterpret_cast<float4*>(a.t4) + img * 10 * bplane + (R - a.t4_row0) * a.w4 + C;
#pragma unroll
                for (int blk = 0; blk < 5; ++blk) {
                    float big[4], small[4];
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        big[e] = tf32_rn_dev(tv[4 * blk + e]);
                        small[e] = tf32_rn_dev(tv[4 * blk + e] - big[e]);
                    }
                    t4[blk * bplane] = make_float4(big[0], big[1], big[2], big[3]);
                    t4[(5 + blk) * bplane] = make_float4(small[0], small[1], small[2], small[3]);
                }
            }
        }
    }
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<512>(tmem);
}

// round to TF32 (10-bit mantissa), nearest even, on the host
float to_tf32(float f) {
    uint32_t u;
    std::memcpy(&u, &f, 4);
    if ((u & 0x7f800000u) == 0x7f800000u) return f;
    u += 0xfffu + ((u >> 13) & 1u);
    u &= 0xffffe000u;
    float r;
    std::memcpy(&r, &u, 4);
    return r;
}

bool set_smem_attr_t32(const void* fn, size_t bytes, std::atomic<uint32_t>& flags) {
    int dev = 0;
    cudaGetDevice(&dev);
    const uint32_t bit = 1u << (dev & 31);
    if (flags.load() & bit) return true;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) != cudaSuccess) return false;
    flags.fetch_or(bit);
    return true;
}

}  // namespace

// B operand of the 3xTF32 C5: [ks < 68][part][half][n < NP][4] fp32 (stages of 4 K-steps are
// contiguous; K-steps 65..67 are zero). K-step ks = 13 i + s of filter row i: s < 10 -> tap
// (i, s/2), half h = channels 4 (2 (s%2) + h) .. +3; s >= 10 -> channels 16..19 of tap
// (i, 2 (s-10) + h) (zero for tap 5). part 0 = tf32_rn(w), part 1 = tf32_rn(w - part 0).
size_t cnn_k5_t32_bytes(int n5) { return (size_t)T3_NST * T3_KST * 2 * 2 * cnn_n5_pad(n5) * 4 * 4; }
void cnn_prepare_k5_t32(const float* k5, int n5, float* dst) {
    const int NP = cnn_n5_pad(n5);
    std::memset(dst, 0, cnn_k5_t32_bytes(n5));
    for (int ks = 0; ks < T3_KS; ++ks) {
        const int i = ks / 13, s = ks % 13;
        for (int h = 0; h < 2; ++h)
            for (int n = 0; n < n5; ++n)
                for (int e = 0; e < 4; ++e) {
                    int ci, j;
                    if (s < 10) {
                        ci = 4 * (2 * (s % 2) + h) + e;
                        j = s / 2;
                    } else {
                        ci = 16 + e;
                        j = 2 * (s - 10) + h;
                    }
                    const float w = j < 5 ? k5[((size_t)n * 20 + ci) * 25 + i * 5 + j] : 0.f;
                    const float big = to_tf32(w), small = to_tf32(w - big);
                    dst[(((size_t)(ks * 2 + 0) * 2 + h) * NP + n) * 4 + e] = big;
                    dst[(((size_t)(ks * 2 + 1) * 2 + h) * NP + n) * 4 + e] = small;
                }
    }
}

// B operand of the 3xTF32 C3: [ks < 25][half][row < 64][4] fp32, K-step ks = tap (i, j) =
// (ks / 5, ks % 5), half h = channels 4h..4h+3; row n < 32: big part tf32_rn(w) of map n,
// row 32 + n: small part tf32_rn(w - big) of map n, w = K3[n][4h + e][i][j]; maps 20..31 zero.
size_t cnn_k3_t32_bytes() { return (size_t)U2T_KS * 2 * 2 * U2T_N * 4 * 4; }
void cnn_prepare_k3_t32(const float* k3, float* dst) {
    std::memset(dst, 0, cnn_k3_t32_bytes());
    for (int ks = 0; ks < U2T_KS; ++ks)
        for (int h = 0; h < 2; ++h)
            for (int n = 0; n < 20; ++n)
                for (int e = 0; e < 4; ++e) {
                    const float w = k3[((size_t)n * 8 + 4 * h + e) * 25 + ks];
                    const float big = to_tf32(w), small = to_tf32(w - big);
                    dst[(((size_t)ks * 2 + h) * 2 * U2T_N + n) * 4 + e] = big;
                    dst[(((size_t)ks * 2 + h) * 2 * U2T_N + U2T_N + n) * 4 + e] = small;
                }
}

cudaError_t launch_cnn_u2_t32(const CnnU2Args& a, cudaStream_t s) {
    if (a.t4_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    if (!a.k3_t32) return cudaErrorInvalidValue;
    if (a.b3_plane && 20 * a.b3_rows * a.w3 >= (1ll << 32)) return cudaErrorInvalidValue;
    static std::atomic<uint32_t> flags{0};
    const size_t smem = sizeof(U2TSmem) + 128;
    if (!set_smem_attr_t32((const void*)cnn_u2_t32_kernel, smem, flags)) return cudaErrorInvalidValue;
    U2TP pw;
    std::memcpy(pw.p4, a.p4_host, sizeof pw.p4);
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t nseg = a.t4_rows * ((a.w3 + kTileM - 1) / kTileM) * a.nimg;
    const unsigned grid = (unsigned)std::min<int64_t>(nseg, sms);
    cnn_u2_t32_kernel<<<grid, kThreads, smem, s>>>(a, pw, nseg);
    return cudaGetLastError();
}

cudaError_t launch_cnn_u3_t32(const CnnU3Args& a, cudaStream_t s) {
    if (a.out_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    if (a.n_pad > T3_NMAX || a.n_pad % 16 || a.n5 > T3_NMAX) return cudaErrorInvalidValue;
    if (a.b5_plane && (int64_t)a.n5 * a.b5_rows * a.w5 >= (1ll << 32)) return cudaErrorInvalidValue;
    const size_t smem = sizeof(T3Smem) + 128;
    const int nch = (a.n_pad + 31) / 32;
    const void* fns[4] = {(const void*)cnn_u3_t32_kernel<1>, (const void*)cnn_u3_t32_kernel<2>,
                          (const void*)cnn_u3_t32_kernel<3>, (const void*)cnn_u3_t32_kernel<4>};
    static std::atomic<uint32_t> flag_n[4];
    if (!set_smem_attr_t32(fns[nch - 1], smem, flag_n[nch - 1])) return cudaErrorInvalidValue;
    const int64_t per_img = (a.out_rows * a.w4 + 2 * kTileM - 1) / (2 * kTileM);
    T3K6 k6w{};
    for (int ch = 0; ch < a.n5; ++ch)
        for (int o = 0; o < 9; ++o) k6w.k6[ch][o] = a.k6_host[o * a.n5 + ch];
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t nbands = per_img * a.nimg;
    const unsigned grid = (unsigned)std::min<int64_t>(nbands, sms);
    switch (nch) {
        case 1: cnn_u3_t32_kernel<1><<<grid, kThreads, smem, s>>>(a, k6w, nbands); break;
        case 2: cnn_u3_t32_kernel<2><<<grid, kThreads, smem, s>>>(a, k6w, nbands); break;
        case 3: cnn_u3_t32_kernel<3><<<grid, kThreads, smem, s>>>(a, k6w, nbands); break;
        default: cnn_u3_t32_kernel<4><<<grid, kThreads, smem, s>>>(a, k6w, nbands); break;
    }
    return cudaGetLastError();
}

}  // namespace tg
