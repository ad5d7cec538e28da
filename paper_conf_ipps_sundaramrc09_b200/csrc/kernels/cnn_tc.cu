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
// Epilogues run on all 4 warps from TMEM (tcgen05.ld 32x32b): bias plane + tanh, then
//   U2: the 2x2 subsample pairs row 2R (tile 0) with row 2R+1 (tile 1) in the same thread and
//       columns c, c+1 across neighbouring lanes (shfl), + tanh -> T4 (fp32);
//   U3: the 1x1 C6 layer as a dot product over n5 in registers, + bias -> output (fp32).
// Precision: bf16 operands, fp32 accumulation; parity bound 2e-2 normwise (R16).
#include <cuda_runtime.h>

#include <atomic>
#include <cstring>
#include <vector>

#include "kernels.h"
#include "tc_sm100.cuh"

namespace tg {
namespace {

__device__ __forceinline__ float tanh_f(float x) {
    x = fminf(fmaxf(x, -15.f), 15.f);
    const float e = __expf(2.f * x);
    return 1.f - __fdividef(2.f, 1.f + e);
}

constexpr int kThreads = 128;
constexpr int kTileM = 128;

// ============================================================================ U2 (C3)
// Band = C3 rows (2R, 2R+1) x 128 columns [c0, c0+128): tile 0 = row 2R, tile 1 = row 2R+1.
// Window: T2 rows [2R, 2R+6) x cols [c0, c0 + 134), 8 channels per pixel (one plane).
constexpr int U2_WR = 6, U2_WP = kTileM + 6;  // +4 taps, +1 for the (4,5) tap pair, +1 spare
constexpr int U2_N = 32;                      // 20 maps padded to 32
constexpr int U2_KS = 15;                     // 5 rows x pairs (0,1) (2,3) (4,5)

struct U2TcShared {
    uint4 a[U2_WR * U2_WP];            // [row][col] -> 8 bf16 channels
    uint4 b[U2_KS * 2 * U2_N];         // [ks][half][n] -> 8 bf16
    float p4[20][4];
    uint64_t mbar;
    uint32_t tmem;
};

__global__ void __launch_bounds__(kThreads) cnn_u2_tc_kernel(const CnnU2Args a) {
    extern __shared__ __align__(128) uint8_t smraw[];
    U2TcShared& S = *reinterpret_cast<U2TcShared*>(smraw);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int bands_per_row = (int)((a.w3 + kTileM - 1) / kTileM);
    const int64_t img = blockIdx.z;
    const int64_t R = a.t4_row0 + blockIdx.y;      // T4 row (global)
    const int64_t c0 = (int64_t)blockIdx.x * kTileM;  // C3 column of position 0
    (void)bands_per_row;

    if (warp == 0) tc::tmem_alloc<64>(&S.tmem);
    if (tid == 0) {
        tc::mbar_init(&S.mbar, 1);
        tc::mbar_fence_init();
    }
    // stage the T2 window: U1 wrote T2 as bf16 pixels [row][col][8 ch] = one 16-byte load each
    const uint4* t2b = reinterpret_cast<const uint4*>(a.t2) + img * a.t2_rows * a.w2;
    for (int idx = tid; idx < U2_WR * U2_WP; idx += kThreads) {
        const int r = idx / U2_WP, c = idx - r * U2_WP;
        const int64_t br = 2 * R + r - a.t2_row0, gc = c0 + c;
        const bool ok = br >= 0 && br < a.t2_rows && gc < a.w2;
        S.a[idx] = ok ? __ldg(t2b + br * a.w2 + gc) : make_uint4(0u, 0u, 0u, 0u);
    }
    const uint4* kb = reinterpret_cast<const uint4*>(a.k3_tc);
    for (int idx = tid; idx < U2_KS * 2 * U2_N; idx += kThreads) S.b[idx] = __ldg(kb + idx);
    for (int idx = tid; idx < 80; idx += kThreads) S.p4[idx / 4][idx % 4] = __ldg(a.p4_dev + idx);
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    const uint32_t tmem = S.tmem;

    if (tid == 0) {
        const uint32_t idesc = tc::make_idesc_bf16(kTileM, U2_N);
        const uint32_t a0 = tc::smem_u32(S.a), b0 = tc::smem_u32(S.b);
        for (int t = 0; t < 2; ++t) {       // tile t = C3 row 2R + t
            for (int ks = 0; ks < U2_KS; ++ks) {
                const int i = ks / 3, j = 2 * (ks % 3);
                const uint32_t a_addr = a0 + (uint32_t)(((t + i) * U2_WP + j) * 16);
                const uint64_t ad = tc::make_desc(a_addr, 16, 128);  // 2nd K-half = next pixel (tap j+1)
                const uint64_t bd = tc::make_desc(b0 + (uint32_t)(ks * 2 * U2_N * 16), U2_N * 16, 128);
                tc::mma_bf16(tmem + (uint32_t)(t * U2_N), ad, bd, idesc, ks > 0 ? 1u : 0u);
            }
        }
        tc::commit(&S.mbar);
    }
    tc::mbar_wait(&S.mbar, 0);
    tc::fence_after_sync();

    // epilogue: thread = C3 column c0 + 32*warp + lane, rows 2R (tile 0) and 2R+1 (tile 1)
    float v0[32], v1[32];
    const uint32_t lane_base = (uint32_t)(32 * warp) << 16;
    tc::tmem_ld32(tmem + lane_base + 0, v0);
    tc::tmem_ld32(tmem + lane_base + U2_N, v1);
    const int64_t c = c0 + 32 * warp + lane;  // C3 column
    const int64_t C = c >> 1;                 // T4 column
    const bool row_ok = R < a.t4_row0 + a.t4_rows;
    const bool col_ok = c < a.w3;
    float tv[20];
#pragma unroll
    for (int co = 0; co < 20; ++co) {
        float t0 = 0.f, t1 = 0.f;
        if (row_ok && col_ok) {
            float b0, b1;
            if (a.b3_plane) {
                b0 = __ldg(a.b3 + ((int64_t)co * a.b3_rows + (2 * R - a.b3_row0)) * a.w3 + c);
                b1 = __ldg(a.b3 + ((int64_t)co * a.b3_rows + (2 * R + 1 - a.b3_row0)) * a.w3 + c);
            } else {
                b0 = b1 = __ldg(a.b3 + co);
            }
            t0 = tanh_f(v0[co] + b0);
            t1 = tanh_f(v1[co] + b1);
        }
        // odd lanes hold column c+1 of the even lane's 2x2 window
        const float t01 = __shfl_down_sync(0xffffffffu, t0, 1);
        const float t11 = __shfl_down_sync(0xffffffffu, t1, 1);
        if (row_ok && !(lane & 1) && C < a.w4) {
            float s = S.p4[co][0] * t0;
            s = fmaf(S.p4[co][1], t01, s);
            s = fmaf(S.p4[co][2], t1, s);
            s = fmaf(S.p4[co][3], t11, s);
            tv[co] = tanh_f(s);
        }
    }
    if (row_ok && !(lane & 1) && C < a.w4) {
        // T4 as bf16 channel blocks [3][rows][w4][8] (U3's tensor-core operand rows)
        const int64_t bplane = a.t4_rows * a.w4;
        uint4* t4 = reinterpret_cast<uint4*>(a.t4) + img * 3 * bplane + (R - a.t4_row0) * a.w4 + C;
        t4[0] = make_uint4(tc::pack_bf16(tv[0], tv[1]), tc::pack_bf16(tv[2], tv[3]), tc::pack_bf16(tv[4], tv[5]),
                           tc::pack_bf16(tv[6], tv[7]));
        t4[bplane] = make_uint4(tc::pack_bf16(tv[8], tv[9]), tc::pack_bf16(tv[10], tv[11]),
                                tc::pack_bf16(tv[12], tv[13]), tc::pack_bf16(tv[14], tv[15]));
        t4[2 * bplane] = make_uint4(tc::pack_bf16(tv[16], tv[17]), tc::pack_bf16(tv[18], tv[19]), 0u, 0u);
    }
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<64>(tmem);
}

// ============================================================================ U3 (C5 + C6)
// Band = 256 output positions (two M=128 tiles). Narrow images (w4 <= kFlatMax): positions are
// the flattened (row, col) index over rows of pitch w4 (columns >= w5 are discarded); wide
// images: one output row, columns [c0, c0+256), window pitch 262.
constexpr int kFlatMax = 180;
constexpr int U3_WR_COL = 5, U3_WP_COL = 2 * kTileM + 6;
constexpr int U3_KS = 40, U3_KS_STAGE = 4;    // 40 K-steps streamed in stages of 4
constexpr int U3_NMAX = 128;
// window pixels per channel block: flat mode <= (256 + 6 * w4) + 8, column mode 5 * 262 + 8
constexpr int U3_APLANE_MAX = 1416;
static_assert(2 * kTileM + 6 * kFlatMax + 8 <= U3_APLANE_MAX && U3_WR_COL * U3_WP_COL + 8 <= U3_APLANE_MAX, "window");

struct U3TcShared {
    uint4 a[3][U3_APLANE_MAX];                      // channel blocks 0-7, 8-15, 16-19(+4 zero)
    uint4 b[2][U3_KS_STAGE * 2 * U3_NMAX];          // double-buffered B stages
    float k6[U3_NMAX][12];                          // [ch][o] (9 used)
    uint64_t mbar[2];
    uint32_t tmem;
};

constexpr int kThreadsU3 = 256;  // 8 warps: warps 0-3 drain tile 0, warps 4-7 tile 1

__global__ void __launch_bounds__(kThreadsU3, 2) cnn_u3_tc_kernel(const CnnU3Args a) {
    extern __shared__ __align__(128) uint8_t smraw[];
    U3TcShared& S = *reinterpret_cast<U3TcShared*>(smraw);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int NP = a.n_pad;                 // n5 padded to a multiple of 16 (<= 128)
    const int64_t img = blockIdx.z;
    const bool flat = a.w4 <= kFlatMax;
    // ---- band geometry
    int64_t q0, wr0;  // first position; first window row (global T4 row)
    int WP, WR, base;
    if (flat) {
        q0 = (int64_t)blockIdx.x * 2 * kTileM;         // flattened over rows [out_row0, +out_rows)
        const int64_t r_first = q0 / a.w4;
        wr0 = a.out_row0 + r_first;
        WP = (int)a.w4;
        base = (int)(q0 - r_first * a.w4);
        WR = (base + 2 * kTileM - 1) / WP + 1 + 4;  // rows the band spans + the 4-row halo
    } else {
        const int64_t bands_per_row = (a.w5 + 2 * kTileM - 1) / (2 * kTileM);
        const int64_t row = blockIdx.x / bands_per_row;
        q0 = (blockIdx.x - row * bands_per_row) * 2 * kTileM;  // column of position 0
        wr0 = a.out_row0 + row;
        WP = U3_WP_COL;
        WR = U3_WR_COL;
        base = 0;
    }
    const int plane_px = WR * WP + 8;  // + spare pixels (read by the zero-weight half of tap pair (4,5))

    if (warp == 0) tc::tmem_alloc<256>(&S.tmem);
    if (tid == 0) {
        tc::mbar_init(&S.mbar[0], 1);
        tc::mbar_init(&S.mbar[1], 1);
        tc::mbar_fence_init();
    }
    // ---- stage the T4 window as bf16 [block][row][col][8]
    // U2 wrote T4 as bf16 channel blocks [3][rows][w4][8]: three 16-byte loads per pixel
    const int64_t bplane = a.t4_rows * a.w4;
    const uint4* t4b = reinterpret_cast<const uint4*>(a.t4) + img * 3 * bplane;
    const int64_t wc0 = flat ? 0 : q0;
    for (int idx = tid; idx < plane_px; idx += kThreadsU3) {
        const int r = idx / WP, c = idx - r * WP;
        const int64_t br = wr0 + r - a.t4_row0, gc = wc0 + c;
        const bool ok = idx < WR * WP && br >= 0 && br < a.t4_rows && gc < a.w4;
        const int64_t o = br * a.w4 + gc;
        const uint4 z = make_uint4(0u, 0u, 0u, 0u);
        S.a[0][idx] = ok ? __ldg(t4b + o) : z;
        S.a[1][idx] = ok ? __ldg(t4b + bplane + o) : z;
        S.a[2][idx] = ok ? __ldg(t4b + 2 * bplane + o) : z;
    }
    for (int idx = tid; idx < U3_NMAX * 9; idx += kThreadsU3) {
        const int ch = idx / 9, o = idx - ch * 9;
        S.k6[ch][o] = ch < a.n5 ? __ldg(a.k6 + o * a.n5 + ch) : 0.f;
    }
    const uint4* kb = reinterpret_cast<const uint4*>(a.k5_tc);
    const int stage_vec = U3_KS_STAGE * 2 * NP;  // uint4 per stage
    for (int idx = tid; idx < stage_vec; idx += kThreadsU3) S.b[0][idx] = __ldg(kb + idx);
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    const uint32_t tmem = S.tmem;
    const uint32_t idesc = tc::make_idesc_bf16(kTileM, NP);
    const uint32_t plane_bytes = (uint32_t)(U3_APLANE_MAX * 16);
    const uint32_t a_base = tc::smem_u32(S.a[0]);

    constexpr int kStages = U3_KS / U3_KS_STAGE;
    for (int st = 0; st < kStages; ++st) {
        if (tid == 0) {
            tc::fence_after_sync();
            const uint32_t b_base = tc::smem_u32(S.b[st & 1]);
            for (int u = 0; u < U3_KS_STAGE; ++u) {
                const int ks = st * U3_KS_STAGE + u;
                const int i = ks / 8, r8 = ks % 8;
                uint32_t a_addr, lbo;
                if (r8 < 5) {  // channels 0-15 of tap (i, r8): blocks 0 and 1
                    a_addr = a_base + (uint32_t)((base + i * WP + r8) * 16);
                    lbo = plane_bytes;
                } else {       // channels 16-19 of taps (i, j) and (i, j+1): block 2, next pixel
                    const int j = 2 * (r8 - 5);
                    a_addr = a_base + 2 * plane_bytes + (uint32_t)((base + i * WP + j) * 16);
                    lbo = 16;
                }
                const uint64_t bd = tc::make_desc(b_base + (uint32_t)(u * 2 * NP * 16), (uint32_t)(NP * 16), 128);
                for (int t = 0; t < 2; ++t) {
                    const uint64_t ad = tc::make_desc(a_addr + (uint32_t)(t * kTileM * 16), lbo, 128);
                    tc::mma_bf16(tmem + (uint32_t)(t * NP), ad, bd, idesc, ks > 0 ? 1u : 0u);
                }
            }
            tc::commit(&S.mbar[st & 1]);
        }
        if (st + 1 < kStages) {
            // buffer (st+1)&1 was read by stage st-1: wait for its MMAs before overwriting
            if (st >= 1) tc::mbar_wait(&S.mbar[(st + 1) & 1], (uint32_t)(((st - 1) >> 1) & 1));
            const uint4* src = kb + (size_t)(st + 1) * stage_vec;
            for (int idx = tid; idx < stage_vec; idx += kThreadsU3) S.b[(st + 1) & 1][idx] = __ldg(src + idx);
            tc::fence_proxy_async();
            tc::fence_before_sync();
            __syncthreads();
        }
    }
    // the last stage's commit covers every MMA issued before it
    tc::mbar_wait(&S.mbar[(kStages - 1) & 1], (uint32_t)(((kStages - 1) >> 1) & 1));
    tc::fence_after_sync();

    // ---- epilogue: warp w drains tile w/4, TMEM lanes 32*(w%4).. (its lane quarter)
    const uint32_t lane_base = (uint32_t)(32 * (warp & 3)) << 16;
    {
        const int t = warp >> 2;
        const int m = t * kTileM + 32 * (warp & 3) + lane;
        int64_t orow, ocol;
        if (flat) {
            const int64_t q = q0 + m;
            orow = a.out_row0 + q / a.w4;
            ocol = q - (q / a.w4) * a.w4;
        } else {
            orow = wr0;
            ocol = q0 + m;
        }
        const bool ok = orow < a.out_row0 + a.out_rows && ocol < a.w5;
        float c6[9];
#pragma unroll
        for (int o = 0; o < 9; ++o) c6[o] = 0.f;
        for (int cb = 0; cb < NP; cb += 32) {
            float v[32];
            tc::tmem_ld32(tmem + lane_base + (uint32_t)(t * NP + cb), v);  // warp-uniform
            if (ok) {
#pragma unroll
                for (int u = 0; u < 32; ++u) {
                    const int ch = cb + u;
                    if (ch < a.n5) {
                        const float b = a.b5_plane
                                            ? __ldg(a.b5 + ((int64_t)ch * a.b5_rows + (orow - a.b5_row0)) * a.w5 + ocol)
                                            : __ldg(a.b5 + ch);
                        const float th = tanh_f(v[u] + b);
#pragma unroll
                        for (int o = 0; o < 9; ++o) c6[o] = fmaf(S.k6[ch][o], th, c6[o]);
                    }
                }
            }
        }
        if (ok) {
            float* ob = a.out + img * a.out_img_stride + (orow - a.out_row0) * a.w5 + ocol;
#pragma unroll
            for (int o = 0; o < 9; ++o) {
                const float b = a.b6_plane ? __ldg(a.b6 + ((int64_t)o * a.b6_rows + (orow - a.b6_row0)) * a.w5 + ocol)
                                           : __ldg(a.b6 + o);
                ob[o * a.out_plane_stride] = c6[o] + b;
            }
        }
    }
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<256>(tmem);
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
    const size_t smem = sizeof(U2TcShared);
    if (!set_smem_attr((const void*)cnn_u2_tc_kernel, smem, flags)) return cudaErrorInvalidValue;
    dim3 grid((unsigned)((a.w3 + kTileM - 1) / kTileM), (unsigned)a.t4_rows, (unsigned)a.nimg);
    cnn_u2_tc_kernel<<<grid, kThreads, smem, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_cnn_u3_tc(const CnnU3Args& a, cudaStream_t s) {
    if (a.out_rows <= 0 || a.nimg <= 0) return cudaSuccess;
    if (a.n_pad > U3_NMAX || a.n_pad % 16) return cudaErrorInvalidValue;
    static std::atomic<uint32_t> flags{0};
    const size_t smem = sizeof(U3TcShared);
    if (!set_smem_attr((const void*)cnn_u3_tc_kernel, smem, flags)) return cudaErrorInvalidValue;
    unsigned bands;
    if (a.w4 <= kFlatMax)
        bands = (unsigned)((a.out_rows * a.w4 + 2 * kTileM - 1) / (2 * kTileM));
    else
        bands = (unsigned)(a.out_rows * ((a.w5 + 2 * kTileM - 1) / (2 * kTileM)));
    dim3 grid(bands, 1, (unsigned)a.nimg);
    cnn_u3_tc_kernel<<<grid, kThreadsU3, smem, s>>>(a);
    return cudaGetLastError();
}

}  // namespace tg
