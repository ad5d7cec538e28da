// kernels.h -- launchers of the fused sm_100a offload-unit kernels (product code).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

namespace tg {

// K1: the whole edge template as one kernel per chunk (the paper's "best
// possible" single kernel): E = max(Im*K1, Im*K2, -(Im*K1), -(Im*K2)),
// SAME zero padding; generally nf <= 4 convolutions combined by max (with remaps), sum,
// max-abs or plain max. Rows are in GLOBAL image coordinates; rows outside [0, H) are zero.
struct EdgeArgs {
    const float* in;        // image rows [in_row0, in_row0 + in_rows) of nimg images
    int64_t in_img_stride;  // floats between consecutive images in `in`
    int64_t in_row0, in_rows;
    float* out;             // output rows [out_row0, out_row0 + out_rows) of nimg images
    int64_t out_img_stride;
    int64_t out_row0, out_rows;
    int64_t H, W;           // full image size
    int64_t nimg;
    const float* k_host[4]; // nf ks x ks filters (host; passed to the kernel by value)
    int nf;                 // 1..4 convolutions
    int ks;                 // 1..16
    int combine;            // 0 max over responses and remaps, 1 sum, 2 max |.|, 3 max
};
cudaError_t launch_edge(const EdgeArgs& a, cudaStream_t s);
// measured FP32 FFMA peak (TFLOP/s, best of a few launches; probe.cu)
cudaError_t probe_fp32_peak(int device, double* tflops);

// CNN offload units (fp32 FFMA path). Row ranges are global level coordinates.
struct CnnU1Args {          // C1(1->8, 5x5) + bias + tanh + S2 + tanh  -> T2
    const float* in; int64_t in_img_stride; int64_t in_row0;   // rows of the input image
    int64_t W;                                                 // input width
    const float* k1_host;   // [8][25] (host; passed by value in the constant bank)
    const float* b1;        // plane [8][b1_rows][w1] starting at global C1 row b1_row0, or scalar [8]
    int64_t b1_row0, b1_rows; int b1_plane;
    const float* p2_host;   // [8][4] (host)
    float* t2; int64_t t2_img_stride; int64_t t2_row0, t2_rows;  // [8][t2_rows][w2]
    int64_t w1, w2;
    int64_t nimg;
    int bf16_out;           // 1: write T2 as bf16 [rows][w2][8] (operand layout of U2 on tcgen05)
    int t2_h3;              // 1 (TG_FP32_TC): write T2 fp16-split [2][rows][w2][8] (x 2^4) for the 3xFP16 U2
};
struct CnnU2Args {          // C3(8->20, 5x5) + bias + tanh + S4 + tanh -> T4
    const float* t2; int64_t t2_img_stride; int64_t t2_row0, t2_rows; int64_t w2;
    const float* k3_host;   // [20][8][25] (host; constant bank)
    const float* b3; int64_t b3_row0, b3_rows; int b3_plane;      // plane [20][b3_rows][w3]
    const float* p4_host;   // [20][4] (host)
    float* t4; int64_t t4_img_stride; int64_t t4_row0, t4_rows; int64_t w3, w4;
    int64_t nimg;
    int bf16_tc;            // 1: tcgen05 bf16 path: T2 read as bf16 [rows][w2][8], T4 written
                            //    as bf16 [3][rows][w4][8] (channel blocks 0-7, 8-15, 16-19+pad)
    const uint16_t* k3_tc;  // bf16 B operand prepared by cnn_prepare_k3_tc (device)
    const float* p4_dev;    // [20][4] (device)
    const uint16_t* k3_h3;  // fp16-split B operand of the 3xFP16 C3 (cnn_prepare_k3_h3, device)
    float w_unscale;        // 3xFP16: 1 / (activation scale x the weight scale of cnn_h3_weight_scale)
};
struct CnnU3Args {          // C5(20->n5, 5x5) + bias + tanh + C6(n5->9, 1x1) + bias -> out
    const float* t4; int64_t t4_img_stride; int64_t t4_row0, t4_rows; int64_t w4;
    const float* k5;        // [n5][20][25]
    const float* b5; int64_t b5_row0, b5_rows; int b5_plane;      // plane [n5][b5_rows][w5]
    int b5_q4;              // tensor-core paths: b5 is channel-quad interleaved [n5/4][b5_rows][w5][4]
    const float* k6;        // [9][n5]
    const float* b6; int64_t b6_row0, b6_rows; int b6_plane;      // plane [9][b6_rows][w5]
    float* out; int64_t out_img_stride; int64_t out_plane_stride; int64_t out_row0, out_rows; int64_t w5;
    int n5;
    int64_t nimg;
    int bf16_tc;            // 1: tcgen05 path, T4 read as bf16 [3][rows][w4][8]
    const uint16_t* k5_tc;  // bf16 B operand prepared by cnn_prepare_k5_tc (device)
    const float* k6_host;   // [9][n5] (host; passed by value to the tensor-core kernel)
    int n_pad;              // n5 rounded up to a multiple of 16
    float w_unscale;        // 3xFP16: 1 / (activation scale x the weight scale of cnn_h3_weight_scale)
};
cudaError_t launch_cnn_u1(const CnnU1Args& a, cudaStream_t s);
cudaError_t launch_cnn_u2(const CnnU2Args& a, cudaStream_t s);
cudaError_t launch_cnn_u3(const CnnU3Args& a, cudaStream_t s);

// Generic per-operator kernels (generic.cu) for the TG_PER_OP / TG_BASELINE modes. Every
// kernel computes output rows [r0, r1) of its operator (a piece of a split operator,
// PAPER.md:359-367, or the whole operator) into a piece buffer laid out [n][c][r1-r0][w].
// Inputs are views: the pieces of a data structure that the operator reads, each a row band
// [r0, r1) stored [n][c][r1-r0][w]; a row is looked up in the first piece that holds it
// (overlapping pieces hold identical rows).
constexpr int kGenMaxSeg = 8;
struct GenSeg {
    const float* p;
    int64_t r0, r1;
};
struct GenView {
    GenSeg seg[kGenMaxSeg];
    int32_t nseg;
};
struct GenConvArgs {
    GenView x, bias;        // image [n][ci][h][w]; bias plane [1][co][ho][wo] or scalar [co]
    const float* k;         // kernel [co][ci][kh][kw] (whole parameter)
    float* y;               // output rows [r0, r1): [n][co][r1-r0][wo]
    int64_t r0, r1;
    int64_t n, ci, h, w, co, kh, kw, wo;
    int pt, pl;             // top/left padding (0 for VALID)
    int bias_kind;          // 0 none, 1 scalar [co], 2 plane [co][ho][wo]
};
constexpr int kGenMaxInputs = 16;
struct GenElemArgs {
    GenView xs[kGenMaxInputs]; int nx;
    float* y;               // rows [r0, r1) of [n][c][h][w]: [n][c][r1-r0][w]
    int64_t r0, r1, planes, w;
    int op;                 // 0 add, 1 neg, 2 affine, 3 abs, 4 tanh, 5 max
    float a, b;
};
struct GenSubArgs {
    GenView x; const float* p; float* y;
    int64_t r0, r1;
    int64_t n, c, h, w, wo; int s;
};
// C = A B over rows [r0, r1) of A and C; A [m][k] (view), B [k][n] (view,
// read whole), C rows [r0, r1) of [m][n]
struct GenMatmulArgs {
    GenView a, b; float* c;
    int64_t r0, r1, k, n;
};
cudaError_t launch_gen_conv(const GenConvArgs& a, cudaStream_t s);
cudaError_t launch_gen_elem(const GenElemArgs& a, cudaStream_t s);
cudaError_t launch_gen_sub(const GenSubArgs& a, cudaStream_t s);
cudaError_t launch_gen_matmul(const GenMatmulArgs& a, cudaStream_t s);

// tcgen05 (bf16 operands, fp32 accumulation in TMEM) variants of U2 and U3 (cnn_tc.cu)
cudaError_t launch_cnn_u2_tc(const CnnU2Args& a, cudaStream_t s);
cudaError_t launch_cnn_u3_tc(const CnnU3Args& a, cudaStream_t s);
// 3xFP16 U2 / U3 (cnn_h3.cu): T2 [2][rows][w2][8] and T4 [2][3][rows][w4][8] fp16-split
// weights are scaled by a power of two (max |w| x scale in [2^13, 2^14)) before the split, so the fp16
// parts neither overflow nor lose their low part for any weight magnitude
float cnn_h3_weight_scale(const float* w, size_t n);
float cnn_h3_act_scale();
size_t cnn_k3_h3_bytes();
void cnn_prepare_k3_h3(const float* k3, float scale, uint16_t* dst);
size_t cnn_k5_h3_bytes(int n5);
void cnn_prepare_k5_h3(const float* k5, int n5, float scale, uint16_t* dst);
cudaError_t launch_cnn_u2_h3(const CnnU2Args& a, cudaStream_t s);
cudaError_t launch_cnn_u3_h3(const CnnU3Args& a, cudaStream_t s);
size_t cnn_k3_tc_bytes();
void cnn_prepare_k3_tc(const float* k3, uint16_t* dst);
int cnn_n5_pad(int n5);
size_t cnn_k5_tc_bytes(int n5);
void cnn_prepare_k5_tc(const float* k5, int n5, uint16_t* dst);

}  // namespace tg
