/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY. A plain, slow, obviously-correct CPU evaluation of
 * the UNSPLIT operator graphs of Sundaram, Raghunathan & Chakradhar (IPDPS 2009).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load this library. The product path (paper_conf_ipps_sundaramrc09_b200/) never
 * links, imports or calls it, and shares no code, header, table or constant with it.
 *
 * Every data structure (DS) is an fp32 array, as the paper's "floats" (PAPER.md:741,
 * Table 1 header). Each operator node reads fp32 inputs and writes ONE fp32 output.
 * Inside a convolution / subsample node the sum is accumulated in fp64 and rounded once
 * (SURVEY §8(c) "Definition"). Operators are evaluated one node at a time, in the order
 * the paper's graphs define (Fig. 1(b)/Fig. 3 for edge detection, Fig. 7 for the CNN
 * layers); nothing is blocked, fused or reordered.
 *
 * Readings of the paper this file depends on:
 *   R1 convolution = cross-correlation (torch5 SpatialConvolution)
 *   R2 edge conv: same-size output (Table 1 I/O count), zero padding,
 *      top/left pad (k-1)/2, bottom/right pad k/2
 *   R3 remap R = elementwise negation
 *   R5 combine = ONE 4-input max operator, left fold (a > b) ? a : b in order E1,E2,E5,E6
 *   R7 CNN = C1 T S2 T C3 T S4 T C5 T C6, Fig. 7 expansion, bias plane per map
 *   R8 subsample = 2x2 window, stride 2, 4-float kernel per plane, no bias
 *   R9 tanh = plain tanh, evaluated in double, rounded to fp32
 *
 * Parallelism: OpenMP `parallel for` over output rows of one node (plain; it does not
 * change any value because every output element is computed independently).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#include "oracle.h"

int orc_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

void orc_set_num_threads(int n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}

/* conv2d VALID, cross-correlation ("a 100x100 matrix
 * convolved with a 5x5 kernel matrix results in an output of size 96x96"):
 *   y[r][c] = sum_{i<kh} sum_{j<kw} x[r+i][c+j] * K[i][j],  y is (H-kh+1) x (W-kw+1). */
void orc_conv2d_valid(const float* x, int64_t H, int64_t W, const float* K, int kh, int kw,
                      float* y) {
    const int64_t Ho = H - kh + 1, Wo = W - kw + 1;
    if (Ho <= 0 || Wo <= 0) return;
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < Ho; ++r) {
        for (int64_t c = 0; c < Wo; ++c) {
            double acc = 0.0;
            for (int i = 0; i < kh; ++i)
                for (int j = 0; j < kw; ++j)
                    acc += (double)x[(r + i) * W + (c + j)] * (double)K[i * kw + j];
            y[r * Wo + c] = (float)acc;
        }
    }
}

/* conv2d SAME (edge template; reading R2): zero outside the image,
 *   y[r][c] = sum_{i<kh} sum_{j<kw} x~[r+i-pt][c+j-pl] * K[i][j],  pt=(kh-1)/2, pl=(kw-1)/2. */
void orc_conv2d_same(const float* x, int64_t H, int64_t W, const float* K, int kh, int kw,
                     float* y) {
    const int pt = (kh - 1) / 2, pl = (kw - 1) / 2;
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < H; ++r) {
        for (int64_t c = 0; c < W; ++c) {
            double acc = 0.0;
            for (int i = 0; i < kh; ++i) {
                const int64_t rr = r + i - pt;
                if (rr < 0 || rr >= H) continue; /* x~ = 0 outside the image */
                for (int j = 0; j < kw; ++j) {
                    const int64_t cc = c + j - pl;
                    if (cc < 0 || cc >= W) continue;
                    acc += (double)x[rr * W + cc] * (double)K[i * kw + j];
                }
            }
            y[r * W + c] = (float)acc;
        }
    }
}

/* data-parallel add (Fig. 7 "A" nodes): y = fl32(a + b) */
void orc_add(const float* a, const float* b, float* y, int64_t n) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) y[i] = (float)((double)a[i] + (double)b[i]);
}

/* add a scalar (bias-scalar variant of O_j = S + B_j): y = fl32(a + b) */
void orc_add_scalar(const float* a, float b, float* y, int64_t n) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) y[i] = (float)((double)a[i] + (double)b);
}

/* remap R (reading R3): y = -x (exact) */
void orc_neg(const float* a, float* y, int64_t n) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) y[i] = -a[i];
}

/* tanh (reading R9; "5 tanh layers"): tanh in double, rounded to fp32 */
void orc_tanh(const float* a, float* y, int64_t n) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) y[i] = (float)tanh((double)a[i]);
}

/* n-ary max combine (reading R5; "combining the results by doing a reduction
 * such as addition/max"): left fold m = x1; m = (xk > m) ? xk : m. */
void orc_max_fold(const float* const* xs, int nx, float* y, int64_t n) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        float m = xs[0][i];
        for (int k = 1; k < nx; ++k) {
            const float v = xs[k][i];
            m = (v > m) ? v : m;
        }
        y[i] = m;
    }
}

/* subsample (reading R8): window s, stride s, kernel P[s][s]:
 *   y[r][c] = sum_{a<s} sum_{b<s} P[a][b] * x[s*r+a][s*c+b],  output floor((D-s)/s)+1. */
void orc_subsample(const float* x, int64_t H, int64_t W, const float* P, int s, float* y) {
    const int64_t Ho = (H - s) / s + 1, Wo = (W - s) / s + 1;
    if (H < s || W < s) return;
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < Ho; ++r) {
        for (int64_t c = 0; c < Wo; ++c) {
            double acc = 0.0;
            for (int a = 0; a < s; ++a)
                for (int b = 0; b < s; ++b)
                    acc += (double)P[a * s + b] * (double)x[(s * r + a) * W + (s * c + b)];
            y[r * Wo + c] = (float)acc;
        }
    }
}

/* matrix-matrix multiply C = A B ("a large matrix-matrix multiply that does not
 * fit in the GPU memory can be split by breaking up one of the input matrices and the output
 * matrix"; the operator itself is the textbook product):
 *   C[i][j] = sum_{l<K} A[i][l] * B[l][j],  A is M x K, B is K x N, C is M x N,
 * accumulated in fp64 over l = 0..K-1 and rounded once to fp32. */
void orc_matmul(const float* A, const float* B, int64_t M, int64_t K, int64_t N, float* C) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < M; ++i) {
        for (int64_t j = 0; j < N; ++j) {
            double acc = 0.0;
            for (int64_t l = 0; l < K; ++l) acc += (double)A[i * K + l] * (double)B[l * N + j];
            C[i * N + j] = (float)acc;
        }
    }
}

/* Edge-detection template, 4 orientations ("16x16 sized edge filter at four
 * different orientations (2 convolutions and 2 remaps) and combined the results using a
 * Max operation"; graph of Fig. 3 / SURVEY F1):
 *   C1: E1 = Im * K1   C2: E2 = Im * K2   R1: E5 = -E1   R2: E6 = -E2
 *   max: E = max(E1, E2, E5, E6)
 * E1/E2 may be NULL (scratch is allocated); when non-NULL they receive C1/C2's outputs. */
int orc_edge(const float* img, int64_t H, int64_t W, const float* K1, const float* K2, int ks,
             float* E, float* E1_out, float* E2_out) {
    const int64_t n = H * W;
    float* E1 = E1_out ? E1_out : (float*)malloc(sizeof(float) * (size_t)n);
    float* E2 = E2_out ? E2_out : (float*)malloc(sizeof(float) * (size_t)n);
    float* E5 = (float*)malloc(sizeof(float) * (size_t)n);
    float* E6 = (float*)malloc(sizeof(float) * (size_t)n);
    if (!E1 || !E2 || !E5 || !E6) return -5;
    orc_conv2d_same(img, H, W, K1, ks, ks, E1);
    orc_conv2d_same(img, H, W, K2, ks, ks, E2);
    orc_neg(E1, E5, n);
    orc_neg(E2, E6, n);
    const float* xs[4] = {E1, E2, E5, E6};
    orc_max_fold(xs, 4, E, n);
    if (!E1_out) free(E1);
    if (!E2_out) free(E2);
    free(E5);
    free(E6);
    return 0;
}

/* One fully connected conv layer expanded as in Fig. 7:
 *   L_ij = In_i * K_ji                      (per-pair convolution, VALID)
 *   S_j1 = L_1j + L_2j,  S_jk = S_j(k-1) + L_(k+1)j
 *   O_j  = S_last + B_j      (O_j = L_1j + B_j when n_in == 1)
 * in: [n_in][H][W], K: [n_out][n_in][k][k], bias: plane [n_out][Ho][Wo] or scalar [n_out]. */
static int conv_layer_fig7(const float* in, int n_in, int64_t H, int64_t W, const float* K,
                           int k, int n_out, const float* bias, int bias_plane, float* out) {
    const int64_t Ho = H - k + 1, Wo = W - k + 1, po = Ho * Wo, pi = H * W;
    float* L = (float*)malloc(sizeof(float) * (size_t)po);
    float* S = (float*)malloc(sizeof(float) * (size_t)po);
    if (!L || !S) return -5;
    for (int j = 0; j < n_out; ++j) {
        float* O = out + (int64_t)j * po;
        /* S holds the running partial sum; for n_in == 1 it is L_1j itself */
        orc_conv2d_valid(in, H, W, K + ((int64_t)j * n_in + 0) * k * k, k, k, S);
        for (int i = 1; i < n_in; ++i) {
            orc_conv2d_valid(in + (int64_t)i * pi, H, W, K + ((int64_t)j * n_in + i) * k * k, k,
                             k, L);
            orc_add(S, L, S, po);
        }
        if (bias_plane)
            orc_add(S, bias + (int64_t)j * po, O, po);
        else
            orc_add_scalar(S, bias[j], O, po);
    }
    free(L);
    free(S);
    return 0;
}

static void tanh_planes(float* x, int64_t n) { orc_tanh(x, x, n); }

static void subsample_planes(const float* in, int c, int64_t H, int64_t W, const float* P,
                             float* out) {
    const int64_t Ho = (H - 2) / 2 + 1, Wo = (W - 2) / 2 + 1;
    for (int i = 0; i < c; ++i)
        orc_subsample(in + (int64_t)i * H * W, H, W, P + 4 * i, 2, out + (int64_t)i * Ho * Wo);
}

/* CNN template (reconstructed in SURVEY F2 / Appendix A):
 *   C1(1->8,5x5) T S2(2x2/2) T C3(8->20,5x5) T S4(2x2/2) T C5(20->n5,5x5) T C6(n5->9,1x1)
 * img: [n][1][H][W]; params in the order K1,B1,P2,K3,B3,P4,K5,B5,K6,B6; bias planes are
 * [1][c][h][w] shared by every image of the batch (reading R7b); out: [n][9][H6][W6]. */
int orc_cnn(const float* img, int64_t n, int64_t H, int64_t W, int n5, const float* const* prm,
            int bias_plane, float* out) {
    const int64_t h1 = H - 4, w1 = W - 4;
    const int64_t h2 = (h1 - 2) / 2 + 1, w2 = (w1 - 2) / 2 + 1;
    const int64_t h3 = h2 - 4, w3 = w2 - 4;
    const int64_t h4 = (h3 - 2) / 2 + 1, w4 = (w3 - 2) / 2 + 1;
    const int64_t h5 = h4 - 4, w5 = w4 - 4;
    if (h5 <= 0 || w5 <= 0) return -2;
    float* a1 = (float*)malloc(sizeof(float) * (size_t)(8 * h1 * w1));
    float* a2 = (float*)malloc(sizeof(float) * (size_t)(8 * h2 * w2));
    float* a3 = (float*)malloc(sizeof(float) * (size_t)(20 * h3 * w3));
    float* a4 = (float*)malloc(sizeof(float) * (size_t)(20 * h4 * w4));
    float* a5 = (float*)malloc(sizeof(float) * (size_t)(n5 * h5 * w5));
    if (!a1 || !a2 || !a3 || !a4 || !a5) return -5;
    int rc = 0;
    for (int64_t b = 0; b < n && rc == 0; ++b) {
        const float* x = img + b * H * W;
        float* o = out + b * 9 * h5 * w5;
        rc |= conv_layer_fig7(x, 1, H, W, prm[0], 5, 8, prm[1], bias_plane, a1); /* C1 */
        tanh_planes(a1, 8 * h1 * w1);                                           /* T  */
        subsample_planes(a1, 8, h1, w1, prm[2], a2);                            /* S2 */
        tanh_planes(a2, 8 * h2 * w2);                                           /* T  */
        rc |= conv_layer_fig7(a2, 8, h2, w2, prm[3], 5, 20, prm[4], bias_plane, a3); /* C3 */
        tanh_planes(a3, 20 * h3 * w3);                                          /* T  */
        subsample_planes(a3, 20, h3, w3, prm[5], a4);                           /* S4 */
        tanh_planes(a4, 20 * h4 * w4);                                          /* T  */
        rc |= conv_layer_fig7(a4, 20, h4, w4, prm[6], 5, n5, prm[7], bias_plane, a5); /* C5 */
        tanh_planes(a5, (int64_t)n5 * h5 * w5);                                 /* T  */
        rc |= conv_layer_fig7(a5, n5, h5, w5, prm[8], 1, 9, prm[9], bias_plane, o);   /* C6 */
    }
    free(a1);
    free(a2);
    free(a3);
    free(a4);
    free(a5);
    return rc;
}
