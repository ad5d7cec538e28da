/* oracle.h -- TEST INFRASTRUCTURE ONLY (see oracle.c). Not included by, linked into, or
 * shared with the product library under paper_conf_ipps_sundaramrc09_b200/. */
#ifndef TG_ORACLE_H
#define TG_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif
int orc_num_threads(void);
void orc_set_num_threads(int n);
void orc_conv2d_valid(const float* x, int64_t H, int64_t W, const float* K, int kh, int kw, float* y);
void orc_conv2d_same(const float* x, int64_t H, int64_t W, const float* K, int kh, int kw, float* y);
void orc_add(const float* a, const float* b, float* y, int64_t n);
void orc_add_scalar(const float* a, float b, float* y, int64_t n);
void orc_neg(const float* a, float* y, int64_t n);
void orc_tanh(const float* a, float* y, int64_t n);
void orc_max_fold(const float* const* xs, int nx, float* y, int64_t n);
void orc_subsample(const float* x, int64_t H, int64_t W, const float* P, int s, float* y);
void orc_matmul(const float* A, const float* B, int64_t M, int64_t K, int64_t N, float* C);
int orc_edge(const float* img, int64_t H, int64_t W, const float* K1, const float* K2, int ks,
             float* E, float* E1_out, float* E2_out);
int orc_cnn(const float* img, int64_t n, int64_t H, int64_t W, int n5, const float* const* prm,
            int bias_plane, float* out);
#ifdef __cplusplus
}
#endif
#endif
