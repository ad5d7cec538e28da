// Probe: which FFMA2 operand forms run on this GPU (uniform-register vs register weights).
#include <cstdio>
#include <cuda_runtime.h>
struct W { float2 w[64]; };
__global__ void k_ur(const float2* in, float2* out, const __grid_constant__ W wt) {
    float2 a = make_float2(0.f, 0.f);
    float2 x = in[threadIdx.x];
#pragma unroll 1
    for (int i = 0; i < 64; ++i) a = __ffma2_rn(x, wt.w[i], a);
    out[threadIdx.x] = a;
}
__global__ void k_reg(const float2* in, float2* out, const float2* w) {
    __shared__ float2 ws[64];
    if (threadIdx.x < 64) ws[threadIdx.x] = w[threadIdx.x];
    __syncthreads();
    float2 a = make_float2(0.f, 0.f);
    float2 x = in[threadIdx.x];
#pragma unroll 1
    for (int i = 0; i < 64; ++i) a = __ffma2_rn(x, ws[i], a);
    out[threadIdx.x] = a;
}
struct WS { float w[64]; };
__global__ void k_bc(const float2* in, float2* out, const __grid_constant__ WS wt) {
    float2 a = make_float2(0.f, 0.f);
    float2 x = in[threadIdx.x];
#pragma unroll 1
    for (int i = 0; i < 64; i += 2) {
        a = __ffma2_rn(x, make_float2(wt.w[i], wt.w[i]), a);
        a = __ffma2_rn(x, make_float2(wt.w[i + 1], wt.w[i + 1]), a);
    }
    out[threadIdx.x] = a;
}
int main() {
    float2 *in, *out, *w;
    cudaMalloc(&in, 256 * 8); cudaMalloc(&out, 256 * 8); cudaMalloc(&w, 64 * 8);
    cudaMemset(in, 0, 256 * 8); cudaMemset(w, 0, 64 * 8);
    W wt{};
    k_reg<<<1, 256>>>(in, out, w);
    printf("reg form: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    k_ur<<<1, 256>>>(in, out, wt);
    printf("uniform-register form: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    WS ws{};
    k_bc<<<1, 256>>>(in, out, ws);
    printf("broadcast .F32 form: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
