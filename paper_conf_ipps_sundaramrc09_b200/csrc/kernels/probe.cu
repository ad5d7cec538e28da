// probe.cu -- measured FP32 FFMA peak of the device (the denominator of the ALU-bound rooflines:
// K1 and the FFMA CNN units). Not part of the paper's method: measurement
// infrastructure (MEASURED_PEAKS.json has no FP32 figure, so the build measures it).
//
// Every thread runs 8 independent FFMA2 chains (paired FP32 FMA, 4 flop per instruction) on
// register operands; 8 warps per SM sub-partition hide the FMA latency, so the FMA pipes issue
// every cycle. A grid of 4 x (SM count) CTAs of 1024 threads, a few tens of milliseconds per launch.
#include <cuda_runtime.h>

#include <algorithm>

#include "kernels.h"

namespace tg {
namespace {

constexpr int kChains = 8;

__global__ void __launch_bounds__(1024) ffma2_peak_kernel(float* out, int iters, float seed) {
    float2 a[kChains];
#pragma unroll
    for (int c = 0; c < kChains; ++c) a[c] = make_float2(seed * (threadIdx.x + c), seed * (c + 1));
    const float2 x = make_float2(0.9999f, 1.0001f), y = make_float2(1e-7f, -1e-7f);
#pragma unroll 1
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int u = 0; u < 16; ++u)
#pragma unroll
            for (int c = 0; c < kChains; ++c) a[c] = __ffma2_rn(a[c], x, y);
    }
    float s = 0.f;
#pragma unroll
    for (int c = 0; c < kChains; ++c) s += a[c].x + a[c].y;
    if (s == 12345.678f) out[blockIdx.x] = s;  // keeps the chains alive, never true in practice
}

}  // namespace

cudaError_t probe_fp32_peak(int device, double* tflops) {
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return e;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    float* out = nullptr;
    if ((e = cudaMalloc(&out, 4096 * sizeof(float))) != cudaSuccess) return e;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int blocks = 4 * sms, threads = 1024, iters = 4096;
    double best = 0.0;
    for (int rep = 0; rep < 6; ++rep) {  // the first launches ramp the clocks up
        cudaEventRecord(a);
        ffma2_peak_kernel<<<blocks, threads>>>(out, iters, 1e-3f);
        cudaEventRecord(b);
        if ((e = cudaEventSynchronize(b)) != cudaSuccess) break;
        float ms = 0.f;
        cudaEventElapsedTime(&ms, a, b);
        const double flop = (double)blocks * threads * iters * 16 * kChains * 4;
        best = std::max(best, flop / (ms * 1e-3) / 1e12);
    }
    if (e == cudaSuccess) e = cudaGetLastError();
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    cudaFree(out);
    *tflops = best;
    return e;
}

}  // namespace tg
