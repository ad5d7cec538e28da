// pipe_probe.cu -- per-SM throughput (results per clock) of the instructions the CNN epilogues
// lean on: MUFU tanh / ex2 / rcp, the bf16x2 pack (cvt.rn.bf16x2.f32 -> F2FP), FFMA, FFMA2.
// One CTA of 1024 threads per SM, 8 independent chains per thread, clock64 around the loop.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/micro/pipe_probe tools/micro/pipe_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

constexpr int kIters = 4096;

template <int kOp>
__global__ void probe(long long* cyc, float* sink) {
    float v[8];
    uint32_t u[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) { v[j] = 0.001f * (threadIdx.x + j); u[j] = threadIdx.x * 7 + j; }
    __syncthreads();
    const long long t0 = clock64();
    for (int i = 0; i < kIters; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            if (kOp == 0) asm volatile("tanh.approx.f32 %0, %0;" : "+f"(v[j]));
            if (kOp == 1) asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(v[j]));
            if (kOp == 2) {  // rcp chain with a dependency the compiler cannot fold
                asm volatile("rcp.approx.ftz.f32 %0, %0;" : "+f"(v[j]));
                v[j] += 1.0f;
            }
            if (kOp == 3) {  // pack two floats to bf16x2, feed the bits back as a float
                uint32_t r;
                asm volatile("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(v[j]), "f"(v[(j + 1) & 7]));
                v[j] = __uint_as_float(r ^ 0x3f800000u);
            }
            if (kOp == 4) asm volatile("fma.rn.f32 %0, %0, %0, %0;" : "+f"(v[j]));
            if (kOp == 5) {
                float2 x = make_float2(v[j], v[(j + 4) & 7]);
                x = __ffma2_rn(x, x, x);
                v[j] = x.x; v[(j + 4) & 7] = x.y;
            }
            if (kOp == 7) {  // HFMA2: two fp16 FMAs per lane
                __half2 h = __floats2half2_rn(v[j], v[(j + 4) & 7]);
                asm volatile("fma.rn.f16x2 %0, %0, %0, %0;" : "+r"(*reinterpret_cast<uint32_t*>(&h)));
                const float2 f = __half22float2(h);
                v[j] = f.x;
            }
            if (kOp == 8) {  // HFMA2 chain kept in half2 registers (the conversion outside the loop)
                asm volatile("fma.rn.f16x2 %0, %0, %0, %0;" : "+r"(u[j]));
            }
            if (kOp == 6) {  // integer bf16 rounding + pack (alu/fma pipes): the F2FP alternative
                const uint32_t a0 = __float_as_uint(v[j]), a1 = __float_as_uint(v[(j + 1) & 7]);
                const uint32_t r0 = a0 + 0x7fffu + ((a0 >> 16) & 1u), r1 = a1 + 0x7fffu + ((a1 >> 16) & 1u);
                v[j] = __uint_as_float(__byte_perm(r0, r1, 0x7632) ^ 0x3f800000u);
            }
        }
    }
    const long long t1 = clock64();
    float s = 0.f;
#pragma unroll
    for (int j = 0; j < 8; ++j) s += v[j] + __uint_as_float(u[j]);
    if (s == 1.2345f) sink[threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int kOp>
void run(const char* name, int per_op_results) {
    long long* d;
    float* sink;
    cudaMalloc(&d, 148 * sizeof(long long));
    cudaMalloc(&sink, 1024 * sizeof(float));
    probe<kOp><<<148, 1024>>>(d, sink);
    probe<kOp><<<148, 1024>>>(d, sink);
    cudaError_t e = cudaDeviceSynchronize();
    long long h = 0;
    cudaMemcpy(&h, d, sizeof h, cudaMemcpyDeviceToHost);
    const double ops = 1024.0 * kIters * 8 * per_op_results;
    printf("%-36s %7.1f results/clk/SM  %s\n", name, ops / (double)h, e == cudaSuccess ? "" : cudaGetErrorString(e));
    cudaFree(d);
    cudaFree(sink);
}

int main() {
    run<0>("MUFU tanh.approx.f32", 1);
    run<1>("MUFU ex2.approx.ftz.f32", 1);
    run<2>("MUFU rcp.approx.ftz.f32", 1);
    run<3>("cvt.rn.bf16x2.f32 (values packed)", 2);
    run<4>("FFMA", 1);
    run<5>("FFMA2 (lanes)", 2);
    run<6>("int bf16 round+pack (values packed)", 2);
    run<8>("HFMA2 (lanes x 2)", 2);
    return 0;
}
