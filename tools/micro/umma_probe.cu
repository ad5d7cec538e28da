// umma_probe.cu -- measured cost of one tcgen05.mma (kind::f16, bf16 in, fp32 accumulate) as the
// CNN units issue them: operands in shared memory, K-major, NO swizzle (8-row x 16-byte core
// matrices), M = 128, N = 16 .. 256, back to back from one thread into one TMEM accumulator.
// Also: A from TMEM (the "ts" form), and the same MMAs with the operands laid out with the 32-byte
// swizzle (rows of one K-step = 32 bytes). Prints cycles per MMA (clock64 around a run of MMAs
// whose completion is awaited through tcgen05.commit + mbarrier).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_ipps_sundaramrc09_b200/csrc/kernels \
//        -o tools/micro/umma_probe tools/micro/umma_probe.cu && tools/micro/umma_probe
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#include "tc_sm100.cuh"

using namespace tg;

constexpr int kReps = 520;
constexpr int kSmem = 200 * 1024;

// layout: 0 = no swizzle (LBO = K-half distance, SBO = 128), 2 = 32-byte swizzle
__device__ __forceinline__ uint64_t desc_sw(uint32_t addr, uint32_t lbo, uint32_t sbo, int swz) {
    uint64_t d = tc::make_desc(addr, lbo, sbo);
    if (swz == 32) d |= (uint64_t)6 << 61;  // layout type SWIZZLE_32B (sm_100 encoding: 6)
    return d;
}

template <int N, bool kTs, int kSwz, int kShift = 0, int kLbo16 = 0, int kRot = 0, int kBRot = 0, int kAltD = 0,
          int kCommit = 0, int kFence = 0>
__global__ void probe(long long* out) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t bar, dummy, done_bar;
    __shared__ uint32_t tm;
    uint8_t* A = sm;                 // 128 rows x 16 K (4 KB) -- plus room
    uint8_t* B = sm + 16384;         // N rows x 16 K (kBRot: 40 such blocks, one per K-step)
    const int tid = threadIdx.x, warp = tid >> 5;
    for (int i = tid; i < kSmem / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0x3c003c00u;  // 1.0
    if (warp == 0) tc::tmem_alloc<512>(&tm);
    if (tid == 0) {
        tc::mbar_init(&bar, 1);
        tc::mbar_init(&dummy, (1 << 20) - 1);   // never completes: a sink for the per-slice commits
        tc::mbar_init(&done_bar, 1);
        tc::mbar_arrive(&done_bar);       // phase 0 complete: waits on it return at once
        tc::mbar_fence_init();
    }
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    if (warp == 0) {
        const uint32_t idesc = tc::make_idesc_bf16(128, N);
        const uint32_t a = tc::smem_u32(A), b = tc::smem_u32(B);
        // no swizzle: K-half at LBO (A: 2048 B, B: N*16), 8-row groups at SBO = 128 B
        // 32-byte swizzle: a row of one K-step is 32 contiguous bytes, 8-row atoms of 256 B
        // kShift: A starts kShift 16-byte rows into its buffer (a tap-shifted implicit-GEMM window);
        // kLbo16: the second K half is the NEXT row (LBO = 16 B, the tap-pair trick); kRot: the A
        // start rotates over 8 shifts MMA by MMA (as the K-steps of one filter row do)
        const uint64_t ad = kSwz ? desc_sw(a, 16, 256, kSwz)
                                 : tc::make_desc(a + 16 * kShift, kLbo16 ? 16u : 2048u, 128);
        const uint64_t bd = kSwz ? desc_sw(b, 16, 256, kSwz) : tc::make_desc(b, (uint32_t)(N * 16), 128);
        long long t0 = 0, t1 = 0;
        for (int pass = 0; pass < 2; ++pass) {
            __syncwarp();
            t0 = clock64();
            if (kFence & 128) {  // one lane; the barrier test is issued 4 MMAs before the end of the
                                         // group (its latency overlaps the last issues), blocking wait only
                                         // if it failed; kFence & 256: commit every 32 MMAs
                if (tc::elect_one()) {
                    bool ok = true;
                    for (int g = 0; g < kReps / 16; ++g) {
                        if (!ok) tc::mbar_wait(&done_bar, 0);
                        const int r0 = 16 * g;
#pragma unroll
                        for (int u = 0; u < 12; ++u)
                            tc::mma_bf16(tm + 128 * (u & 1), ad + (uint64_t)(u & 7), bd + (uint64_t)((((r0 + u) >> 1) % 40) * 2 * N),
                                         idesc, (r0 + u) > 1 ? 1u : 0u);
                        if (!(kFence & 512)) ok = tc::mbar_test(&done_bar, 0);
#pragma unroll
                        for (int u = 12; u < 16; ++u)
                            tc::mma_bf16(tm + 128 * (u & 1), ad + (uint64_t)(u & 7), bd + (uint64_t)((((r0 + u) >> 1) % 40) * 2 * N),
                                         idesc, 1u);
                        if (!(kFence & 256) || (g & 1)) tc::commit(&dummy);
                    }
                    tc::commit(&bar);
                }
                __syncwarp();
            } else if (kFence & 8) {   // the same per-16 pattern from ONE lane (the kernels' current issue loop)
                if (tc::elect_one()) {
                    for (int r0 = 0; r0 < kReps; r0 += 16) {
                        if (kFence & 2) tc::mbar_wait(&done_bar, 0);
                        if (kFence & 4) tc::fence_after_sync();
                        if (kFence & 16) (void)tc::mbar_test(&dummy, 0);
                        for (int r = r0; r < r0 + 16 && r < kReps; ++r) {
                            if (kTs)
                                tc::mma_bf16_ts(tm + 256, tm + 8 * (r & 7), bd + (uint64_t)(((r >> 1) % 40) * 2 * N), idesc,
                                                r > 0 ? 1u : 0u);
                            else
                                tc::mma_bf16(tm + 128 * (r & 1), ad + (uint64_t)(r & 7), bd + (uint64_t)(((r >> 1) % 40) * 2 * N),
                                             idesc, r > 1 ? 1u : 0u);
                        }
                        tc::commit(&dummy);
                        if (kFence & 32) tc::commit(&dummy);
                    }
                    tc::commit(&bar);
                }
                __syncwarp();
            } else if (kFence) {   // the kernels' per-slice pattern: the whole warp waits on a (completed)
                           // barrier, fences, re-elects a lane and issues 16 MMAs
                for (int r0 = 0; r0 < kReps; r0 += 16) {
                    if (kFence & 2) tc::mbar_wait(&done_bar, 0);
                    if (kFence & 4) tc::fence_after_sync();
                    if (tc::elect_one()) {
                        for (int r = r0; r < r0 + 16 && r < kReps; ++r)
                            tc::mma_bf16(tm + 128 * (r & 1), ad + (uint64_t)(r & 7), bd + (uint64_t)(((r >> 1) % 40) * 2 * N),
                                         idesc, r > 1 ? 1u : 0u);
                        tc::commit(&dummy);
                    }
                    __syncwarp();
                }
                if (tc::elect_one()) tc::commit(&bar);
            } else if (tc::elect_one()) {
                for (int r = 0; r < kReps; ++r) {
                    if (kTs)
                        tc::mma_bf16_ts(tm + 256, tm + 8 * (r & 7), bd, idesc, r > 0 ? 1u : 0u);
                    else
                        tc::mma_bf16(kAltD ? tm + 128 * (r & 1) : tm + 256, kRot ? ad + (uint64_t)(r & 7) : ad,
                                     kBRot ? bd + (uint64_t)(((r >> (kAltD ? 1 : 0)) % 40) * 2 * N) : bd, idesc,
                                     r > (kAltD ? 1 : 0) ? 1u : 0u);
                    if (kCommit && (r % kCommit) == kCommit - 1) tc::commit(&dummy);
                }
                tc::commit(&bar);
            }
            __syncwarp();
            tc::mbar_wait(&bar, (uint32_t)pass);
            t1 = clock64();
        }
        if (tid == 0) out[blockIdx.x] = (t1 - t0);
    }
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<512>(tm);
}

template <int N, bool kTs, int kSwz, int kShift = 0, int kLbo16 = 0, int kRot = 0, int kBRot = 0, int kAltD = 0,
          int kCommit = 0, int kFence = 0>
void run(const char* what, int grid = 1) {
    long long* d;
    cudaMalloc(&d, 256 * sizeof(long long));
    cudaFuncSetAttribute(probe<N, kTs, kSwz, kShift, kLbo16, kRot, kBRot, kAltD, kCommit, kFence>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem);
    probe<N, kTs, kSwz, kShift, kLbo16, kRot, kBRot, kAltD, kCommit, kFence><<<grid, 128, kSmem>>>(d);
    cudaError_t e = cudaDeviceSynchronize();
    long long h = 0;
    cudaMemcpy(&h, d, sizeof h, cudaMemcpyDeviceToHost);
    const double floor_cyc = 128.0 * N / 256.0;
    printf("%-32s N=%3d grid %3d %7.1f cycles/MMA  (floor %5.1f)  %s\n", what, N, grid, (double)h / kReps, floor_cyc,
           e == cudaSuccess ? "" : cudaGetErrorString(e));
    cudaFree(d);
}

// Contention: warp 0 issues the MMAs (N = 128, A rotating over 8 shifts, B over 40 K-steps, two
// accumulators -- the U3 pattern) while warps 1..15 keep another SM unit busy until the MMAs finish:
// 1 = LDS.128 from shared memory outside the operands, 2 = LDG.128 hitting L1 (16 KB buffer),
// 3 = STS.128, 4 = FFMA chains, 5 = tcgen05.ld from TMEM columns the MMAs do not write, 6 = MUFU ex2.
// If the tensor core's operand reads share the shared-memory datapath, modes 1-3 slow the MMAs.
template <int kMode>
__global__ void contend(long long* out, const float4* g) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tm;
    __shared__ volatile int stop;
    constexpr int N = 128;
    uint8_t* A = sm;
    uint8_t* B = sm + 16384;
    const int tid = threadIdx.x, warp = tid >> 5;
    for (int i = tid; i < kSmem / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0x3c003c00u;
    if (warp == 0) tc::tmem_alloc<512>(&tm);
    if (tid == 0) {
        stop = 0;
        tc::mbar_init(&bar, 1);
        tc::mbar_fence_init();
    }
    tc::fence_proxy_async();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    float acc = 0.f;
    if (warp == 0) {
        const uint32_t idesc = tc::make_idesc_bf16(128, N);
        const uint64_t ad = tc::make_desc(tc::smem_u32(A), 2048u, 128);
        const uint64_t bd = tc::make_desc(tc::smem_u32(B), (uint32_t)(N * 16), 128);
        long long t0 = 0, t1 = 0;
        for (int pass = 0; pass < 2; ++pass) {
            __syncwarp();
            t0 = clock64();
            if (tc::elect_one()) {
                for (int r = 0; r < kReps; ++r)
                    tc::mma_bf16(tm + 128 * (r & 1), ad + (uint64_t)(r & 7), bd + (uint64_t)(((r >> 1) % 40) * 2 * N),
                                 idesc, r > 1 ? 1u : 0u);
                tc::commit(&bar);
            }
            __syncwarp();
            tc::mbar_wait(&bar, (uint32_t)pass);
            t1 = clock64();
        }
        if (tid == 0) { out[blockIdx.x] = t1 - t0; stop = 1; }
    } else if (kMode != 0) {
        // the busy warps: operands they touch lie above the MMA buffers (B spans 40 x 4 KB)
        const uint32_t base = tc::smem_u32(sm + 180 * 1024) + (uint32_t)((tid & 511) * 16 % 16384);
        uint32_t v0 = 0, v1 = 0, v2 = 0, v3 = 0;
        float f0 = (float)tid, f1 = 1.f, f2 = 2.f, f3 = 3.f;
        float t[16];
        while (!stop) {
#pragma unroll
            for (int k = 0; k < 16; ++k) {
                if (kMode == 1) {
                    uint32_t a0, a1, a2, a3;
                    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a0), "=r"(a1), "=r"(a2), "=r"(a3) : "r"(base ^ (k * 512)));
                    v0 ^= a0; v1 ^= a1; v2 ^= a2; v3 ^= a3;
                } else if (kMode == 2) {
                    const float4 x = __ldg(g + ((tid * 16 + k * 64) & 1023));
                    f0 += x.x; f1 += x.y; f2 += x.z; f3 += x.w;
                } else if (kMode == 3) {
                    asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" :: "r"(base ^ (k * 512)), "r"(v0), "r"(v1), "r"(v2), "r"(k) : "memory");
                } else if (kMode == 4) {
                    f0 = fmaf(f0, 1.0001f, 0.5f); f1 = fmaf(f1, 1.0001f, 0.5f);
                    f2 = fmaf(f2, 1.0001f, 0.5f); f3 = fmaf(f3, 1.0001f, 0.5f);
                } else if (kMode == 5) {
                    if (k == 0) {
                        tc::tmem_ld16_async(tm + 256 + ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)(16 * (warp >> 2)), t);
                        tc::tmem_wait_ld();
                        f0 += t[0] + t[15];
                    }
                } else if (kMode == 6) {
                    asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(f0));
                    asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(f1));
                }
            }
        }
        acc = f0 + f1 + f2 + f3 + (float)(v0 ^ v1 ^ v2 ^ v3);
    }
    if (acc == 12345.f) out[1 + blockIdx.x] = 1;   // keep the busy work live
    tc::fence_before_sync();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<512>(tm);
}

template <int kMode>
void run_contend(const char* what) {
    long long* d;
    float4* g;
    cudaMalloc(&d, 256 * sizeof(long long));
    cudaMalloc(&g, 1024 * sizeof(float4));
    cudaMemset(g, 0, 1024 * sizeof(float4));
    cudaFuncSetAttribute(contend<kMode>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem);
    contend<kMode><<<1, 512, kSmem>>>(d, g);
    cudaError_t e = cudaDeviceSynchronize();
    long long h = 0;
    cudaMemcpy(&h, d, sizeof h, cudaMemcpyDeviceToHost);
    printf("%-40s N=128 %7.1f cycles/MMA  (floor  64.0)  %s\n", what, (double)h / kReps,
           e == cudaSuccess ? "" : cudaGetErrorString(e));
    cudaFree(d);
    cudaFree(g);
}

int main(int argc, char** argv) {
    setvbuf(stdout, nullptr, _IONBF, 0);
    if (argc > 1) {   // the issue-loop variants only, one per invocation: umma_probe <k>
        switch (atoi(argv[1])) {
            case 0: run<128, false, 0, 0, 0, 1, 1, 1, 0, 8>("1 lane per-16: commit"); break;
            case 1: run<128, false, 0, 0, 0, 1, 1, 1, 0, 10>("1 lane per-16: + mbar wait"); break;
            case 2: run<128, true, 0, 0, 0, 0, 1, 0, 0, 8>("TS 1 lane per-16: commit"); break;
            case 3: run<128, true, 0, 0, 0, 0, 1, 0, 0, 10>("TS 1 lane per-16: + mbar wait"); break;
            case 4: run<128, false, 0, 0, 0, 1, 1, 1, 0, 26>("1 lane per-16: + wait + test"); break;
            case 5: run<32, false, 0, 0, 0, 1, 1, 1, 0, 8>("1 lane per-16: commit"); break;
            case 6: run<32, false, 0, 0, 0, 1, 1, 1, 0, 10>("1 lane per-16: + mbar wait"); break;
            case 9: run<32, false, 0, 0, 0, 1, 1, 1, 0, 128>("1 lane: early test, commit/16"); break;
            case 10: run<128, false, 0, 0, 0, 1, 1, 1, 0, 8 + 2>("1 lane: wait, commit/16 (=1)"); break;
            case 11: run<128, false, 0, 0, 0, 1, 1, 1, 0, 512 + 128>("1 lane: same loop, no test"); break;
        }
        return 0;
    }
    run<16, false, 0>("SS no-swizzle");
    run<32, false, 0>("SS no-swizzle");
    run<48, false, 0>("SS no-swizzle");
    run<64, false, 0>("SS no-swizzle");
    run<96, false, 0>("SS no-swizzle");
    run<128, false, 0>("SS no-swizzle");
    run<256, false, 0>("SS no-swizzle");
    run<64, true, 0>("TS (A in TMEM) no-swizzle B");
    run<96, true, 0>("TS (A in TMEM) no-swizzle B");
    run<128, true, 0>("TS (A in TMEM) no-swizzle B");
    run<256, true, 0>("TS (A in TMEM) no-swizzle B");
    run<64, false, 32>("SS 32B-swizzle");
    run<128, false, 32>("SS 32B-swizzle");
    run<256, false, 32>("SS 32B-swizzle");
    run<128, false, 0, 1>("SS A shifted 1 row");
    run<128, false, 0, 3>("SS A shifted 3 rows");
    run<128, false, 0, 8>("SS A shifted 8 rows");
    run<128, false, 0, 0, 1>("SS A LBO=16 (next pixel)");
    run<128, false, 0, 1, 1>("SS A shift 1, LBO=16");
    run<128, false, 0, 0, 0, 1>("SS A rotating shifts");
    run<32, false, 0, 1>("SS A shifted 1 row");
    run<48, false, 0, 1>("SS A shifted 1 row");
    run<48, false, 0, 0, 0, 1>("SS A rotating shifts");
    run<128, false, 0, 0, 0, 1, 1>("SS A rot, B over 40 K-steps");
    run<64, false, 0, 0, 0, 1, 1>("SS A rot, B over 40 K-steps");
    run<48, false, 0, 0, 0, 1, 1>("SS A rot, B over 40 K-steps");
    run<96, true, 0, 0, 0, 0, 1>("TS, B over 40 K-steps");
    run<128, false, 0, 0, 0, 1, 1, 1>("SS A rot, B rot, 2 accumulators");
    run<128, false, 0, 0, 0, 1, 1, 1>("SS A rot, B rot, 2 accumulators", 148);
    run<128, false, 0, 0, 0, 1, 1, 0>("SS A rot, B rot", 148);
    run<128, false, 0, 0, 0, 1, 1, 1, 16>("SS 2 acc, commit every 16");
    run<128, false, 0, 0, 0, 1, 1, 1, 4>("SS 2 acc, commit every 4");
    run<128, false, 0, 0, 0, 1, 1, 1, 1>("SS 2 acc, commit every MMA");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 1>("per-16: elect+syncwarp+commit");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 3>("per-16: + mbar wait");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 5>("per-16: + fence");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 7>("per-16: + wait + fence");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 64>("warp-1 wait, bar.sync handoff");
    run<128, true, 0, 0, 0, 0, 1, 0, 0, 8>("TS 1 lane per-16: commit");
    run<128, true, 0, 0, 0, 0, 1, 0, 0, 10>("TS 1 lane per-16: + mbar wait");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 8>("1 lane per-16: commit");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 10>("1 lane per-16: + mbar wait");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 14>("1 lane per-16: + wait + fence");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 30>("1 lane per-16: + wait + fence + test");
    run<128, false, 0, 0, 0, 1, 1, 1, 0, 62>("1 lane per-16: + 2 commits");
    run<32, false, 0, 0, 0, 1, 1, 1, 0, 8>("1 lane per-16: commit");
    run<32, false, 0, 0, 0, 1, 1, 1, 0, 62>("1 lane per-16: all");
    run<32, false, 0, 0, 0, 1, 1, 1>("2 acc, no sync");
    run_contend<0>("contend: idle warps");
    run_contend<1>("contend: 15 warps LDS.128");
    run_contend<2>("contend: 15 warps LDG.128 (L1 hit)");
    run_contend<3>("contend: 15 warps STS.128");
    run_contend<4>("contend: 15 warps FFMA");
    run_contend<5>("contend: 15 warps tcgen05.ld");
    run_contend<6>("contend: 15 warps MUFU");
    return 0;
}
