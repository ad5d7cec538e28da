// Probe: cp.async.bulk (1-D, global -> shared) throughput per SM on B200 as a function of copy size and
// copies in flight. One CTA per SM (148), one thread issues copies into a ring of NBUF slots; the
// same thread waits for slot completion before reusing it. Source: a 64 MB buffer (L2-resident after
// warm-up) or 1 GB (HBM). Prints GB/s aggregate and bytes/cycle/SM.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/bcp bulk_copy_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sm32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void probe(const uint8_t* src, size_t src_bytes, int copy_bytes, int nbuf, int copies_per_cta, int ncopy_per_slot) {
    extern __shared__ __align__(128) uint8_t sm[];
    __shared__ __align__(8) uint64_t bar[16];
    if (threadIdx.x != 0) return;
    for (int i = 0; i < nbuf; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sm32(&bar[i])));
    asm volatile("fence.mbarrier_init.release.cluster;");
    const uint32_t mask = (uint32_t)(src_bytes / copy_bytes) - 1;  // power of two
    uint32_t pos = blockIdx.x * 977u;
    const int slot_bytes = copy_bytes * ncopy_per_slot;
    for (int k = 0; k < copies_per_cta; ++k) {
        const int b = k % nbuf;
        if (k >= nbuf) {
            const uint32_t par = ((k / nbuf) - 1) & 1;
            asm volatile("{.reg .pred p; W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W;}" ::"r"(sm32(&bar[b])), "r"(par));
        }
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sm32(&bar[b])), "r"(slot_bytes));
        for (int c = 0; c < ncopy_per_slot; ++c) {
            pos = (pos + 7919u) & mask;
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             sm32(sm + (size_t)b * slot_bytes + (size_t)c * copy_bytes)),
                         "l"(src + (size_t)pos * copy_bytes), "r"(copy_bytes), "r"(sm32(&bar[b])));
        }
    }
    for (int k = copies_per_cta; k < copies_per_cta + nbuf; ++k) {
        const int b = k % nbuf;
        const uint32_t par = ((k / nbuf) - 1) & 1;
        if (k - nbuf >= 0)
            asm volatile("{.reg .pred p; W2: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W2;}" ::"r"(sm32(&bar[b])), "r"(par));
    }
}

int main() {
    size_t big = 1ull << 30;
    uint8_t* src;
    cudaMalloc(&src, big);
    cudaMemset(src, 1, big);
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (size_t srcb : {(size_t)64 << 20, big}) {
        for (int cb : {2048, 4096, 16384, 32768}) {
            for (int per_slot : {1, 6}) {
                for (int nbuf : {2, 4, 8}) {
                    const int slot = cb * per_slot;
                    if ((size_t)slot * nbuf > 190 * 1024) continue;
                    const int n = (int)std::max<long>(64, (long)(256ll << 20) / sms / slot);
                    probe<<<sms, 32, slot * nbuf>>>(src, srcb, cb, nbuf, n, per_slot);
                    cudaEventRecord(e0);
                    probe<<<sms, 32, slot * nbuf>>>(src, srcb, cb, nbuf, n, per_slot);
                    cudaEventRecord(e1);
                    cudaEventSynchronize(e1);
                    float ms = 0;
                    cudaEventElapsedTime(&ms, e0, e1);
                    const double bytes = (double)sms * n * slot;
                    printf("src %4zu MB copy %6d B x%d per slot, %d slots: %7.1f GB/s  %6.1f B/clk/SM\n", srcb >> 20, cb,
                           per_slot, nbuf, bytes / ms / 1e6, bytes / (ms * 1e-3) / (clk * 1e3) / sms);
                }
            }
        }
    }
    cudaError_t e = cudaGetLastError();
    printf("err %s\n", cudaGetErrorString(e));
}
