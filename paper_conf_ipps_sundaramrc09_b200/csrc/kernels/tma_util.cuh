// tma_util.cuh -- shared helpers for kernels that stage tiles with the TMA engine
// (cp.async.bulk.tensor) into shared memory, completing on an mbarrier. Product code.
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>

namespace tg {

// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda); nullptr if
// unavailable (callers then take their non-TMA path). Defined in edge.cu.
PFN_cuTensorMapEncodeTiled_v12000 tma_encode_fn();

// Encode a 3-D fp32 tensor map: dims {d0 (contiguous), d1, d2}, byte strides of d1 and d2,
// box {b0, b1, b2}; out-of-bounds elements of a box are filled with zeros.
inline bool tma_make_3d(CUtensorMap* m, const void* base, uint64_t d0, uint64_t d1, uint64_t d2, uint64_t s1,
                        uint64_t s2, uint32_t b0, uint32_t b1, uint32_t b2) {
    PFN_cuTensorMapEncodeTiled_v12000 enc = tma_encode_fn();
    if (!enc) return false;
    const cuuint64_t gdim[3] = {d0, d1, d2};
    const cuuint64_t gstride[2] = {s1, s2};
    const cuuint32_t box[3] = {b0, b1, b2};
    const cuuint32_t estride[3] = {1, 1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<void*>(base), gdim, gstride, box, estride,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

__device__ __forceinline__ uint32_t tma_smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void tma_mbar_init(uint64_t* mbar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(tma_smem_u32(mbar)), "r"(count) : "memory");
}
__device__ __forceinline__ void tma_fence_init() { asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory"); }
__device__ __forceinline__ void tma_expect_tx(uint64_t* mbar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(tma_smem_u32(mbar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void tma_wait(uint64_t* mbar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred done;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 done, [%0], %1;\n\t"
        "@!done bra WAIT_%=;\n\t}\n" ::"r"(tma_smem_u32(mbar)),
        "r"(parity)
        : "memory");
}
// box origin (x, y, z) in elements; x * 4 bytes must be a multiple of 16
__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, int x, int y, int z, uint64_t* mbar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], "
        "[%5];\n" ::"r"(tma_smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(z), "r"(tma_smem_u32(mbar))
        : "memory");
}
__device__ __forceinline__ void tma_prefetch_map(const CUtensorMap* map) {
    asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

}  // namespace tg
