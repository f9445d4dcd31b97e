// tma.cuh -- mbarrier + TMA (cp.async.bulk.tensor) helpers for the CUDA-core kernels (v8's TMA-fed
// column phase).  The tcgen05 kernel keeps its own set in ntt_tc4.cuh (namespace wd::tc4).
#pragma once
#include <cuda.h>
#include <cstdint>

namespace wd {

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(b)), "r"(n));
}
__device__ __forceinline__ void mb_init_fence() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void mb_wait(uint64_t* b, uint32_t parity) {
#ifdef WD_TM_DEBUG
    // debug builds: trap instead of hanging when a phase never completes (~2 s at B200 clocks)
    const long long t0 = clock64();
    for (;;) {
        uint32_t ok;
        asm volatile("{\n\t.reg .pred P1;\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
                     "selp.u32 %0, 1, 0, P1;\n\t}" : "=r"(ok) : "r"(smem_u32(b)), "r"(parity) : "memory");
        if (ok) break;
        if (clock64() - t0 > (1LL << 32)) __trap();
    }
#else
    asm volatile("{\n\t.reg .pred P1;\n\tMBW_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
                 "@!P1 bra MBW_%=;\n\t}\n" :: "r"(smem_u32(b)), "r"(parity) : "memory");
#endif
}
__device__ __forceinline__ void mb_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mb_expect(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(b)), "r"(bytes) : "memory");
}
// generic-proxy accesses to a buffer before this point are ordered before later async-proxy (TMA) writes
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
// this thread's generic-proxy global writes are ordered before later async-proxy (TMA) reads of them
// (after a barrier that makes them visible to the issuing thread)
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ void tma2_load(void* dst, const CUtensorMap* m, int c0, int c1, uint64_t* b) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
                 " [%0], [%1, {%2, %3}], [%4];"
                 :: "r"(smem_u32(dst)), "l"(m), "r"(c0), "r"(c1), "r"(smem_u32(b)) : "memory");
}
// an L2 policy that marks the lines a load brings in as first to evict (streamed, read-once input):
// keeps them from displacing the L2-resident intermediates (the register loads they replace were
// ld.global.cs)
__device__ __forceinline__ uint64_t l2_evict_first_policy() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void tma2_load_hint(void* dst, const CUtensorMap* m, int c0, int c1, uint64_t* b, uint64_t pol) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
                 " [%0], [%1, {%2, %3}], [%4], %5;"
                 :: "r"(smem_u32(dst)), "l"(m), "r"(c0), "r"(c1), "r"(smem_u32(b)), "l"(pol) : "memory");
}
__device__ __forceinline__ void tma3_load_hint(void* dst, const CUtensorMap* m, int c0, int c1, int c2, uint64_t* b,
                                               uint64_t pol) {
    asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
                 " [%0], [%1, {%2, %3, %4}], [%5], %6;"
                 :: "r"(smem_u32(dst)), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(b)), "l"(pol) : "memory");
}
}  // namespace wd
