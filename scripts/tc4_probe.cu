// tc4_probe.cu -- measurements and layout checks for the 4-step tensor kernel (not part of the product).
//   peak_i8      : sustained tcgen05.mma kind::i8 rate, one CTA per SM, MMAs issued back to back
//                  (no per-tile wait), M=128 x N x K=32 -> the int8 denominator of roofline_tensor
//   sw64_check   : TMA (CU_TENSOR_MAP_SWIZZLE_64B) loads a [128 rows][64 B] K-major operand tile that
//                  an MMA reads through a SWIZZLE_64B smem descriptor; D compared with the host product.
//                  Variant 1: box (16 words, 128 rows); variant 2: box (8 words, 2 halves, 128 rows)
//                  (two 32-byte pieces of one 64-byte K row, the forward row-pass operand of tc4)
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

#define DEVI __device__ __forceinline__

DEVI uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
DEVI uint64_t desc_none(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | ((uint64_t)1 << 46);
}
DEVI uint64_t desc_sw64(uint32_t saddr) {      // K-major SWIZZLE_64B: 8-row atoms of 512 B (SBO), LBO unused
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)(512 >> 4) << 32) |
           ((uint64_t)1 << 46) | ((uint64_t)4 << 61);
}
__host__ __device__ constexpr uint32_t idesc_i8(int M, int N) {
    return (2u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
DEVI void mma_i8(uint32_t d, uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
                 :: "r"(d), "l"(a), "l"(b), "r"(id), "r"(acc));
}
DEVI void commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(smem_u32(bar)) : "memory");
}
DEVI void mbar_init(uint64_t* bar, uint32_t n) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(n)); }
DEVI void mbar_wait(uint64_t* bar, uint32_t ph) {
    asm volatile("{\n\t.reg .pred P1;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t@!P1 bra W_%=;\n\t}\n"
                 :: "r"(smem_u32(bar)), "r"(ph) : "memory");
}
DEVI void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
DEVI void tma_load_2d(void* dst, const CUtensorMap* m, int c0, int c1, uint64_t* bar) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 :: "r"(smem_u32(dst)), "l"(m), "r"(c0), "r"(c1), "r"(smem_u32(bar)) : "memory");
}
DEVI void tma_load_3d(void* dst, const CUtensorMap* m, int c0, int c1, int c2, uint64_t* bar) {
    asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                 :: "r"(smem_u32(dst)), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(bar)) : "memory");
}
DEVI void tma_load_5d(void* dst, const CUtensorMap* m, int c0, int c1, int c2, int c3, int c4, uint64_t* bar) {
    asm volatile("cp.async.bulk.tensor.5d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 :: "r"(smem_u32(dst)), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "r"(smem_u32(bar)) : "memory");
}
DEVI void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
DEVI void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
DEVI void tmem_ld32(uint32_t taddr, uint32_t* r) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 "
                 "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                 "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
                   "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
                   "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                 : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// ------------------------------------------------------------------------------------ int8 peak
template <int N>
__global__ void __launch_bounds__(128, 1) k_peak(int iters, uint32_t* sink) {
    extern __shared__ __align__(1024) uint8_t sm[];
    uint8_t* sA = sm;                 // 128 x 32 B
    uint8_t* sB = sm + 4096;          // N x 32 B
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tslot;
    const int t = threadIdx.x;
    for (int i = t; i < 4096 + N * 32; i += 128) sm[i] = (uint8_t)(i * 7 + 1);
    if (t == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
    if (t < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(smem_u32(&tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    fence_before(); __syncthreads(); fence_after();
    const uint32_t tm = tslot;
    if (t == 0) {
        const uint64_t da = desc_none(smem_u32(sA), 128, 256), db = desc_none(smem_u32(sB), 128, 256);
        const uint32_t id = idesc_i8(128, N);
        for (int i = 0; i < iters; ++i) mma_i8(tm + (uint32_t)((i & 1) * N), da, db, id, i > 1);
        commit(&bar);
    }
    mbar_wait(&bar, 0);
    fence_after();
    uint32_t r[32];
    tmem_ld32(tm + ((uint32_t)((t >> 5) * 32) << 16), r);
    sink[blockIdx.x * 128 + t] = r[0] ^ r[31];
    fence_before(); __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tm));
}

extern "C" float peak_i8(int n, int blocks, int iters) {
    uint32_t* sink; cudaMalloc(&sink, blocks * 128 * 4);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const int smem = 4096 + n * 32;
    auto launch = [&]() {
        if (n == 256) k_peak<256><<<blocks, 128, smem>>>(iters, sink);
        else if (n == 128) k_peak<128><<<blocks, 128, smem>>>(iters, sink);
        else k_peak<64><<<blocks, 128, smem>>>(iters, sink);
    };
    launch(); cudaDeviceSynchronize();
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
        cudaEventRecord(a); launch(); cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
    }
    int e = (int)cudaGetLastError();
    cudaFree(sink); cudaEventDestroy(a); cudaEventDestroy(b);
    return e ? -(float)e : best;
}

// ------------------------------------------------------------------------------- SW64 TMA -> UMMA
__device__ __forceinline__ uint32_t aoff_none(int m, int k) { return (m & 7) * 16 + (m >> 3) * 512 + (k >> 4) * 128 + (k & 15); }

__global__ void __launch_bounds__(128) k_sw64(const __grid_constant__ CUtensorMap tmap, int variant, int e,
                                              const uint8_t* Bg, int32_t* D, uint8_t* Adump) {
    __shared__ __align__(1024) uint8_t sA[128 * 64];
    __shared__ __align__(1024) uint8_t sB[64 * 64];
    __shared__ __align__(8) uint64_t bar[2];
    __shared__ uint32_t tslot;
    const int t = threadIdx.x;
    for (int i = t; i < 64 * 64; i += 128) sB[aoff_none(i / 64, i % 64)] = Bg[i];   // B given [n][k]
    if (t == 0) { mbar_init(&bar[0], 1); mbar_init(&bar[1], 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
    if (t < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" :: "r"(smem_u32(&tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    fence_before(); __syncthreads(); fence_after();
    if (t == 0) {
        mbar_expect_tx(&bar[0], 128 * 64);
        if (variant == 1) tma_load_2d(sA, &tmap, 0, 0, &bar[0]);
        else if (variant == 2) tma_load_3d(sA, &tmap, 8 * e, 0, 0, &bar[0]);
        else tma_load_5d(sA, &tmap, 8 * e, 0, 0, 0, 0, &bar[0]);
    }
    mbar_wait(&bar[0], 0);
    for (int i = t; i < 128 * 64; i += 128) Adump[i] = sA[i];
    fence_before(); __syncthreads(); fence_after();
    const uint32_t tm = tslot;
    if (t == 0) {
        const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB);
        const uint32_t id = idesc_i8(128, 64);
        if (variant == 3) {           // SWIZZLE_NONE canonical: LBO 128 (K core matrices), SBO 512 (8-row groups)
            mma_i8(tm, desc_none(a0, 128, 512), desc_none(b0, 128, 512), id, 0);
            mma_i8(tm, desc_none(a0 + 256, 128, 512), desc_none(b0 + 256, 128, 512), id, 1);
        } else {
            mma_i8(tm, desc_sw64(a0), desc_none(b0, 128, 512), id, 0);
            mma_i8(tm, desc_sw64(a0 + 32), desc_none(b0 + 256, 128, 512), id, 1);
        }
        commit(&bar[1]);
    }
    mbar_wait(&bar[1], 0);
    fence_after();
    uint32_t r[32];
    for (int h = 0; h < 2; ++h) {
        tmem_ld32(tm + ((uint32_t)((t >> 5) * 32) << 16) + 32 * h, r);
        for (int c = 0; c < 32; ++c) D[t * 64 + 32 * h + c] = (int32_t)r[c];
    }
    fence_before(); __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" :: "r"(tm));
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// G: [128 rows][256 words] u32 (row stride 1 KB).  variant 1: A[m] = words [m][0..16);
// variant 2: A[m] = words [m][8e..8e+8) ++ [m][128+8e..128+8e+8).  Returns 0 or an error code.
extern "C" int sw64_check(int variant, int e, const uint32_t* hG, const uint8_t* hB, int32_t* hD, uint8_t* hAdump) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) return 1001;
    EncodeFn enc = (EncodeFn)fn;
    uint32_t* dG; uint8_t* dB; int32_t* dD; uint8_t* dA;
    cudaMalloc(&dG, 128 * 1024); cudaMalloc(&dB, 4096); cudaMalloc(&dD, 128 * 64 * 4); cudaMalloc(&dA, 8192);
    cudaMemcpy(dG, hG, 128 * 1024, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB, 4096, cudaMemcpyHostToDevice);
    alignas(64) CUtensorMap m;
    CUresult r;
    if (variant == 1) {
        cuuint64_t dims[2] = {256, 128}, strides[1] = {1024};
        cuuint32_t box[2] = {16, 128}, es[2] = {1, 1};
        r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, dG, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    } else if (variant == 3) {
        // (w4: 4 words, row8: 8 rows, kc_lo: 2, h: 2, rg: 16) -> smem [rg][h][kc_lo][row8][w4]: the
        // SWIZZLE_NONE K-major canonical layout (core matrix 8 rows x 16 B, LBO 128 B, SBO 512 B);
        // the word at dim-0 coordinate c0 + w4 + 4 kc_lo + 128 h of row 8 rg + row8
        cuuint64_t dims[5] = {128, 8, 2, 2, 16}, strides[4] = {1024, 16, 512, 8192};
        cuuint32_t box[5] = {4, 8, 2, 2, 16}, es[5] = {1, 1, 1, 1, 1};
        r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 5, dG, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    } else {
        cuuint64_t dims[3] = {128, 2, 128}, strides[2] = {512, 1024};
        cuuint32_t box[3] = {8, 2, 128}, es[3] = {1, 1, 1};
        r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 3, dG, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    }
    if (r != CUDA_SUCCESS) return 2000 + (int)r;
    k_sw64<<<1, 128>>>(m, variant, e, dB, dD, dA);
    int err = (int)cudaDeviceSynchronize();
    cudaMemcpy(hD, dD, 128 * 64 * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(hAdump, dA, 8192, cudaMemcpyDeviceToHost);
    cudaFree(dG); cudaFree(dB); cudaFree(dD); cudaFree(dA);
    return err;
}
