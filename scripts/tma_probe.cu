// tma_probe.cu -- TMA throughput by box shape (not part of the product).  One CTA per SM, one thread
// streams 8 KB tiles through a ring of NS slots (loads: mbarrier complete_tx; stores: bulk groups).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>

#define DEVI __device__ __forceinline__
DEVI uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
DEVI void bar_init(uint64_t* b, uint32_t n) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(sa(b)), "r"(n)); }
DEVI void bar_wait(uint64_t* b, uint32_t ph) {
    asm volatile("{\n\t.reg .pred P1;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n\t@!P1 bra W_%=;\n\t}\n"
                 :: "r"(sa(b)), "r"(ph), "r"(1000000) : "memory");
}
DEVI void bar_expect(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(sa(b)), "r"(n) : "memory");
}
DEVI void ld2(void* d, const CUtensorMap* m, int c0, int c1, uint64_t* b) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 :: "r"(sa(d)), "l"(m), "r"(c0), "r"(c1), "r"(sa(b)) : "memory");
}
DEVI void ld3(void* d, const CUtensorMap* m, int c0, int c1, int c2, uint64_t* b) {
    asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                 :: "r"(sa(d)), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(sa(b)) : "memory");
}
DEVI void ld5(void* d, const CUtensorMap* m, int c0, int c1, int c2, int c3, int c4, uint64_t* b) {
    asm volatile("cp.async.bulk.tensor.5d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 :: "r"(sa(d)), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "r"(sa(b)) : "memory");
}
DEVI void ld1(void* d, const void* src, uint32_t n, uint64_t* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(sa(d)), "l"(src), "r"(n), "r"(sa(b)) : "memory");
}
DEVI void st2(const CUtensorMap* m, int c0, int c1, const void* s) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.tile.bulk_group [%0, {%1, %2}], [%3];"
                 :: "l"(m), "r"(c0), "r"(c1), "r"(sa(s)) : "memory");
}
DEVI void st1(void* dst, const void* s, uint32_t n) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" :: "l"(dst), "r"(sa(s)), "r"(n) : "memory");
}

constexpr int NS = 8, TB = 8192;

// mode: 0 = 2D (128 w x 16 rows), 1 = 2D (16 w x 128 rows, SW64), 2 = 3D (8 w x 128 rows x 2, SW32),
//       3 = 5D canonical (16-B rows), 4 = 1D bulk 8 KB
//       10 = store 2D (128 x 16), 11 = store 2D (16 x 128, SW64), 12 = store 2D (32 x 128, SW128: 16 KB),
//       14 = store 1D bulk 8 KB
__global__ void __launch_bounds__(32, 1) k_tma(const __grid_constant__ CUtensorMap m, uint32_t* g, int mode, int tiles,
                                               uint32_t rows_total) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t bar[NS];
    if (threadIdx.x != 0) return;
    for (int i = 0; i < NS; ++i) bar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    const uint32_t cta = blockIdx.x;
    for (int t = 0; t < tiles; ++t) {
        const int s = t % NS;
        // the tile's rows: 128 matrix rows per 8 KB (row = 1 KB wide buffer); spread CTAs and tiles
        const uint32_t tile = (cta * tiles + t) % (rows_total / 128);
        const int r0 = (int)(tile * 128);
        uint8_t* dst = sm + s * 16384;
        if (mode < 10) {
            if (t >= NS) bar_wait(&bar[s], ((t / NS) - 1) & 1);
            bar_expect(&bar[s], TB);
            switch (mode) {
                case 0: ld2(dst, &m, 0, r0 / 8, &bar[s]); break;          // 128 words x 16 rows = 8 KB
                case 1: ld2(dst, &m, 0, r0, &bar[s]); break;              // 16 words x 128 rows
                case 2: ld3(dst, &m, 0, r0, 0, &bar[s]); break;           // 8 words x 128 rows x 2
                case 3: ld5(dst, &m, 0, 0, 0, 0, r0 / 8, &bar[s]); break;
                default: ld1(dst, g + (size_t)r0 * 256, TB, &bar[s]); break;
            }
        } else {
            if (t >= NS) asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(NS - 1) : "memory");
            switch (mode) {
                case 10: st2(&m, 0, r0 / 8, dst); break;
                case 11: st2(&m, 0, r0, dst); break;
                case 12: st2(&m, 0, r0, dst); break;
                default: st1(g + (size_t)r0 * 256, dst, TB); break;
            }
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
    }
    if (mode < 10) {
        for (int t = tiles - NS; t < tiles; ++t) if (t >= 0) bar_wait(&bar[t % NS], (t / NS) & 1);
    } else {
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// buffer of rows_total rows x 256 words; returns ms (negative = error)
extern "C" float tma_probe(int mode, int ctas, int tiles, uint32_t rows_total) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) return -1;
    EncodeFn enc = (EncodeFn)fn;
    uint32_t* g = nullptr;
    if (cudaMalloc(&g, (size_t)rows_total * 1024) != cudaSuccess) return -2;
    cudaMemset(g, 1, (size_t)rows_total * 1024);
    alignas(64) CUtensorMap m;
    cuuint32_t es[5] = {1, 1, 1, 1, 1};
    CUresult r = CUDA_SUCCESS;
    const int md = mode % 10;
    if (md == 0) {
        cuuint64_t d[2] = {256, rows_total}, st[1] = {1024}; cuuint32_t b[2] = {128, 16};
        r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, g, d, st, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    } else if (md == 1) {
        cuuint64_t d[2] = {256, rows_total}, st[1] = {1024}; cuuint32_t b[2] = {16, 128};
        r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, g, d, st, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B,
                CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    } else if (md == 2 && mode < 10) {
        cuuint64_t d[3] = {128, rows_total, 2}, st[2] = {1024, 512}; cuuint32_t b[3] = {8, 128, 2};
        r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 3, g, d, st, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B,
                CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    } else if (md == 2) {
        cuuint64_t d[2] = {256, rows_total}, st[1] = {1024}; cuuint32_t b[2] = {32, 128};
        r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, g, d, st, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    } else if (md == 3) {
        cuuint64_t d[5] = {128, 8, 2, 2, rows_total / 8}, st[4] = {1024, 16, 512, 8192}; cuuint32_t b[5] = {4, 8, 2, 2, 16};
        r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 5, g, d, st, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    }
    if (r != CUDA_SUCCESS) { cudaFree(g); return -1000 - (float)r; }
    cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, NS * 16384);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    k_tma<<<ctas, 32, NS * 16384>>>(m, g, mode, tiles, rows_total);
    cudaDeviceSynchronize();
    cudaEventRecord(a);
    k_tma<<<ctas, 32, NS * 16384>>>(m, g, mode, tiles, rows_total);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0; cudaEventElapsedTime(&ms, a, b);
    int e = (int)cudaGetLastError();
    cudaFree(g); cudaEventDestroy(a); cudaEventDestroy(b);
    return e ? -(float)e : ms;
}
