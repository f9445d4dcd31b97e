// tc_probe.cu -- microbenchmarks / layout probes for the tensor path (not part of the product).
//   probe_mma        : one tcgen05.mma kind::i8 (M=128,N=64,K=64) with K-major SWIZZLE_NONE
//                      operands; returns D for a host-side check of the descriptor layout.
//   probe_mma_loop   : throughput of MMA(128x64x64) + tcgen05.ld epilogue loop, many CTAs
//   probe_ldtm_loop  : throughput of tcgen05.ld 32x32b.x64 alone
//   probe_int_loop   : Shoup-butterfly integer throughput
//   probe_copy       : global copy kernel (L2-resident or HBM-sized buffers)
#include <cuda_runtime.h>
#include <cstdint>

#define DEVI __device__ __forceinline__

DEVI uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

DEVI uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= (uint64_t)1 << 46;                      // version = 1 (sm100)
    return d;                                    // base_offset 0, lbo_mode 0, layout SWIZZLE_NONE
}

// kind::i8 : c_format S32 (2) at [4,6); a/b format u8 (0); K-major; N>>3 at [17,23); M>>4 at [24,29)
__host__ __device__ constexpr uint32_t idesc_i8(int M, int N) {
    return (2u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

DEVI void mma_i8(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
        :: "r"(tmem_d), "l"(da), "l"(db), "r"(idesc), "r"(acc));
}
DEVI void mma_i8_mask(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc,
                      uint32_t m0, uint32_t m1, uint32_t m2, uint32_t m3) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, {%5, %6, %7, %8}, p;\n\t}\n"
        :: "r"(tmem_d), "l"(da), "l"(db), "r"(idesc), "r"(acc), "r"(m0), "r"(m1), "r"(m2), "r"(m3));
}
DEVI void mma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                 :: "r"(smem_u32(bar)) : "memory");
}
DEVI void mbar_init(uint64_t* bar, uint32_t cnt) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(cnt));
}
DEVI void mbar_wait(uint64_t* bar, uint32_t phase) {
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra WAIT_%=;\n\t}\n" :: "r"(smem_u32(bar)), "r"(phase) : "memory");
}
DEVI void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
DEVI void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
DEVI void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

template <int NC>
DEVI void tmem_alloc(uint32_t* dst_smem) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                 :: "r"(smem_u32(dst_smem)), "n"(NC));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
}
template <int NC>
DEVI void tmem_free(uint32_t taddr) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(taddr), "n"(NC));
}

// 32 lanes x 32 columns (32-bit): thread t of the warp gets lane (base_lane + t), columns c..c+31
DEVI void tmem_ld32(uint32_t taddr, uint32_t* r) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}
DEVI void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// A: 128 x 64 bytes (row m, byte k) canonical K-major no-swizzle: (m%8)*16 + (m/8)*SBO + (k/16)*LBO + k%16
// LBO = 128, SBO = 512.  B: 64(N) x 64(K) bytes, same form (n plays m).
constexpr uint32_t LBO = 128, SBO = 512;
DEVI uint32_t aoff(int m, int k) { return (m & 7) * 16 + (m >> 3) * SBO + (k >> 4) * LBO + (k & 15); }

extern "C" __global__ void k_probe_mma(const uint8_t* A, const uint8_t* B, int32_t* D) {
    __shared__ __align__(1024) uint8_t sA[128 * 64];
    __shared__ __align__(1024) uint8_t sB[64 * 64];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t taddr_s;
    const int t = threadIdx.x;
    for (int i = t; i < 128 * 64; i += blockDim.x) sA[aoff(i / 64, i % 64)] = A[i];
    for (int i = t; i < 64 * 64; i += blockDim.x) sB[aoff(i / 64, i % 64)] = B[i];   // B given as [n][k]
    if (t == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
    if (t < 32) tmem_alloc<64>(&taddr_s);
    fence_proxy_async();
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = taddr_s;
    if (t == 0) {
        const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB);
        const uint32_t id = idesc_i8(128, 64);
        mma_i8(tmem, make_desc(a0, LBO, SBO), make_desc(b0, LBO, SBO), id, 0);
        mma_i8(tmem, make_desc(a0 + 2 * LBO, LBO, SBO), make_desc(b0 + 2 * LBO, LBO, SBO), id, 1);
        mma_commit(&bar);
    }
    mbar_wait(&bar, 0);
    fence_after();
    uint32_t r[32];
    const int warp = t >> 5;
    for (int half = 0; half < 2; ++half) {
        tmem_ld32(tmem + ((warp * 32) << 16) + half * 32, r);
        tmem_wait_ld();
        for (int c = 0; c < 32; ++c) D[t * 64 + half * 32 + c] = (int32_t)r[c];
    }
    fence_before();
    __syncthreads();
    if (t < 32) tmem_free<64>(tmem);
}

// masked: 4 B matrices (64x64 each, [g][n][k]); MMA g writes only lanes 32g..32g+31 (mask bit 1 = disabled?)
extern "C" __global__ void k_probe_mask(const uint8_t* A, const uint8_t* B4, int32_t* D) {
    __shared__ __align__(1024) uint8_t sA[128 * 64];
    __shared__ __align__(1024) uint8_t sB[4][64 * 64];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t taddr_s;
    const int t = threadIdx.x;
    for (int i = t; i < 128 * 64; i += blockDim.x) sA[aoff(i / 64, i % 64)] = A[i];
    for (int g = 0; g < 4; ++g)
        for (int i = t; i < 64 * 64; i += blockDim.x) sB[g][aoff(i / 64, i % 64)] = B4[g * 4096 + i];
    if (t == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
    if (t < 32) tmem_alloc<64>(&taddr_s);
    fence_proxy_async();
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = taddr_s;
    if (t == 0) {
        const uint32_t a0 = smem_u32(sA);
        const uint32_t id = idesc_i8(128, 64);
        for (int g = 0; g < 4; ++g) {
            const uint32_t b0 = smem_u32(sB[g]);
            uint32_t m[4] = {0xffffffffu, 0xffffffffu, 0xffffffffu, 0xffffffffu};
            m[g] = 0;
            mma_i8_mask(tmem, make_desc(a0, LBO, SBO), make_desc(b0, LBO, SBO), id, 0, m[0], m[1], m[2], m[3]);
            mma_i8_mask(tmem, make_desc(a0 + 2 * LBO, LBO, SBO), make_desc(b0 + 2 * LBO, LBO, SBO), id, 1,
                        m[0], m[1], m[2], m[3]);
        }
        mma_commit(&bar);
    }
    mbar_wait(&bar, 0);
    fence_after();
    uint32_t r[32];
    const int warp = t >> 5;
    for (int half = 0; half < 2; ++half) {
        tmem_ld32(tmem + ((warp * 32) << 16) + half * 32, r);
        tmem_wait_ld();
        for (int c = 0; c < 32; ++c) D[t * 64 + half * 32 + c] = (int32_t)r[c];
    }
    fence_before();
    __syncthreads();
    if (t < 32) tmem_free<64>(tmem);
}

// A from TMEM: lane m holds row m; K bytes 4c..4c+3 in TMEM column c (little-endian, assumed)
extern "C" __global__ void k_probe_tmem_a(const uint8_t* A, const uint8_t* B, int32_t* D) {
    __shared__ __align__(1024) uint8_t sB[64 * 64];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t taddr_s;
    const int t = threadIdx.x, warp = t >> 5;
    for (int i = t; i < 64 * 64; i += blockDim.x) sB[aoff(i / 64, i % 64)] = B[i];
    if (t == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
    if (t < 32) tmem_alloc<128>(&taddr_s);
    fence_proxy_async();
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = taddr_s;                 // cols [0,64): D ; cols [64,80): A
    // each thread writes its row (64 bytes = 16 words) into columns 64..79 of its lane
    for (int c = 0; c < 16; ++c) {
        const uint32_t w = (uint32_t)A[t * 64 + 4 * c] | ((uint32_t)A[t * 64 + 4 * c + 1] << 8) |
                           ((uint32_t)A[t * 64 + 4 * c + 2] << 16) | ((uint32_t)A[t * 64 + 4 * c + 3] << 24);
        asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};"
                     :: "r"(tmem + ((uint32_t)(warp * 32) << 16) + 64 + c), "r"(w));
    }
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    fence_before();
    __syncthreads();
    fence_after();
    if (t == 0) {
        const uint32_t b0 = smem_u32(sB);
        const uint32_t id = idesc_i8(128, 64);
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t}\n"
                     :: "r"(tmem), "r"(tmem + 64), "l"(make_desc(b0, LBO, SBO)), "r"(id), "r"(0));
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t}\n"
                     :: "r"(tmem), "r"(tmem + 64 + 8), "l"(make_desc(b0 + 2 * LBO, LBO, SBO)), "r"(id), "r"(1));
        mma_commit(&bar);
    }
    mbar_wait(&bar, 0);
    fence_after();
    uint32_t r[32];
    for (int half = 0; half < 2; ++half) {
        tmem_ld32(tmem + ((warp * 32) << 16) + half * 32, r);
        tmem_wait_ld();
        for (int c = 0; c < 32; ++c) D[t * 64 + half * 32 + c] = (int32_t)r[c];
    }
    fence_before();
    __syncthreads();
    if (t < 32) tmem_free<128>(tmem);
}

// loop: ITER x (2 MMAs 128x64x32 -> commit -> wait -> 128 threads tcgen05.ld 64 cols)
extern "C" __global__ void __launch_bounds__(128) k_probe_mma_loop(int iters, int do_ld, int do_mma, uint32_t* sink) {
    __shared__ __align__(1024) uint8_t sA[128 * 64];
    __shared__ __align__(1024) uint8_t sB[64 * 64];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t taddr_s;
    const int t = threadIdx.x;
    for (int i = t; i < 128 * 64; i += blockDim.x) sA[i] = (uint8_t)(i * 7);
    for (int i = t; i < 64 * 64; i += blockDim.x) sB[i] = (uint8_t)(i * 13);
    if (t == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
    if (t < 32) tmem_alloc<64>(&taddr_s);
    fence_proxy_async();
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = taddr_s;
    uint32_t acc = 0, phase = 0;
    const int warp = t >> 5;
    for (int it = 0; it < iters; ++it) {
        if (do_mma) {
            if (t == 0) {
                const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB);
                const uint32_t id = idesc_i8(128, 64);
                mma_i8(tmem, make_desc(a0, LBO, SBO), make_desc(b0, LBO, SBO), id, 0);
                mma_i8(tmem, make_desc(a0 + 2 * LBO, LBO, SBO), make_desc(b0 + 2 * LBO, LBO, SBO), id, 1);
                mma_commit(&bar);
            }
            mbar_wait(&bar, phase);
            phase ^= 1;
            fence_after();
        }
        if (do_ld) {
            uint32_t r[32];
#pragma unroll
            for (int half = 0; half < 2; ++half) {
                tmem_ld32(tmem + ((warp * 32) << 16) + half * 32, r);
                tmem_wait_ld();
#pragma unroll
                for (int c = 0; c < 32; ++c) acc += r[c];
            }
        }
        fence_before();
        __syncthreads();
        fence_after();
    }
    sink[blockIdx.x * 128 + t] = acc;
    if (t < 32) tmem_free<64>(tmem);
}

DEVI void bfly(uint32_t& X, uint32_t& Y, uint32_t w, uint32_t ws, uint32_t q, uint32_t q2) {
    uint32_t x = min(X, X - q2);
    uint32_t t = Y * w - __umulhi(Y, ws) * q;
    X = x + t;
    Y = x - t + q2;
}
extern "C" __global__ void k_probe_int(int iters, uint32_t q, uint32_t w, uint32_t ws, uint32_t* sink) {
    uint32_t x[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) x[i] = threadIdx.x * 16 + i;
    const uint32_t q2 = 2 * q;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int h = 8; h >= 1; h >>= 1)
#pragma unroll
            for (int g = 0; g < 16; g += 2 * h)
#pragma unroll
                for (int r = 0; r < h; ++r) bfly(x[g + r], x[g + r + h], w + h, ws + g, q, q2);
    }
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < 16; ++i) s ^= x[i];
    sink[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

extern "C" __global__ void k_copy(const uint4* __restrict__ in, uint4* __restrict__ out, size_t n16) {
    size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (; i < n16; i += stride) out[i] = in[i];
}

// ------------------------------------------------------------ host wrappers
extern "C" int probe_mma(const uint8_t* hA, const uint8_t* hB, int32_t* hD) {
    uint8_t *dA, *dB; int32_t* dD;
    cudaMalloc(&dA, 128 * 64); cudaMalloc(&dB, 64 * 64); cudaMalloc(&dD, 128 * 64 * 4);
    cudaMemcpy(dA, hA, 128 * 64, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB, 64 * 64, cudaMemcpyHostToDevice);
    k_probe_mma<<<1, 128>>>(dA, dB, dD);
    int e = (int)cudaDeviceSynchronize();
    cudaMemcpy(hD, dD, 128 * 64 * 4, cudaMemcpyDeviceToHost);
    cudaFree(dA); cudaFree(dB); cudaFree(dD);
    return e;
}

extern "C" int probe_mask(const uint8_t* hA, const uint8_t* hB4, int32_t* hD) {
    uint8_t *dA, *dB; int32_t* dD;
    cudaMalloc(&dA, 128 * 64); cudaMalloc(&dB, 4 * 64 * 64); cudaMalloc(&dD, 128 * 64 * 4);
    cudaMemcpy(dA, hA, 128 * 64, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB4, 4 * 64 * 64, cudaMemcpyHostToDevice);
    k_probe_mask<<<1, 128>>>(dA, dB, dD);
    int e = (int)cudaDeviceSynchronize();
    cudaMemcpy(hD, dD, 128 * 64 * 4, cudaMemcpyDeviceToHost);
    cudaFree(dA); cudaFree(dB); cudaFree(dD);
    return e;
}

extern "C" int probe_tmem_a(const uint8_t* hA, const uint8_t* hB, int32_t* hD) {
    uint8_t *dA, *dB; int32_t* dD;
    cudaMalloc(&dA, 128 * 64); cudaMalloc(&dB, 64 * 64); cudaMalloc(&dD, 128 * 64 * 4);
    cudaMemcpy(dA, hA, 128 * 64, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB, 64 * 64, cudaMemcpyHostToDevice);
    k_probe_tmem_a<<<1, 128>>>(dA, dB, dD);
    int e = (int)cudaDeviceSynchronize();
    cudaMemcpy(hD, dD, 128 * 64 * 4, cudaMemcpyDeviceToHost);
    cudaFree(dA); cudaFree(dB); cudaFree(dD);
    return e;
}

static float time_it(void (*launch)(void*), void* arg) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    launch(arg);
    cudaDeviceSynchronize();
    cudaEventRecord(a);
    launch(arg);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    cudaEventDestroy(a); cudaEventDestroy(b);
    return ms;
}

struct LoopArg { int blocks, iters, do_ld, do_mma; uint32_t* sink; };
static void launch_loop(void* p) {
    LoopArg* a = (LoopArg*)p;
    k_probe_mma_loop<<<a->blocks, 128>>>(a->iters, a->do_ld, a->do_mma, a->sink);
}
extern "C" float probe_mma_loop(int blocks, int iters, int do_ld, int do_mma) {
    LoopArg a{blocks, iters, do_ld, do_mma, nullptr};
    cudaMalloc(&a.sink, blocks * 128 * 4);
    float ms = time_it(launch_loop, &a);
    int e = (int)cudaGetLastError();
    cudaFree(a.sink);
    return e ? -(float)e : ms;
}

struct IntArg { int blocks, threads, iters; uint32_t* sink; };
static void launch_int(void* p) {
    IntArg* a = (IntArg*)p;
    k_probe_int<<<a->blocks, a->threads>>>(a->iters, 1073479681u, 12345u, 54321u, a->sink);
}
extern "C" float probe_int(int blocks, int threads, int iters) {
    IntArg a{blocks, threads, iters, nullptr};
    cudaMalloc(&a.sink, (size_t)blocks * threads * 4);
    float ms = time_it(launch_int, &a);
    cudaFree(a.sink);
    return ms;
}

struct CopyArg { const uint4* in; uint4* out; size_t n16; int blocks; };
static void launch_copy(void* p) {
    CopyArg* a = (CopyArg*)p;
    k_copy<<<a->blocks, 512>>>(a->in, a->out, a->n16);
}
extern "C" float probe_copy(size_t bytes, int blocks, int reps) {
    CopyArg a;
    uint4 *i, *o;
    cudaMalloc(&i, bytes); cudaMalloc(&o, bytes);
    cudaMemset(i, 1, bytes);
    a.in = i; a.out = o; a.n16 = bytes / 16; a.blocks = blocks;
    float tot = 0;
    for (int r = 0; r < reps; ++r) tot += time_it(launch_copy, &a);
    cudaFree(i); cudaFree(o);
    return tot / reps;
}
