// ntt_smem.cuh -- shared-memory-resident CUDA-core NTT/INTT for N = 2^15 and 2^16
// (SURVEY.md 8 rows a2-a4, a6-a8).  No global intermediate.
//
// A CTA of 1024 threads holds 2^15 words (128 KB) in shared memory and runs
// 15 merged-CT layers as three radix-32 register passes (5 layers each, 32
// words per thread, exchanges through shared memory):
//   pass A: blocks at stride 2^10 (lanes walk consecutive words, no conflicts)
//   pass B: blocks at stride 2^5
//   pass C: contiguous 32-word blocks (16-byte chunks XOR-swizzled by block)
//
//  * N = 2^15: one CTA per row; pass A reads the row straight from global.
//  * N = 2^16: a CTA PAIR per row, CTA c owning output half c (global index
//    c*2^15 + i).  Forward: layer 0 couples the two halves (x[j], x[j+N/2]);
//    each CTA reads both halves and computes only its own half of layer 0
//    (a redundant multiply, +2 ops/word) fused into pass A, so the pair never
//    exchanges data.  Inverse: layers 15..1 stay inside each half; layer 0
//    (with N^-1 folded in) needs both halves, so the pair is a 2-CTA thread
//    block cluster and each CTA reads the partner's half through distributed
//    shared memory (ld.shared::cluster) for its quarter of the outputs.
// This is the paper's "dual kernel when N*w > S_shared" case
// re-derived for B200: 2^16 words (256 KB) exceed the 227 KB per-CTA shared
// memory, so the row is split over two SMs instead of two launches.
#pragma once
#include <cstdint>
#include "modarith.cuh"
#include "ntt_cuda_core.cuh"

namespace wd {

constexpr int SM_T = 1024;                     // threads per CTA
constexpr int SM_WORDS = 1 << 15;              // words held per CTA
constexpr int SM_BYTES = SM_WORDS * 4;

// physical word of local index i: 16-byte chunks of each 32-word block XOR-swizzled by the block index
__device__ __forceinline__ int sw(int i) { return i ^ (((i >> 5) & 7) << 2); }

// 5 forward layers on 32 registers, twiddles of layer ls+t group (hi<<t)+g, fetched
// just in time as 16-byte pairs (keeps the 1024-thread CTA within 64 registers)
__device__ __forceinline__ void fwd32(uint32_t* x, const uint2* __restrict__ tw, int ls, uint32_t hi,
                                      uint32_t q, uint32_t q2) {
    {
        const uint2 w = __ldg(tw + (1u << ls) + hi);
#pragma unroll
        for (int r = 0; r < 16; ++r) ct_bfly(x[r], x[r + 16], w, q, q2);
    }
#pragma unroll
    for (int t = 1; t < 5; ++t) {
        const int h = 16 >> t;
        const uint4* p = reinterpret_cast<const uint4*>(tw + (1u << (ls + t)) + (hi << t));
#pragma unroll
        for (int g2 = 0; g2 < (1 << t); g2 += 2) {
            const uint4 v = __ldg(p + g2 / 2);
            const uint2 wa = make_uint2(v.x, v.y), wb = make_uint2(v.z, v.w);
#pragma unroll
            for (int r = 0; r < h; ++r) ct_bfly(x[2 * g2 * h + r], x[2 * g2 * h + r + h], wa, q, q2);
#pragma unroll
            for (int r = 0; r < h; ++r) ct_bfly(x[2 * (g2 + 1) * h + r], x[2 * (g2 + 1) * h + r + h], wb, q, q2);
        }
    }
}
template <bool LAST>
__device__ __forceinline__ void inv32(uint32_t* x, const uint2* __restrict__ tw, int ls, uint32_t hi,
                                      const LimbConst& c) {
#pragma unroll
    for (int t = 4; t >= 1; --t) {
        const int h = 16 >> t;
        const uint4* p = reinterpret_cast<const uint4*>(tw + (1u << (ls + t)) + (hi << t));
#pragma unroll
        for (int g2 = 0; g2 < (1 << t); g2 += 2) {
            const uint4 v = __ldg(p + g2 / 2);
            const uint2 wa = make_uint2(v.x, v.y), wb = make_uint2(v.z, v.w);
#pragma unroll
            for (int r = 0; r < h; ++r) gs_bfly(x[2 * g2 * h + r], x[2 * g2 * h + r + h], wa, c.q, c.q2);
#pragma unroll
            for (int r = 0; r < h; ++r) gs_bfly(x[2 * (g2 + 1) * h + r], x[2 * (g2 + 1) * h + r + h], wb, c.q, c.q2);
        }
    }
    if (LAST) {
#pragma unroll
        for (int r = 0; r < 16; ++r) gs_bfly_last(x[r], x[r + 16], c);
    } else {
        const uint2 w = __ldg(tw + (1u << ls) + hi);
#pragma unroll
        for (int r = 0; r < 16; ++r) gs_bfly(x[r], x[r + 16], w, c.q, c.q2);
    }
}

__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t map_peer(const void* p, uint32_t rank) {
    uint32_t a = (uint32_t)__cvta_generic_to_shared(p), r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(rank));
    return r;
}
__device__ __forceinline__ uint4 ld_dsmem4(uint32_t addr) {
    uint4 v;
    asm volatile("ld.shared::cluster.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
    return v;
}
__device__ __forceinline__ void st_dsmem4(uint32_t addr, uint4 v) {
    asm volatile("st.shared::cluster.v4.u32 [%0], {%1,%2,%3,%4};" :: "r"(addr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ void cpa16(void* smem_dst, const void* gsrc) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"((uint32_t)__cvta_generic_to_shared(smem_dst)), "l"(gsrc) : "memory");
}
// prefetch 2^15 contiguous words (one half-row) into S in the swizzled layout
__device__ __forceinline__ void prefetch_half(uint32_t* S, const uint32_t* src) {
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        const int u = threadIdx.x + SM_T * k;           // 16-byte chunk index
        cpa16(S + sw(4 * u), src + 4 * u);
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}
__device__ __forceinline__ void prefetch_wait() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// ------------------------------------------------------------------ forward
// LOGN = 15: one CTA per row; LOGN = 16: a 2-CTA cluster per row, CTA c owning half c.
// Row t+1's input half is prefetched into S (cp.async) as soon as pass C of row t
// has pulled its words into registers, so the load overlaps pass C's compute.
template <int LOGN>
__global__ void __launch_bounds__(SM_T, 1) ntt_fwd_smem(NttArgs a, uint32_t rows) {
    constexpr int HALF = 1 << (LOGN - 15);
    constexpr int L0 = LOGN - 15;
    extern __shared__ __align__(16) uint32_t S[];
    const int t = threadIdx.x;
    const uint32_t c = HALF == 2 ? cluster_rank() : 0;
    const uint32_t unit = HALF == 2 ? (blockIdx.x >> 1) : blockIdx.x;
    const uint32_t units = HALF == 2 ? (gridDim.x >> 1) : gridDim.x;
    if (unit >= rows) return;
    prefetch_half(S, a.in + ((size_t)unit << LOGN) + (c << 15));

    for (uint32_t row_id = unit; row_id < rows; row_id += units) {
        const uint32_t limb = row_id % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q, q2 = lc.q2;
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        uint32_t* out = a.out + ((size_t)row_id << LOGN) + (c << 15);
        uint32_t x[32];
        prefetch_wait();
        __syncthreads();
        if constexpr (HALF == 2) {
            // ---- layer 0 across the pair (DSMEM): CTA c does j in [c*2^14, (c+1)*2^14)
            cluster_sync();
            const uint2 w0 = __ldg(tw + 1);
            const uint32_t peer = map_peer(S, c ^ 1);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const int pj = sw((int)(c << 14) + 4 * t + 4096 * k);
                uint4* lp = reinterpret_cast<uint4*>(S + pj);
                const uint4 mine = *lp, other = ld_dsmem4(peer + 4 * pj);
                const uint4 U = c == 0 ? mine : other, V = c == 0 ? other : mine;
                uint32_t u[4] = {U.x, U.y, U.z, U.w}, v[4] = {V.x, V.y, V.z, V.w};
#pragma unroll
                for (int e = 0; e < 4; ++e) ct_bfly(u[e], v[e], w0, q, q2);
                const uint4 Y0 = make_uint4(u[0], u[1], u[2], u[3]), Y1 = make_uint4(v[0], v[1], v[2], v[3]);
                *lp = c == 0 ? Y0 : Y1;
                st_dsmem4(peer + 4 * pj, c == 0 ? Y1 : Y0);
            }
            cluster_sync();
        }
        // ---- pass A: local i = t + 1024 r, layers L0 .. L0+4
#pragma unroll
        for (int r = 0; r < 32; ++r) x[r] = S[sw(t + 1024 * r)];
        fwd32(x, tw, L0, c, q, q2);
#pragma unroll
        for (int r = 0; r < 32; ++r) S[sw(t + 1024 * r)] = x[r];
        __syncthreads();
        // ---- pass B: i = hb*1024 + r*32 + lo
        {
            const int hb = t >> 5, lo = t & 31;
#pragma unroll
            for (int r = 0; r < 32; ++r) x[r] = S[sw(hb * 1024 + r * 32 + lo)];
            fwd32(x, tw, L0 + 5, (c << 5) + hb, q, q2);
#pragma unroll
            for (int r = 0; r < 32; ++r) S[sw(hb * 1024 + r * 32 + lo)] = x[r];
        }
        __syncthreads();
        // ---- pass C: contiguous block t, layers L0+10 .. L0+14, then store
#pragma unroll
        for (int v = 0; v < 8; ++v) {
            const uint4 u = *reinterpret_cast<const uint4*>(S + t * 32 + ((v ^ (t & 7)) << 2));
            x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
        }
        __syncthreads();
        if (row_id + units < rows) prefetch_half(S, a.in + ((size_t)(row_id + units) << LOGN) + (c << 15));
        fwd32(x, tw, L0 + 10, (c << 10) + t, q, q2);
        uint4* o = reinterpret_cast<uint4*>(out + t * 32);
#pragma unroll
        for (int v = 0; v < 8; ++v)
            __stcs(o + v, make_uint4(canon4(x[4 * v], q, q2), canon4(x[4 * v + 1], q, q2),
                                     canon4(x[4 * v + 2], q, q2), canon4(x[4 * v + 3], q, q2)));
    }
    if constexpr (HALF == 2) cluster_sync();        // no CTA leaves while its partner may touch its S
}

// ------------------------------------------------------------------ inverse
// LOGN = 16: layers 15..1 stay in each half; layer 0 (N^-1 folded) goes through
// the row's output slot: both CTAs store their half after layer 1, cluster
// barrier (release/acquire), then CTA c finishes j in [c*2^14, (c+1)*2^14).
template <int LOGN, bool PW>
__global__ void __launch_bounds__(SM_T, 1) ntt_inv_smem(NttArgs a, uint32_t rows) {
    constexpr int HALF = 1 << (LOGN - 15);
    constexpr int L0 = LOGN - 15;
    extern __shared__ __align__(16) uint32_t S[];
    const int t = threadIdx.x;
    const uint32_t c = HALF == 2 ? cluster_rank() : 0;
    const uint32_t unit = HALF == 2 ? (blockIdx.x >> 1) : blockIdx.x;
    const uint32_t units = HALF == 2 ? (gridDim.x >> 1) : gridDim.x;
    if (unit >= rows) return;
    prefetch_half(S, a.in + ((size_t)unit << LOGN) + (c << 15));

    for (uint32_t row_id = unit; row_id < rows; row_id += units) {
        const uint32_t limb = row_id % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q;
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        const uint32_t* in2 = a.in2 + ((size_t)row_id << LOGN) + (c << 15);
        uint32_t* outrow = a.out + ((size_t)row_id << LOGN);
        uint32_t* out = outrow + (c << 15);
        uint32_t x[32];
        prefetch_wait();
        __syncthreads();
        // ---- pass C': contiguous block t of this half, layers L0+14 .. L0+10
        {
#pragma unroll
            for (int v = 0; v < 8; ++v) {
                const uint4 u = *reinterpret_cast<const uint4*>(S + t * 32 + ((v ^ (t & 7)) << 2));
                x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
            }
            if constexpr (PW) {
                const uint4* ip2 = reinterpret_cast<const uint4*>(in2 + t * 32);
#pragma unroll
                for (int v = 0; v < 8; ++v) {
                    const uint4 u = __ldcs(ip2 + v);
                    x[4 * v] = mul_mod(x[4 * v], u.x, lc); x[4 * v + 1] = mul_mod(x[4 * v + 1], u.y, lc);
                    x[4 * v + 2] = mul_mod(x[4 * v + 2], u.z, lc); x[4 * v + 3] = mul_mod(x[4 * v + 3], u.w, lc);
                }
            }
            inv32<false>(x, tw, L0 + 10, (c << 10) + t, lc);
#pragma unroll
            for (int v = 0; v < 8; ++v)
                *reinterpret_cast<uint4*>(S + t * 32 + ((v ^ (t & 7)) << 2)) =
                    make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
        }
        __syncthreads();
        // ---- pass B'
        {
            const int hb = t >> 5, lo = t & 31;
#pragma unroll
            for (int r = 0; r < 32; ++r) x[r] = S[sw(hb * 1024 + r * 32 + lo)];
            inv32<false>(x, tw, L0 + 5, (c << 5) + hb, lc);
#pragma unroll
            for (int r = 0; r < 32; ++r) S[sw(hb * 1024 + r * 32 + lo)] = x[r];
        }
        __syncthreads();
        // ---- pass A': layers L0+4 .. L0 ; S is free once the words are in registers
#pragma unroll
        for (int r = 0; r < 32; ++r) x[r] = S[sw(t + 1024 * r)];
        __syncthreads();
        if (row_id + units < rows) prefetch_half(S, a.in + ((size_t)(row_id + units) << LOGN) + (c << 15));
        if constexpr (HALF == 1) {
            inv32<true>(x, tw, 0, 0, lc);
#pragma unroll
            for (int r = 0; r < 32; ++r) __stcs(out + t + 1024 * r, canon2(x[r], q));
        } else {
            inv32<false>(x, tw, 1, c, lc);
#pragma unroll
            for (int r = 0; r < 32; ++r) out[t + 1024 * r] = x[r];      // layer-1 result, [0, 2q)
            cluster_sync();                                              // release/acquire: both halves stored
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const int j = (int)(c << 14) + 4 * t + 4096 * k;
                const uint4 U = __ldcg(reinterpret_cast<const uint4*>(outrow + j));
                const uint4 V = __ldcg(reinterpret_cast<const uint4*>(outrow + (1 << 15) + j));
                uint32_t u[4] = {U.x, U.y, U.z, U.w}, v[4] = {V.x, V.y, V.z, V.w};
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    gs_bfly_last(u[e], v[e], lc);
                    u[e] = canon2(u[e], q);
                    v[e] = canon2(v[e], q);
                }
                __stcs(reinterpret_cast<uint4*>(outrow + j), make_uint4(u[0], u[1], u[2], u[3]));
                __stcs(reinterpret_cast<uint4*>(outrow + (1 << 15) + j), make_uint4(v[0], v[1], v[2], v[3]));
            }
        }
    }
}

}  // namespace wd
