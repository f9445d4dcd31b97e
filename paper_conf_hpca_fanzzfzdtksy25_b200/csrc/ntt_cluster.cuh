// ntt_cluster.cuh -- cluster-resident CUDA-core NTT/INTT for N = 2^14 .. 2^17.
//
// A row of N = 2^LOGN words is split over a thread-block cluster of CL = 2^(LOGN-14) CTAs; CTA c
// keeps the 2^14-word slice c (global index c*2^14 + i) in shared memory (64 KB), so there is
// no global intermediate and DRAM traffic is the algorithmic 8N bytes per transform.
//   forward: the first L0 = log2(CL) merged-CT layers couple the slices (index bits above 14):
//            after a cluster barrier, CTA c runs that radix-CL butterfly network for its share
//            j in [c*2^14/CL, (c+1)*2^14/CL) of every slice, reading and writing the peers'
//            shared memory directly (ld/st.shared::cluster), then a second cluster barrier;
//            the remaining 14 layers run locally as radix-32, radix-32, radix-16 register passes.
//   inverse: the local passes first, then the radix-CL GS network with N^-1 over DSMEM, whose
//            outputs go straight to global memory.
// 512 threads x 32 words per CTA, 64 registers: two CTAs (two different rows) share an SM, so
// one CTA's barrier / twiddle-load stalls overlap the other's arithmetic.  The next row's slice
// is prefetched with cp.async as soon as the last pass has pulled its words into registers.
// This is the paper's large-N "dual kernel" case and its step-4 "transposition
// of the large matrix ... GMEM operation potentially needed" re-derived for
// B200: the cross-slice step goes through distributed shared memory instead of GMEM.
#pragma once
#include <cstdint>
#include "modarith.cuh"
#include "ntt_cuda_core.cuh"
#include "common.cuh"

namespace wd {

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

__device__ __forceinline__ void cpa16(void* smem_dst, const void* gsrc) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"((uint32_t)__cvta_generic_to_shared(smem_dst)), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void prefetch_wait() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

constexpr int CL_T = 512;                        // threads per CTA
constexpr int CL_WORDS = 1 << 14;                // words per CTA
constexpr int CL_BYTES = (CL_WORDS + 16 * (CL_WORDS >> 9)) * 4;   // + 16 words of padding per 512

// Shared-memory layout of local index i: the 16-byte chunk index (bits 2..4) is XORed with
// bits 4..6, and 16 words of padding follow every 512 words.  Checked exhaustively (no bank
// conflicts for passes A/B/C, the cp.async prefetch and the DSMEM exchange; 16-B chunks stay
// contiguous), and every pass address is a per-thread base plus a compile-time offset:
//   pass A  i = t + 512 r              -> swz(t) + 528 r
//   pass B  i = hb*512 + 16 r + lo     -> hb*528 + 16 (r ^ ((r>>2)&1)) + (lo ^ 4 (r&3))
//   pass C  i = 16 b + 4 v (16-B)      -> (16b ^ 16((b>>2)&1)) + 16 (b>>5) + 4 (v ^ (b&3))
__device__ __forceinline__ int swz(int i) { return i ^ (((i >> 4) & 7) << 2); }
__device__ __forceinline__ int csw(int i) { return swz(i) + ((i >> 9) << 4); }
__device__ __forceinline__ int pc_base(int b) { return ((16 * b) ^ (((b >> 2) & 1) << 4)) + ((b >> 5) << 4); }

__device__ __forceinline__ void cl_prefetch(uint32_t* S, const uint32_t* src) {
#pragma unroll
    for (int k = 0; k < CL_WORDS / 4 / CL_T; ++k) {
        const int u = threadIdx.x + CL_T * k;            // 16-byte chunk index
        cpa16(S + csw(4 * u), src + 4 * u);
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

// 4 forward layers on 16 registers (pass C), twiddles of layer ls+t group (hi<<t)+g as 16-B pairs
__device__ __forceinline__ void fwd16p(uint32_t* x, const uint2* __restrict__ tw, int ls, uint32_t hi,
                                       uint32_t q, uint32_t q2) {
    fwd_radix<4>(x, tw, ls, hi, q, q2);
}

template <int LOGN>
__global__ void __launch_bounds__(CL_T, 2) ntt_fwd_cl(NttArgs a, uint32_t rows) {
    constexpr int CL = 1 << (LOGN - 14);
    constexpr int L0 = LOGN - 14;
    extern __shared__ __align__(16) uint32_t S[];
    const int t = threadIdx.x;
    const uint32_t c = CL > 1 ? cluster_rank() : 0;
    const uint32_t unit = blockIdx.x / CL, units = gridDim.x / CL;
    if (unit >= rows) return;
    cl_prefetch(S, a.in + ((size_t)unit << LOGN) + (c << 14));

    for (uint32_t row_id = unit; row_id < rows; row_id += units) {
        const uint32_t limb = row_id % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q, q2 = lc.q2;
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        uint32_t* out = a.out + ((size_t)row_id << LOGN) + (c << 14);
        uint32_t x[32];
        prefetch_wait();
        __syncthreads();
        if constexpr (CL > 1) {
            // ---- layers 0 .. L0-1 across the cluster: CTA c owns j in [c*2^14/CL, (c+1)*2^14/CL)
            cluster_sync();
            uint32_t peer[CL];
#pragma unroll
            for (int p = 0; p < CL; ++p) peer[p] = map_peer(S, p);
            constexpr int JV = CL_WORDS / CL / 4 / CL_T;          // 4-word vectors per thread (>= 1)
#pragma unroll
            for (int k = 0; k < JV; ++k) {
                const int j = (int)c * (CL_WORDS / CL) + 4 * (t + CL_T * k);
                const uint32_t pj = 4u * (uint32_t)csw(j);
                uint32_t v[4][CL];
#pragma unroll
                for (int p = 0; p < CL; ++p) {
                    const uint4 u = ld_dsmem4(peer[p] + pj);
                    v[0][p] = u.x; v[1][p] = u.y; v[2][p] = u.z; v[3][p] = u.w;
                }
#pragma unroll
                for (int e = 0; e < 4; ++e) fwd_radix<L0>(v[e], tw, 0, 0, q, q2);
#pragma unroll
                for (int p = 0; p < CL; ++p) st_dsmem4(peer[p] + pj, make_uint4(v[0][p], v[1][p], v[2][p], v[3][p]));
            }
            cluster_sync();
        }
        // ---- pass A: i = t + 512 r, layers L0 .. L0+4
        {
            uint32_t* pa = S + swz(t);
#pragma unroll
            for (int r = 0; r < 32; ++r) x[r] = pa[528 * r];
            fwd32(x, tw, L0, c, q, q2);
#pragma unroll
            for (int r = 0; r < 32; ++r) pa[528 * r] = x[r];
        }
        __syncthreads();
        // ---- pass B: i = hb*512 + r*16 + lo, layers L0+5 .. L0+9
        {
            const int hb = t >> 4, lo = t & 15;
            uint32_t* pb[4];
#pragma unroll
            for (int m = 0; m < 4; ++m) pb[m] = S + hb * 528 + (lo ^ (4 * m));
#pragma unroll
            for (int r = 0; r < 32; ++r) x[r] = pb[r & 3][16 * (r ^ ((r >> 2) & 1))];
            fwd32(x, tw, L0 + 5, (c << 5) + hb, q, q2);
#pragma unroll
            for (int r = 0; r < 32; ++r) pb[r & 3][16 * (r ^ ((r >> 2) & 1))] = x[r];
        }
        __syncthreads();
        // ---- pass C: 16-word blocks b = t and t + 512, layers L0+10 .. L0+13
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int b = t + 512 * h;
            const uint32_t* pcb = S + pc_base(b);
#pragma unroll
            for (int v = 0; v < 4; ++v) {
                const uint4 u = *reinterpret_cast<const uint4*>(pcb + 4 * (v ^ (b & 3)));
                x[16 * h + 4 * v] = u.x; x[16 * h + 4 * v + 1] = u.y; x[16 * h + 4 * v + 2] = u.z; x[16 * h + 4 * v + 3] = u.w;
            }
        }
        __syncthreads();
        if (row_id + units < rows) cl_prefetch(S, a.in + ((size_t)(row_id + units) << LOGN) + (c << 14));
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int b = t + 512 * h;
            fwd16p(x + 16 * h, tw, L0 + 10, (c << 10) + b, q, q2);
            uint4* o = reinterpret_cast<uint4*>(out + 16 * b);
#pragma unroll
            for (int v = 0; v < 4; ++v) {
                const uint32_t* y = x + 16 * h + 4 * v;
                __stcs(o + v, make_uint4(canon4(y[0], q, q2), canon4(y[1], q, q2), canon4(y[2], q, q2),
                                         canon4(y[3], q, q2)));
            }
        }
    }
    if constexpr (CL > 1) cluster_sync();
}

template <int LOGN, bool PW>
__global__ void __launch_bounds__(CL_T, 2) ntt_inv_cl(NttArgs a, uint32_t rows) {
    constexpr int CL = 1 << (LOGN - 14);
    constexpr int L0 = LOGN - 14;
    extern __shared__ __align__(16) uint32_t S[];
    const int t = threadIdx.x;
    const uint32_t c = CL > 1 ? cluster_rank() : 0;
    const uint32_t unit = blockIdx.x / CL, units = gridDim.x / CL;
    if (unit >= rows) return;
    cl_prefetch(S, a.in + ((size_t)unit << LOGN) + (c << 14));

    for (uint32_t row_id = unit; row_id < rows; row_id += units) {
        const uint32_t limb = row_id % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q;
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        const uint32_t* in2 = a.in2 + ((size_t)row_id << LOGN) + (c << 14);
        uint32_t* outrow = a.out + ((size_t)row_id << LOGN);
        uint32_t x[32];
        prefetch_wait();
        __syncthreads();
        // ---- pass C': blocks t, t+512, layers L0+13 .. L0+10
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int b = t + 512 * h;
            uint32_t* pcb = S + pc_base(b);
#pragma unroll
            for (int v = 0; v < 4; ++v) {
                const uint4 u = *reinterpret_cast<const uint4*>(pcb + 4 * (v ^ (b & 3)));
                x[16 * h + 4 * v] = u.x; x[16 * h + 4 * v + 1] = u.y; x[16 * h + 4 * v + 2] = u.z; x[16 * h + 4 * v + 3] = u.w;
            }
            if constexpr (PW) {
                const uint4* ip2 = reinterpret_cast<const uint4*>(in2 + 16 * b);
#pragma unroll
                for (int v = 0; v < 4; ++v) {
                    const uint4 u = __ldcs(ip2 + v);
                    uint32_t* y = x + 16 * h + 4 * v;
                    y[0] = mul_mod(y[0], u.x, lc); y[1] = mul_mod(y[1], u.y, lc);
                    y[2] = mul_mod(y[2], u.z, lc); y[3] = mul_mod(y[3], u.w, lc);
                }
            }
            inv_radix<4, false>(x + 16 * h, tw, L0 + 10, (c << 10) + b, lc);
#pragma unroll
            for (int v = 0; v < 4; ++v)
                *reinterpret_cast<uint4*>(pcb + 4 * (v ^ (b & 3))) =
                    make_uint4(x[16 * h + 4 * v], x[16 * h + 4 * v + 1], x[16 * h + 4 * v + 2], x[16 * h + 4 * v + 3]);
        }
        __syncthreads();
        // ---- pass B'
        {
            const int hb = t >> 4, lo = t & 15;
            uint32_t* pb[4];
#pragma unroll
            for (int m = 0; m < 4; ++m) pb[m] = S + hb * 528 + (lo ^ (4 * m));
#pragma unroll
            for (int r = 0; r < 32; ++r) x[r] = pb[r & 3][16 * (r ^ ((r >> 2) & 1))];
            inv32<false>(x, tw, L0 + 5, (c << 5) + hb, lc);
#pragma unroll
            for (int r = 0; r < 32; ++r) pb[r & 3][16 * (r ^ ((r >> 2) & 1))] = x[r];
        }
        __syncthreads();
        // ---- pass A': layers L0+4 .. L0
        uint32_t* pa = S + swz(t);
#pragma unroll
        for (int r = 0; r < 32; ++r) x[r] = pa[528 * r];
        if constexpr (CL == 1) {
            __syncthreads();
            if (row_id + units < rows) cl_prefetch(S, a.in + ((size_t)(row_id + units) << LOGN));
            inv32<true>(x, tw, 0, 0, lc);
#pragma unroll
            for (int r = 0; r < 32; ++r) __stcs(outrow + t + 512 * r, canon2(x[r], q));
        } else {
            inv32<false>(x, tw, L0, c, lc);
#pragma unroll
            for (int r = 0; r < 32; ++r) pa[528 * r] = x[r];
            // ---- layers L0-1 .. 0 (N^-1 folded) across the cluster, outputs straight to global
            cluster_sync();
            uint32_t peer[CL];
#pragma unroll
            for (int p = 0; p < CL; ++p) peer[p] = map_peer(S, p);
            constexpr int JV = CL_WORDS / CL / 4 / CL_T;
#pragma unroll
            for (int k = 0; k < JV; ++k) {
                const int j = (int)c * (CL_WORDS / CL) + 4 * (t + CL_T * k);
                const uint32_t pj = 4u * (uint32_t)csw(j);
                uint32_t v[4][CL];
#pragma unroll
                for (int p = 0; p < CL; ++p) {
                    const uint4 u = ld_dsmem4(peer[p] + pj);
                    v[0][p] = u.x; v[1][p] = u.y; v[2][p] = u.z; v[3][p] = u.w;
                }
#pragma unroll
                for (int e = 0; e < 4; ++e) inv_radix<L0, true>(v[e], tw, 0, 0, lc);
#pragma unroll
                for (int p = 0; p < CL; ++p)
                    __stcs(reinterpret_cast<uint4*>(outrow + ((size_t)p << 14) + j),
                           make_uint4(canon2(v[0][p], q), canon2(v[1][p], q), canon2(v[2][p], q), canon2(v[3][p], q)));
            }
            cluster_sync();                                  // peers done reading my slice
            if (row_id + units < rows) cl_prefetch(S, a.in + ((size_t)(row_id + units) << LOGN) + (c << 14));
        }
    }
}

}  // namespace wd
