// ntt_rns.cuh -- RNS operations built around the NTT as PE kernels.
//
// RESCALE ("RSCALE(ct0) = (a0', b0') in R^2_{Q_{l-1}}"; reading C-18):
// a' = round(a / q_last) coefficient-wise, inputs and outputs in the NTT domain.  The RNS
// algorithm (oracle/rns.py is its independent CPU statement):
//   1. c  = INTT_{q_last}(a_last)                         -- one row per polynomial
//   2. v  = c - q_last [c >= q_last - floor(q_last/2)]     -- centred residue of A mod q_last
//   3. a'_i = (a_i - NTT_{q_i}(v mod q_i)) * q_last^{-1}   -- every i < last
// Launches (all polynomials of the batch in each, the PE-kernel rule of PAPER.md:334-352):
//   K1 rs_gather   copies the last-limb rows into the caller's work buffer (batch x N words),
//   K2 inverse NTT of those rows (the plan's CUDA-core kernels, a 1-limb view of the plan),
//   K3 ntt_v8<..., EPI = 1>: the forward NTT of all batch x (L-1) output rows whose phase-1
//      load applies step 2 (+ reduction mod q_i) to the shared row of its polynomial and whose
//      final store applies step 3 against the input limb -- no intermediate v_i rows in HBM.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include "common.cuh"
#include "launch.h"

namespace wd {

// work[p][n] = in[p][L-1][n]: 16-byte vectors, grid-stride
__global__ void __launch_bounds__(256) rs_gather(const uint4* __restrict__ in, uint4* __restrict__ work,
                                                 uint32_t n4, uint32_t L, uint32_t batch) {
    const size_t total = (size_t)batch * n4;
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total; i += (size_t)gridDim.x * blockDim.x) {
        const size_t p = i / n4, j = i - p * n4;
        work[i] = __ldcs(in + (p * L + (L - 1)) * n4 + j);
    }
}

}  // namespace wd

// ---------------------------------------------------------------------------------------------
// Fast basis conversion (ModUp / ModDown; reading C-19):
//   out_j = sum_i [x_i * (Q/q_i)^-1]_{q_i} * [(Q/q_i) mod p_j]  mod p_j,  coefficient domain.
// One thread per (polynomial, coefficient): the S source residues are scaled (Shoup) into shared
// memory, then each of the D outputs is a 64-bit multiply-accumulate over them, reduced every 15
// terms (15 * 2^60 + 2^30 < 2^64) with a 64-bit Barrett step.  Loads and stores walk the
// coefficient index across the warp, so every access is a coalesced 128-byte line.
namespace wd {

constexpr int BC_T = 128;                 // coefficients per CTA

__device__ __forceinline__ uint32_t reduce64(uint64_t v, uint32_t p, uint64_t mu) {
    const uint64_t quo = __umul64hi(v, mu);
    uint64_t r = v - quo * p;                 // < 3p
    while (r >= p) r -= p;
    return (uint32_t)r;
}

// x: [batch][x_ls][N] (source limbs start at row 0 of each polynomial's block);
// y: [batch][y_ls][N], targets written at rows y_off .. y_off + D - 1 of each block.
// The tables live in shared memory; the source loads are issued 8 at a time and the target
// loop is unrolled by 4 so each thread keeps several independent memory operations in flight.
// y64 != nullptr (limb-sharded ModUp): the canonical residues go to y64 [batch][D][N] as 64-bit
// words instead, so the shards' partial sums can be added by an integer all-reduce.
__global__ void __launch_bounds__(BC_T) rns_bconv(const uint32_t* __restrict__ x, uint32_t x_ls,
                                                  uint32_t* __restrict__ y, uint32_t y_ls, uint32_t y_off,
                                                  BconvTab tab, uint32_t N, uint32_t batch,
                                                  unsigned long long* __restrict__ y64 = nullptr) {
    extern __shared__ uint4 bsm4[];
    uint4* src = bsm4;                                   // [S]
    uint4* dst = bsm4 + tab.S;                           // [D]
    uint2* ws = reinterpret_cast<uint2*>(bsm4 + tab.S + tab.D);              // [S][D]
    uint32_t* ys = reinterpret_cast<uint32_t*>(ws + tab.S * tab.D);          // [S][BC_T]
    for (uint32_t i = threadIdx.x; i < tab.S; i += BC_T) src[i] = tab.src[i];
    for (uint32_t i = threadIdx.x; i < tab.D; i += BC_T) dst[i] = tab.dst[i];
    for (uint32_t i = threadIdx.x; i < tab.S * tab.D; i += BC_T) ws[i] = tab.w[i];
    const uint32_t per_poly = N / BC_T;
    __syncthreads();
    for (uint32_t blk = blockIdx.x; blk < batch * per_poly; blk += gridDim.x) {
        const uint32_t b = blk / per_poly, n = (blk % per_poly) * BC_T + threadIdx.x;
        const uint32_t* xb = x + (size_t)b * x_ls * N + n;
        for (uint32_t i0 = 0; i0 < tab.S; i0 += 8) {
            uint32_t v[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) v[u] = i0 + u < tab.S ? __ldcs(xb + (size_t)(i0 + u) * N) : 0u;
#pragma unroll
            for (int u = 0; u < 8; ++u)
                if (i0 + u < tab.S) {
                    const uint4 sc = src[i0 + u];
                    ys[(i0 + u) * BC_T + threadIdx.x] = canon2(shoup_mul(v[u], sc.y, sc.z, sc.x), sc.x);
                }
        }
        uint32_t* yb = y + ((size_t)b * y_ls + y_off) * N + n;
        if (tab.S <= 4) {                                // few terms: lazy Shoup products in [0, 2p)
            for (uint32_t j0 = 0; j0 < tab.D; j0 += 4) {
                uint32_t r[4] = {0, 0, 0, 0};
                for (uint32_t i = 0; i < tab.S; ++i) {
                    const uint32_t yi = ys[i * BC_T + threadIdx.x];
#pragma unroll
                    for (int u = 0; u < 4; ++u)
                        if (j0 + u < tab.D) {
                            const uint32_t p = dst[j0 + u].x;
                            const uint2 w = ws[i * tab.D + j0 + u];
                            r[u] += shoup_mul(yi, w.x, w.y, p);
                            r[u] = umin32(r[u], r[u] - 2 * p);
                        }
                }
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    if (j0 + u < tab.D) {
                        const uint32_t res = canon2(r[u], dst[j0 + u].x);
                        if (y64) y64[((size_t)b * tab.D + j0 + u) * N + n] = res;
                        else __stcs(yb + (size_t)(j0 + u) * N, res);
                    }
            }
        } else {                                         // many terms: 64-bit MACs, Barrett every 15
            for (uint32_t j = 0; j < tab.D; ++j) {
                const uint4 d = dst[j];
                const uint64_t mu = ((uint64_t)d.z << 32) | d.y;
                uint64_t acc = 0;
                uint32_t i = 0;
                while (i < tab.S) {
                    const uint32_t e = min(tab.S, i + 15);
                    for (; i < e; ++i) acc += (uint64_t)ys[i * BC_T + threadIdx.x] * ws[i * tab.D + j].x;
                    acc = reduce64(acc, d.x, mu);
                }
                if (y64) y64[((size_t)b * tab.D + j) * N + n] = acc;
                else __stcs(yb + (size_t)j * N, (uint32_t)acc);
            }
        }
    }
}

// Few targets (D <= 4: ModUp with k <= 4 special primes) and many sources: each thread takes 4
// consecutive coefficients (16-byte loads: a CTA reads 2 KB contiguous per source row, where
// rns_bconv reads 512 B with scalar loads), the per-source terms [x_i (Q/q_i)^-1]_{q_i} go
// straight from registers into 64-bit accumulators -- no shared-memory staging of the S terms --
// and BCF_U source rows are loaded per batch.  Same arithmetic and the same result as
// rns_bconv's 64-bit MAC path: a Barrett reduction after every BCF_U (< 15) products.
constexpr int BCF_U = 8;
constexpr int BCF_C = 4 * BC_T;                  // coefficients per CTA
template <int D>
__global__ void __launch_bounds__(BC_T) rns_bconv_few(const uint32_t* __restrict__ x, uint32_t x_ls,
                                                      uint32_t* __restrict__ y, uint32_t y_ls, uint32_t y_off,
                                                      BconvTab tab, uint32_t N, uint32_t batch) {
    extern __shared__ uint4 bsm4[];
    uint4* src = bsm4;                                   // [S]
    uint4* dst = bsm4 + tab.S;                           // [D]
    uint2* ws = reinterpret_cast<uint2*>(bsm4 + tab.S + D);                  // [S][D]
    for (uint32_t i = threadIdx.x; i < tab.S; i += BC_T) src[i] = tab.src[i];
    for (uint32_t i = threadIdx.x; i < D; i += BC_T) dst[i] = tab.dst[i];
    for (uint32_t i = threadIdx.x; i < tab.S * D; i += BC_T) ws[i] = tab.w[i];
    __syncthreads();
    const uint32_t per_poly = N / BCF_C;
    for (uint32_t blk = blockIdx.x; blk < batch * per_poly; blk += gridDim.x) {
        const uint32_t b = blk / per_poly, n = (blk % per_poly) * BCF_C + 4 * threadIdx.x;
        const uint4* xb = reinterpret_cast<const uint4*>(x + (size_t)b * x_ls * N + n);
        const uint32_t n4 = N / 4;
        uint64_t acc[4][D];
#pragma unroll
        for (int c = 0; c < 4; ++c)
#pragma unroll
            for (int j = 0; j < D; ++j) acc[c][j] = 0;
        for (uint32_t i0 = 0; i0 < tab.S; i0 += BCF_U) {
            uint4 v[BCF_U];
#pragma unroll
            for (int u = 0; u < BCF_U; ++u) v[u] = i0 + u < tab.S ? __ldcs(xb + (size_t)(i0 + u) * n4) : make_uint4(0, 0, 0, 0);
#pragma unroll
            for (int u = 0; u < BCF_U; ++u)
                if (i0 + u < tab.S) {
                    const uint4 sc = src[i0 + u];
                    const uint32_t yv[4] = {canon2(shoup_mul(v[u].x, sc.y, sc.z, sc.x), sc.x),
                                            canon2(shoup_mul(v[u].y, sc.y, sc.z, sc.x), sc.x),
                                            canon2(shoup_mul(v[u].z, sc.y, sc.z, sc.x), sc.x),
                                            canon2(shoup_mul(v[u].w, sc.y, sc.z, sc.x), sc.x)};
#pragma unroll
                    for (int j = 0; j < D; ++j) {
                        const uint32_t w = ws[(i0 + u) * D + j].x;
#pragma unroll
                        for (int c = 0; c < 4; ++c) acc[c][j] += (uint64_t)yv[c] * w;
                    }
                }
#pragma unroll
            for (int j = 0; j < D; ++j) {
                const uint4 d = dst[j];
                const uint64_t mu = ((uint64_t)d.z << 32) | d.y;
#pragma unroll
                for (int c = 0; c < 4; ++c) acc[c][j] = reduce64(acc[c][j], d.x, mu);
            }
        }
        uint32_t* yb = y + ((size_t)b * y_ls + y_off) * N + n;
#pragma unroll
        for (int j = 0; j < D; ++j)
            __stcs(reinterpret_cast<uint4*>(yb + (size_t)j * N),
                   make_uint4((uint32_t)acc[0][j], (uint32_t)acc[1][j], (uint32_t)acc[2][j], (uint32_t)acc[3][j]));
    }
}

// Few sources (S <= 4: ModDown with k <= 4 special primes) and many targets: 4 consecutive
// coefficients per thread, the S terms in registers, and one 16-byte streaming store per target
// row (a CTA writes 2 KB contiguous per target row; rns_bconv writes 512 B with scalar stores).
// Same lazy Shoup sum in [0, 2p) and the same canonical result as rns_bconv's few-terms path.
template <int S>
__global__ void __launch_bounds__(BC_T) rns_bconv_fewsrc(const uint32_t* __restrict__ x, uint32_t x_ls,
                                                         uint32_t* __restrict__ y, uint32_t y_ls, uint32_t y_off,
                                                         BconvTab tab, uint32_t N, uint32_t batch) {
    extern __shared__ uint4 bsm4[];
    uint4* src = bsm4;                                   // [S]
    uint4* dst = bsm4 + S;                               // [D]
    uint2* ws = reinterpret_cast<uint2*>(bsm4 + S + tab.D);                  // [S][D]
    for (uint32_t i = threadIdx.x; i < S; i += BC_T) src[i] = tab.src[i];
    for (uint32_t i = threadIdx.x; i < tab.D; i += BC_T) dst[i] = tab.dst[i];
    for (uint32_t i = threadIdx.x; i < S * tab.D; i += BC_T) ws[i] = tab.w[i];
    __syncthreads();
    const uint32_t per_poly = N / BCF_C;
    for (uint32_t blk = blockIdx.x; blk < batch * per_poly; blk += gridDim.x) {
        const uint32_t b = blk / per_poly, n = (blk % per_poly) * BCF_C + 4 * threadIdx.x;
        const uint4* xb = reinterpret_cast<const uint4*>(x + (size_t)b * x_ls * N + n);
        uint32_t yv[S][4];
#pragma unroll
        for (int i = 0; i < S; ++i) {
            const uint4 v = __ldcs(xb + (size_t)i * (N / 4));
            const uint4 sc = src[i];
            yv[i][0] = canon2(shoup_mul(v.x, sc.y, sc.z, sc.x), sc.x);
            yv[i][1] = canon2(shoup_mul(v.y, sc.y, sc.z, sc.x), sc.x);
            yv[i][2] = canon2(shoup_mul(v.z, sc.y, sc.z, sc.x), sc.x);
            yv[i][3] = canon2(shoup_mul(v.w, sc.y, sc.z, sc.x), sc.x);
        }
        uint32_t* yb = y + ((size_t)b * y_ls + y_off) * N + n;
#pragma unroll 2
        for (uint32_t j = 0; j < tab.D; ++j) {
            const uint32_t p = dst[j].x;
            uint32_t r[4] = {0, 0, 0, 0};
#pragma unroll
            for (int i = 0; i < S; ++i) {
                const uint2 w = ws[i * tab.D + j];
#pragma unroll
                for (int c = 0; c < 4; ++c) {
                    r[c] += shoup_mul(yv[i][c], w.x, w.y, p);
                    r[c] = umin32(r[c], r[c] - 2 * p);
                }
            }
            __stcs(reinterpret_cast<uint4*>(yb + (size_t)j * N),
                   make_uint4(canon2(r[0], p), canon2(r[1], p), canon2(r[2], p), canon2(r[3], p)));
        }
    }
}

// sum [rows][N] 64-bit (the all-reduced shard partials) -> canonical residue mod p_{row % D}
__global__ void __launch_bounds__(256) rns_reduce64(const unsigned long long* __restrict__ sum, uint32_t* __restrict__ out,
                                                    const uint4* __restrict__ dst, uint32_t D, uint32_t N, uint32_t rows) {
    const size_t total = (size_t)rows * N;
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total; i += (size_t)gridDim.x * blockDim.x) {
        const uint4 d = dst[(i / N) % D];
        out[i] = reduce64(sum[i], d.x, ((uint64_t)d.z << 32) | d.y);
    }
}

}  // namespace wd
