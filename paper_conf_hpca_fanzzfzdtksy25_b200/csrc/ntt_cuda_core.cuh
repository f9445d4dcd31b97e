// ntt_cuda_core.cuh -- CUDA-core radix-2^k NTT/INTT kernels.
//
// WD-BO role of the paper (high-radix butterflies with the
// intermediates in registers).  B200 design:
//
//   * one CTA per (polynomial, limb) row; grid = batch*L in ONE launch
//     (the PE-kernel idea);
//   * N = N1 x N2 with N2 = 256 (rows, contiguous) and N1 = N/256 (columns,
//     stride 256).  Phase 1 runs the first log2(N1) merged-CT layers on the
//     columns, phase 2 the last 8 layers on the rows -- the paper's 4-step
//     decomposition without the transpose, which
//     keeps the merged-psi bit-reversed output order;
//   * each phase is two register stages (radix 2^a, 2^b <= 32) with one
//     shared-memory exchange between them; global loads/stores are coalesced
//     (lanes walk consecutive columns, or 16-B vectors along a row);
//   * N <= 2^14: the phase-1 -> phase-2 intermediate stays in shared memory.
//     N >= 2^15 (one limb > 227 KB SMEM at 2^16): the intermediate goes
//     through the row's own output slot in global memory (L2-resident, the
//     CTA reads back what it just wrote) -- the paper's "dual kernel" case
//      folded into one launch.
//   * N < 2^12: a simple shared-memory kernel (debug sizes).
#pragma once
#include <cstdint>
#include "modarith.cuh"
#include "common.cuh"

namespace wd {

constexpr int RS = 272;       // padded row stride (words) of 256-wide rows in SMEM

template <int LOGN> struct CcCfg;
//                         T    A0 A1
template <> struct CcCfg<12> { static constexpr int T = 256, A0 = 4, A1 = 0; };
template <> struct CcCfg<13> { static constexpr int T = 512, A0 = 3, A1 = 2; };
template <> struct CcCfg<14> { static constexpr int T = 512, A0 = 3, A1 = 3; };
template <> struct CcCfg<15> { static constexpr int T = 512, A0 = 4, A1 = 3; };
template <> struct CcCfg<16> { static constexpr int T = 512, A0 = 4, A1 = 4; };
template <> struct CcCfg<17> { static constexpr int T = 512, A0 = 5, A1 = 4; };

template <int LOGN>
struct CcShape {
    using C = CcCfg<LOGN>;
    static constexpr int T = C::T, A0 = C::A0, A1 = C::A1;
    static constexpr int B1 = LOGN - 8, N1 = 1 << B1, N2 = 256;
    static constexpr int R0 = 1 << A0, R1 = 1 << A1;
    static constexpr int E1 = R0 > R1 ? R0 : R1;     // elements per thread, phase 1
    static constexpr int G1 = N1 / E1;               // threads per column
    static constexpr int W1 = T / G1;                // columns per chunk
    static constexpr int NCH1 = N2 / W1;
    static constexpr int INST0 = E1 / R0, INST1 = E1 / R1;
    static constexpr int W2 = T / 16;                // rows per chunk
    static constexpr int NCH2 = N1 / W2;
    static constexpr bool GINTER = LOGN >= 15;       // intermediate through global
    static constexpr int X_WORDS = (A1 > 0 ? N1 * W1 : 0);
    static constexpr int Y_WORDS = W2 * RS;
    static constexpr int XY_WORDS = X_WORDS > Y_WORDS ? X_WORDS : Y_WORDS;
    static constexpr int S_WORDS = GINTER ? 0 : N1 * RS;
    static constexpr int SMEM_BYTES = 4 * (XY_WORDS + S_WORDS);
    static_assert(W1 >= 32 && N2 % W1 == 0, "phase-1 chunking");
    static_assert(N1 % W2 == 0, "phase-2 chunking");
};

__device__ __forceinline__ int ywords(int w, int chi, int clo) {   // swizzled row-exchange slot
    return w * RS + chi * 16 + ((((clo >> 2) ^ (chi >> 1)) & 3) << 2) + (clo & 3);
}

// ------------------------------------------------------------------ forward
template <int LOGN>
__global__ void __launch_bounds__(CcCfg<LOGN>::T, 1) ntt_fwd_cc(NttArgs a) {
    using S = CcShape<LOGN>;
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* XY = smem;                       // stage-exchange buffer (phase 1 / phase 2)
    uint32_t* SB = smem + S::XY_WORDS;         // whole-limb buffer (N <= 2^14)

    const uint32_t row_id = blockIdx.x;
    const uint32_t limb = row_id % a.L;
    const LimbConst lc = a.lc[limb];
    const uint32_t q = lc.q, q2 = lc.q2;
    const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
    const uint32_t* in = a.in + ((size_t)row_id << LOGN);
    uint32_t* out = a.out + ((size_t)row_id << LOGN);
    const int tid = threadIdx.x;

    // ---- phase 1: columns c (stride 256), layers 0 .. B1-1
    {
        const int w = tid % S::W1, j = tid / S::W1;
#pragma unroll 1
        for (int ch = 0; ch < S::NCH1; ++ch) {
            const int c = ch * S::W1 + w;
            uint32_t x[S::E1];
#pragma unroll
            for (int u = 0; u < S::INST0; ++u) {
                const int i0 = j * S::INST0 + u;
#pragma unroll
                for (int r = 0; r < S::R0; ++r)
                    x[u * S::R0 + r] = __ldcs(in + (size_t)((i0 + (r << S::A1)) * 256 + c));
            }
#pragma unroll
            for (int u = 0; u < S::INST0; ++u) fwd_radix<S::A0>(x + u * S::R0, tw, 0, 0, q, q2);
            if constexpr (S::A1 == 0) {
#pragma unroll
                for (int u = 0; u < S::INST0; ++u) {
                    const int i0 = j * S::INST0 + u;
#pragma unroll
                    for (int r = 0; r < S::R0; ++r) {
                        const int p = i0 + (r << S::A1);
                        if constexpr (S::GINTER) out[p * 256 + c] = x[u * S::R0 + r];
                        else SB[p * RS + c] = x[u * S::R0 + r];
                    }
                }
            } else {
#pragma unroll
                for (int u = 0; u < S::INST0; ++u) {
                    const int i0 = j * S::INST0 + u;
#pragma unroll
                    for (int r = 0; r < S::R0; ++r) XY[(i0 + (r << S::A1)) * S::W1 + w] = x[u * S::R0 + r];
                }
                __syncthreads();
#pragma unroll
                for (int u = 0; u < S::INST1; ++u) {
                    const int i1 = j * S::INST1 + u;
#pragma unroll
                    for (int r = 0; r < S::R1; ++r) x[u * S::R1 + r] = XY[((i1 << S::A1) + r) * S::W1 + w];
                    fwd_radix<S::A1>(x + u * S::R1, tw, S::A0, i1, q, q2);
#pragma unroll
                    for (int r = 0; r < S::R1; ++r) {
                        const int p = (i1 << S::A1) + r;
                        if constexpr (S::GINTER) out[p * 256 + c] = x[u * S::R1 + r];
                        else SB[p * RS + c] = x[u * S::R1 + r];
                    }
                }
                __syncthreads();
            }
        }
    }
    __syncthreads();

    // ---- phase 2: rows (256 contiguous), layers B1 .. LOGN-1, radix 16 x 16
    {
        const int c = tid & 15, w = tid >> 4;
#pragma unroll 1
        for (int ch = 0; ch < S::NCH2; ++ch) {
            const int row = ch * S::W2 + w;
            uint32_t x[16];
#pragma unroll
            for (int r = 0; r < 16; ++r) {
                if constexpr (S::GINTER) x[r] = __ldcg(out + row * 256 + c + 16 * r);
                else x[r] = SB[row * RS + c + 16 * r];
            }
            fwd_radix<4>(x, tw, S::B1, row, q, q2);
#pragma unroll
            for (int r = 0; r < 16; ++r) XY[ywords(w, r, c)] = x[r];
            __syncthreads();
#pragma unroll
            for (int v = 0; v < 4; ++v) {
                const uint4 t = *reinterpret_cast<const uint4*>(XY + w * RS + c * 16 + (((v ^ (c >> 1)) & 3) << 2));
                x[4 * v] = t.x; x[4 * v + 1] = t.y; x[4 * v + 2] = t.z; x[4 * v + 3] = t.w;
            }
            fwd_radix<4>(x, tw, S::B1 + 4, (uint32_t)row * 16 + c, q, q2);
            uint4* o = reinterpret_cast<uint4*>(out + row * 256 + c * 16);
#pragma unroll
            for (int v = 0; v < 4; ++v)
                o[v] = make_uint4(canon4(x[4 * v], q, q2), canon4(x[4 * v + 1], q, q2),
                                  canon4(x[4 * v + 2], q, q2), canon4(x[4 * v + 3], q, q2));
            __syncthreads();
        }
    }
}

// ------------------------------------------------------------------ inverse
template <int LOGN, bool PW>
__global__ void __launch_bounds__(CcCfg<LOGN>::T, 1) ntt_inv_cc(NttArgs a) {
    using S = CcShape<LOGN>;
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* XY = smem;
    uint32_t* SB = smem + S::XY_WORDS;

    const uint32_t row_id = blockIdx.x;
    const uint32_t limb = row_id % a.L;
    const LimbConst lc = a.lc[limb];
    const uint32_t q = lc.q;
    const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
    const uint32_t* in = a.in + ((size_t)row_id << LOGN);
    const uint32_t* in2 = a.in2 + ((size_t)row_id << LOGN);
    uint32_t* out = a.out + ((size_t)row_id << LOGN);
    const int tid = threadIdx.x;

    // ---- phase 2': rows, layers LOGN-1 .. B1
    {
        const int c = tid & 15, w = tid >> 4;
#pragma unroll 1
        for (int ch = 0; ch < S::NCH2; ++ch) {
            const int row = ch * S::W2 + w;
            uint32_t x[16];
            const uint4* ip = reinterpret_cast<const uint4*>(in + row * 256 + c * 16);
#pragma unroll
            for (int v = 0; v < 4; ++v) {
                const uint4 t = __ldcs(ip + v);
                x[4 * v] = t.x; x[4 * v + 1] = t.y; x[4 * v + 2] = t.z; x[4 * v + 3] = t.w;
            }
            if constexpr (PW) {
                const uint4* ip2 = reinterpret_cast<const uint4*>(in2 + row * 256 + c * 16);
#pragma unroll
                for (int v = 0; v < 4; ++v) {
                    const uint4 t = __ldcs(ip2 + v);
                    x[4 * v] = mul_mod(x[4 * v], t.x, lc); x[4 * v + 1] = mul_mod(x[4 * v + 1], t.y, lc);
                    x[4 * v + 2] = mul_mod(x[4 * v + 2], t.z, lc); x[4 * v + 3] = mul_mod(x[4 * v + 3], t.w, lc);
                }
            }
            inv_radix<4, false>(x, tw, S::B1 + 4, (uint32_t)row * 16 + c, lc);
#pragma unroll
            for (int v = 0; v < 4; ++v)
                *reinterpret_cast<uint4*>(XY + w * RS + c * 16 + (((v ^ (c >> 1)) & 3) << 2)) =
                    make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
            __syncthreads();
#pragma unroll
            for (int r = 0; r < 16; ++r) x[r] = XY[ywords(w, r, c)];
            inv_radix<4, false>(x, tw, S::B1, row, lc);
#pragma unroll
            for (int r = 0; r < 16; ++r) {
                if constexpr (S::GINTER) out[row * 256 + c + 16 * r] = x[r];
                else SB[row * RS + c + 16 * r] = x[r];
            }
            __syncthreads();
        }
    }
    __syncthreads();

    // ---- phase 1': columns, layers B1-1 .. 0 (N^-1 folded into layer 0)
    {
        const int w = tid % S::W1, j = tid / S::W1;
#pragma unroll 1
        for (int ch = 0; ch < S::NCH1; ++ch) {
            const int c = ch * S::W1 + w;
            uint32_t x[S::E1];
            if constexpr (S::A1 > 0) {
#pragma unroll
                for (int u = 0; u < S::INST1; ++u) {
                    const int i1 = j * S::INST1 + u;
#pragma unroll
                    for (int r = 0; r < S::R1; ++r) {
                        const int p = (i1 << S::A1) + r;
                        if constexpr (S::GINTER) x[u * S::R1 + r] = __ldcg(out + p * 256 + c);
                        else x[u * S::R1 + r] = SB[p * RS + c];
                    }
                    inv_radix<S::A1, false>(x + u * S::R1, tw, S::A0, i1, lc);
#pragma unroll
                    for (int r = 0; r < S::R1; ++r) XY[((i1 << S::A1) + r) * S::W1 + w] = x[u * S::R1 + r];
                }
                __syncthreads();
#pragma unroll
                for (int u = 0; u < S::INST0; ++u) {
                    const int i0 = j * S::INST0 + u;
#pragma unroll
                    for (int r = 0; r < S::R0; ++r) x[u * S::R0 + r] = XY[(i0 + (r << S::A1)) * S::W1 + w];
                }
            } else {
#pragma unroll
                for (int u = 0; u < S::INST0; ++u) {
                    const int i0 = j * S::INST0 + u;
#pragma unroll
                    for (int r = 0; r < S::R0; ++r) {
                        const int p = i0 + (r << S::A1);
                        if constexpr (S::GINTER) x[u * S::R0 + r] = __ldcg(out + p * 256 + c);
                        else x[u * S::R0 + r] = SB[p * RS + c];
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < S::INST0; ++u) {
                const int i0 = j * S::INST0 + u;
                inv_radix<S::A0, true>(x + u * S::R0, tw, 0, 0, lc);
#pragma unroll
                for (int r = 0; r < S::R0; ++r)
                    __stcs(out + (size_t)((i0 + (r << S::A1)) * 256 + c), canon2(x[u * S::R0 + r], q));
            }
            if constexpr (S::A1 > 0) __syncthreads();
        }
    }
}

// ------------------------------------------------------------------ small N (debug sizes)
// One CTA per row, whole row in SMEM, one merged-CT / GS layer per barrier.
template <bool FWD, bool PW>
__global__ void __launch_bounds__(256) ntt_small(NttArgs a, int logn) {
    extern __shared__ __align__(16) uint32_t smem[];
    const int n = 1 << logn;
    const uint32_t row_id = blockIdx.x;
    const uint32_t limb = row_id % a.L;
    const LimbConst lc = a.lc[limb];
    const uint32_t q = lc.q, q2 = lc.q2;
    const uint2* __restrict__ tw = a.tw + ((size_t)limb << logn);
    const uint32_t* in = a.in + ((size_t)row_id << logn);
    uint32_t* out = a.out + ((size_t)row_id << logn);
    for (int i = threadIdx.x; i < n; i += blockDim.x)
        smem[i] = PW ? mul_mod(in[i], a.in2[((size_t)row_id << logn) + i], lc) : in[i];
    __syncthreads();
    if (FWD) {
        for (int l = 0; l < logn; ++l) {
            const int t = n >> (l + 1);
            for (int b = threadIdx.x; b < n / 2; b += blockDim.x) {
                const int grp = b / t, off = b % t;
                const int j = 2 * grp * t + off;
                uint32_t X = smem[j], Y = smem[j + t];
                ct_bfly(X, Y, tw[(1 << l) + grp], q, q2);
                smem[j] = X; smem[j + t] = Y;
            }
            __syncthreads();
        }
        for (int i = threadIdx.x; i < n; i += blockDim.x) out[i] = canon4(smem[i], q, q2);
    } else {
        for (int l = logn - 1; l >= 0; --l) {
            const int t = n >> (l + 1);
            for (int b = threadIdx.x; b < n / 2; b += blockDim.x) {
                const int grp = b / t, off = b % t;
                const int j = 2 * grp * t + off;
                uint32_t X = smem[j], Y = smem[j + t];
                if (l == 0) gs_bfly_last(X, Y, lc);
                else gs_bfly(X, Y, tw[(1 << l) + grp], q, q2);
                smem[j] = X; smem[j + t] = Y;
            }
            __syncthreads();
        }
        for (int i = threadIdx.x; i < n; i += blockDim.x) out[i] = canon2(smem[i], q);
    }
}

}  // namespace wd
