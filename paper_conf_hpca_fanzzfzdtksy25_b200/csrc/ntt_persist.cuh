// ntt_persist.cuh -- cp.async-pipelined CUDA-core chunk workers for N = 2^15..2^17, used by the
// CUDA-core warps of the FUSED pipeline (ntt_fused.cuh).  (Round 1 also
// built a persistent kernel on them, v2/v6; it was superseded by v8 and removed.)
//
// One CTA per SM loops over its share of the batch*L rows (PE-kernel idea,
// PAPER.md:334-352).  A row is N = N1 x 256: phase 1 = the first log2(N1)
// merged-CT layers on 256 columns (stride 256), phase 2 = the last 8 layers on
// N1 contiguous 256-word rows (the paper's 4-step / 7-step decomposition,
// PAPER.md:93-100, 272-282, without the transpose -> bit-reversed output).
// Each phase is cut into CHUNKS of ~8192 words.  A chunk is copied global ->
// shared with 16-byte cp.async (LDGSTS) one chunk ahead of its use (double
// buffer), then two register stages run on it IN PLACE in shared memory
// (radix 2^A0 then 2^A1 on columns, radix 16 x 16 on rows), so the
// inter-stage exchange needs no extra buffer.  Phase-1 results go to the
// row's own output slot (L2-resident), phase 2 reads them back.
#pragma once
#include <cstdint>
#include "modarith.cuh"
#include "ntt_cuda_core.cuh"

namespace wd {

// barrier among the 512 CUDA-core threads: __syncthreads when they are the whole CTA,
// a named barrier when they share the CTA with the tensor group (ntt_fused.cuh)
template <int BAR>
__device__ __forceinline__ void pbar() {
    if constexpr (BAR == 0) __syncthreads();
    else asm volatile("bar.sync %0, 512;" :: "n"(BAR) : "memory");
}

template <int LOGN> struct PCfg;
template <> struct PCfg<15> { static constexpr int A0 = 4, A1 = 3; };
template <> struct PCfg<16> { static constexpr int A0 = 4, A1 = 4; };
template <> struct PCfg<17> { static constexpr int A0 = 5, A1 = 4; };

template <int LOGN, int TT = 512>
struct PGeo {
    static constexpr int T = TT;
    static constexpr int A0 = PCfg<LOGN>::A0, A1 = PCfg<LOGN>::A1;
    static constexpr int B1 = LOGN - 8, N1 = 1 << B1;
    static constexpr int R0 = 1 << A0, R1 = 1 << A1;
    static constexpr int E1 = R0 > R1 ? R0 : R1;
    static constexpr int G1 = N1 / E1;               // threads per column
    static constexpr int W1 = T / G1;                // columns per phase-1 chunk
    static constexpr int C1 = 256 / W1;              // phase-1 chunks per row
    static constexpr int INST0 = E1 / R0, INST1 = E1 / R1;
    static constexpr int W2 = T / 16;                // rows per phase-2 chunk
    static constexpr int C2 = N1 / W2;               // phase-2 chunks per row
    // phase-1 word of (row p, column w) is p1(p) + w.  With W1 = 8 a warp spans 4 values of
    // j whose stage-1 rows (p = j*R1 + r) would sit 8*R1 words apart, i.e. in the same banks:
    // one extra W1 of padding per 2^A1 rows (monotone, so rows never overlap) moves them
    // to 4 different bank groups; in stage 0 (p = j + r*R1) it is a warp-uniform offset.
    static constexpr int P1_PAD = W1 >= 16 ? 0 : (N1 >> A1) * W1;
    __device__ __forceinline__ static int p1(int p) { return p * W1 + (W1 >= 16 ? 0 : (p >> A1) * W1); }
    static constexpr int P1_WORDS = N1 * W1 + P1_PAD;
    static constexpr int P2_WORDS = W2 * RS;
    static constexpr int BUF_WORDS = P1_WORDS > P2_WORDS ? P1_WORDS : P2_WORDS;
    static constexpr int SMEM_BYTES = 2 * 4 * BUF_WORDS;
    static_assert(W1 % 4 == 0 && (W1 >= 16 || W1 == 8) && 256 % W1 == 0, "phase-1 chunk");
    static_assert(N1 % W2 == 0, "phase-2 chunk");
};

// ---- chunk loads (all T threads) --------------------------------------------------------
// phase-1 chunk: columns [c0, c0+W1) of every one of the N1 256-word rows -> S[p*W1 + w]
template <int LOGN, int TT = 512>
__device__ __forceinline__ void load_p1(uint32_t* S, const uint32_t* src, int c0) {
    using G = PGeo<LOGN, TT>;
    constexpr int SEG = G::W1 / 4, NSEG = G::N1 * SEG;
    static_assert(NSEG % G::T == 0, "whole segments per thread");
#pragma unroll
    for (int k = 0; k < NSEG / G::T; ++k) {
        const int i = threadIdx.x % G::T + k * G::T;
        const int p = i / SEG, s = i % SEG;
        cp_async16(S + G::p1(p) + 4 * s, src + p * 256 + c0 + 4 * s);
    }
}
// phase-2 chunk: rows [r0, r0+W2), 256 words each -> swizzled ywords() layout
template <int LOGN, int TT = 512>
__device__ __forceinline__ void load_p2(uint32_t* S, const uint32_t* src, int r0) {
    using G = PGeo<LOGN, TT>;
    constexpr int NSEG = G::W2 * 64;
    static_assert(NSEG % G::T == 0, "whole segments per thread");
#pragma unroll
    for (int k = 0; k < NSEG / G::T; ++k) {
        const int i = threadIdx.x % G::T + k * G::T;
        const int w = i >> 6, v4 = i & 63, chi = v4 >> 2, v = v4 & 3;
        cp_async16(S + w * RS + chi * 16 + (((v ^ (chi >> 1)) & 3) << 2), src + (r0 + w) * 256 + 4 * v4);
    }
}

// ---- forward chunk compute ------------------------------------------------------------
template <int LOGN, int BAR = 0, int TT = 512>
__device__ __forceinline__ void fwd_p1_chunk(uint32_t* S, uint32_t* out, int c0, const uint2* __restrict__ tw,
                                             uint32_t q, uint32_t q2) {
    using G = PGeo<LOGN, TT>;
    const int w = threadIdx.x % G::W1, j = threadIdx.x / G::W1;
    uint32_t x[G::E1];
#pragma unroll
    for (int u = 0; u < G::INST0; ++u) {
        const int i0 = j * G::INST0 + u;
#pragma unroll
        for (int r = 0; r < G::R0; ++r) x[u * G::R0 + r] = S[G::p1((i0 + (r << G::A1))) + w];
        fwd_radix<G::A0>(x + u * G::R0, tw, 0, 0, q, q2);
#pragma unroll
        for (int r = 0; r < G::R0; ++r) S[G::p1((i0 + (r << G::A1))) + w] = x[u * G::R0 + r];
    }
    pbar<BAR>();
    const int c = c0 + w;
#pragma unroll
    for (int u = 0; u < G::INST1; ++u) {
        const int i1 = j * G::INST1 + u;
#pragma unroll
        for (int r = 0; r < G::R1; ++r) x[r] = S[G::p1(((i1 << G::A1) + r)) + w];
        fwd_radix<G::A1>(x, tw, G::A0, i1, q, q2);
#pragma unroll
        for (int r = 0; r < G::R1; ++r) out[((i1 << G::A1) + r) * 256 + c] = x[r];
    }
}

template <int LOGN, int BAR = 0, int TT = 512>
__device__ __forceinline__ void fwd_p2_chunk(uint32_t* S, uint32_t* out, int r0, const uint2* __restrict__ tw,
                                             uint32_t q, uint32_t q2) {
    using G = PGeo<LOGN, TT>;
    const int c = threadIdx.x & 15, w = threadIdx.x >> 4;
    const int row = r0 + w;
    uint32_t x[16];
    uint2 w3[15];
    load_tw16(w3, tw, G::B1 + 4, (uint32_t)row * 16 + c);      // in flight during stage 2
#pragma unroll
    for (int r = 0; r < 16; ++r) x[r] = S[ywords(w, r, c)];
    fwd_radix<4>(x, tw, G::B1, row, q, q2);
#pragma unroll
    for (int r = 0; r < 16; ++r) S[ywords(w, r, c)] = x[r];
    pbar<BAR>();
#pragma unroll
    for (int v = 0; v < 4; ++v) {
        const uint4 t = *reinterpret_cast<const uint4*>(S + w * RS + c * 16 + (((v ^ (c >> 1)) & 3) << 2));
        x[4 * v] = t.x; x[4 * v + 1] = t.y; x[4 * v + 2] = t.z; x[4 * v + 3] = t.w;
    }
    fwd16_tw(x, w3, q, q2);
    uint4* o = reinterpret_cast<uint4*>(out + row * 256 + c * 16);
#pragma unroll
    for (int v = 0; v < 4; ++v)
        __stcs(o + v, make_uint4(canon4(x[4 * v], q, q2), canon4(x[4 * v + 1], q, q2),
                                 canon4(x[4 * v + 2], q, q2), canon4(x[4 * v + 3], q, q2)));
}

// ---- inverse chunk compute (phase 2' then phase 1') ---------------------------------------
template <int LOGN, bool PW, int BAR = 0, int TT = 512>
__device__ __forceinline__ void inv_p2_chunk(uint32_t* S, uint32_t* out, const uint32_t* in2, int r0,
                                             const uint2* __restrict__ tw, const LimbConst& lc) {
    using G = PGeo<LOGN, TT>;
    const int c = threadIdx.x & 15, w = threadIdx.x >> 4;
    const int row = r0 + w;
    uint32_t x[16];
    uint2 w3[15];
    load_tw16(w3, tw, G::B1 + 4, (uint32_t)row * 16 + c);
#pragma unroll
    for (int v = 0; v < 4; ++v) {
        const uint4 t = *reinterpret_cast<const uint4*>(S + w * RS + c * 16 + (((v ^ (c >> 1)) & 3) << 2));
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
    inv16_tw(x, w3, lc.q, lc.q2);
#pragma unroll
    for (int v = 0; v < 4; ++v)
        *reinterpret_cast<uint4*>(S + w * RS + c * 16 + (((v ^ (c >> 1)) & 3) << 2)) =
            make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
    pbar<BAR>();
#pragma unroll
    for (int r = 0; r < 16; ++r) x[r] = S[ywords(w, r, c)];
    inv_radix<4, false>(x, tw, G::B1, row, lc);
#pragma unroll
    for (int r = 0; r < 16; ++r) out[row * 256 + c + 16 * r] = x[r];
}

template <int LOGN, int BAR = 0, int TT = 512>
__device__ __forceinline__ void inv_p1_chunk(uint32_t* S, uint32_t* out, int c0, const uint2* __restrict__ tw,
                                             const LimbConst& lc) {
    using G = PGeo<LOGN, TT>;
    const int w = threadIdx.x % G::W1, j = threadIdx.x / G::W1;
    uint32_t x[G::E1];
#pragma unroll
    for (int u = 0; u < G::INST1; ++u) {
        const int i1 = j * G::INST1 + u;
#pragma unroll
        for (int r = 0; r < G::R1; ++r) x[r] = S[G::p1(((i1 << G::A1) + r)) + w];
        inv_radix<G::A1, false>(x, tw, G::A0, i1, lc);
#pragma unroll
        for (int r = 0; r < G::R1; ++r) S[G::p1(((i1 << G::A1) + r)) + w] = x[r];
    }
    pbar<BAR>();
    const int c = c0 + w;
#pragma unroll
    for (int u = 0; u < G::INST0; ++u) {
        const int i0 = j * G::INST0 + u;
#pragma unroll
        for (int r = 0; r < G::R0; ++r) x[u * G::R0 + r] = S[G::p1((i0 + (r << G::A1))) + w];
        inv_radix<G::A0, true>(x + u * G::R0, tw, 0, 0, lc);
#pragma unroll
        for (int r = 0; r < G::R0; ++r)
            __stcs(out + (i0 + (r << G::A1)) * 256 + c, canon2(x[u * G::R0 + r], lc.q));
    }
}

// ---- the persistent kernel ---------------------------------------------------------------
// chunk k of a row: forward  k <  C1 -> phase-1 chunk k (src = in),  else phase-2 chunk k-C1 (src = out)
//                   inverse  k <  C2 -> phase-2' chunk k (src = in), else phase-1' chunk k-C2 (src = out)
}  // namespace wd
