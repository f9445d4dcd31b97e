// modarith.cuh -- device modular arithmetic for the NTT hot path (sm_100a).
//
// Word size: 32-bit residues, q < 2^30 so 4q < 2^32 (PAPER.md:375,399 use
// 32-bit words).  Multiplication by a precomputed constant w
// uses Shoup's method with w' = floor(w * 2^32 / q): for ANY 32-bit a,
//     a*w - umulhi(a, w')*q  (mod 2^32)  lies in [0, 2q).
// (The paper uses Montgomery for the NTT; reading C-8: the
// canonical outputs are unique, so the reduction scheme is free.)
// Butterflies are Harvey's lazy forms:
//   CT (forward):  inputs/outputs in [0, 4q)     -- 3 IMAD + 4 ALU ops
//   GS (inverse):  inputs/outputs in [0, 2q)
#pragma once
#include <cstdint>

namespace wd {

__device__ __forceinline__ uint32_t umin32(uint32_t a, uint32_t b) { return a < b ? a : b; }

struct __align__(32) LimbConst {
    uint32_t q, q2;          // q, 2q
    uint32_t ninv, ninv_sh;  // N^-1 mod q and its Shoup companion
    uint32_t wn, wn_sh;      // psi^-brv(1) * N^-1 (last inverse layer) + Shoup
    uint64_t mu;             // floor((2^64-1)/q): Barrett constant for a*b mod q (pointwise)
    uint32_t qinv;           // q^-1 mod 2^32 (Montgomery product of the v8 pointwise inverse)
    uint32_t ninv_r, ninv_r_sh;  // N^-1 * 2^32 mod q + Shoup: the last layer undoes 2^-32
    uint32_t wn_r, wn_r_sh;      // wn * 2^32 mod q + Shoup
    uint32_t pad_[3];
};

// a * b * 2^-32 mod q in (0, 2q) for a, b < q (Montgomery, R = 2^32): t = a*b < q^2 < q*2^32,
// m = t * q^-1 mod 2^32, so t - m*q = 0 (mod 2^32) and (t - m*q) / 2^32 = hi(t) - hi(m*q) lies in
// (-q, q); + q.  One IMAD.WIDE, one IMAD, one IMAD.HI, one IADD3 (Barrett's mul_mod: ~12 ops).
__device__ __forceinline__ uint32_t mont_mul(uint32_t a, uint32_t b, const LimbConst& c) {
    const uint64_t t = (uint64_t)a * b;
    const uint32_t m = (uint32_t)t * c.qinv;
    return (uint32_t)(t >> 32) - __umulhi(m, c.q) + c.q;
}

// a * b mod q for two variable residues (< 2^32 each, product < 2^62 for q < 2^30): Barrett
__device__ __forceinline__ uint32_t mul_mod(uint32_t a, uint32_t b, const LimbConst& c) {
    const uint64_t p = (uint64_t)a * b;
    const uint64_t quo = __umul64hi(p, c.mu);
    uint32_t r = (uint32_t)(p - quo * c.q);      // in [0, 3q)
    r = umin32(r, r - c.q);
    return umin32(r, r - c.q);
}

// a * w mod q, result in [0, 2q), any 32-bit a
__device__ __forceinline__ uint32_t shoup_mul(uint32_t a, uint32_t w, uint32_t ws, uint32_t q) {
    const uint32_t hq = __umulhi(a, ws);
    return a * w - hq * q;
}

// forward Cooley-Tukey butterfly (merged psi): (X, Y) -> (X + wY, X - wY), lazy in [0,4q)
__device__ __forceinline__ void ct_bfly(uint32_t& X, uint32_t& Y, uint2 w, uint32_t q, uint32_t q2) {
    const uint32_t x = umin32(X, X - q2);          // [0, 2q)
    const uint32_t t = shoup_mul(Y, w.x, w.y, q);  // [0, 2q)
#ifdef WD_BFLY_ALU
    X = umin32(x + t, q2 << 1);                    // = x + t (< 4q): VIADDMNMX, kept off the fma pipe
#else
    X = x + t;
#endif
    Y = x - t + q2;
}

// inverse Gentleman-Sande butterfly: (X, Y) -> (X + Y, (X - Y) w), lazy in [0,2q)
__device__ __forceinline__ void gs_bfly(uint32_t& X, uint32_t& Y, uint2 w, uint32_t q, uint32_t q2) {
#ifdef WD_BFLY_ALU
    uint32_t u = umin32(X + Y, q2 << 1);           // = X + Y (< 4q): VIADDMNMX, kept off the fma pipe
#else
    uint32_t u = X + Y;
#endif
    u = umin32(u, u - q2);
    const uint32_t t = X - Y + q2;
    Y = shoup_mul(t, w.x, w.y, q);
    X = u;
}

// last inverse layer (layer 0) with N^-1 folded in: (X, Y) -> ((X+Y) n, (X-Y) w n), in [0,2q)
__device__ __forceinline__ void gs_bfly_last(uint32_t& X, uint32_t& Y, const LimbConst& c) {
    const uint32_t u = X + Y;
    const uint32_t t = X - Y + c.q2;
    X = shoup_mul(u, c.ninv, c.ninv_sh, c.q);
    Y = shoup_mul(t, c.wn, c.wn_sh, c.q);
}

__device__ __forceinline__ uint32_t canon4(uint32_t v, uint32_t q, uint32_t q2) {  // [0,4q) -> [0,q)
    v = umin32(v, v - q2);
    return umin32(v, v - q);
}
__device__ __forceinline__ uint32_t canon2(uint32_t v, uint32_t q) {                // [0,2q) -> [0,q)
    return umin32(v, v - q);
}

// K forward layers on R = 2^K registers.  The block's elements sit at global
// indices g0 + r*D; layer ls+t pairs r and r + 2^(K-1-t) with twiddle
// Psi[2^(ls+t) + (hi << t) + (r >> (K-t))], hi = g0 >> (logN - ls) (the
// group index of the block at its first layer).  Same index rule as the
// textbook merged-psi loop, restricted to one block.
// One CT layer t (t >= 1) of a radix-2^K block: 2^t twiddle groups, the twiddle
// pairs of adjacent groups fetched as one 16-byte vector.  A template per layer
// (instead of a nested runtime-bounded loop) so NVVM always fully unrolls and x[]
// stays in registers even at K = 5.
template <int K, int t>
__device__ __forceinline__ void fwd_layer(uint32_t* x, const uint2* __restrict__ tw, int ls,
                                          uint32_t hi, uint32_t q, uint32_t q2) {
    constexpr int h = 1 << (K - 1 - t);
    const uint4* tp = reinterpret_cast<const uint4*>(tw + (1u << (ls + t)) + (hi << t));
#pragma unroll
    for (int g = 0; g < (1 << t); g += 2) {
        const uint4 v = __ldg(tp + g / 2);
        const uint2 wa = make_uint2(v.x, v.y), wb = make_uint2(v.z, v.w);
#pragma unroll
        for (int r = 0; r < h; ++r) ct_bfly(x[2 * g * h + r], x[2 * g * h + r + h], wa, q, q2);
#pragma unroll
        for (int r = 0; r < h; ++r) ct_bfly(x[2 * (g + 1) * h + r], x[2 * (g + 1) * h + r + h], wb, q, q2);
    }
    if constexpr (t + 1 < K) fwd_layer<K, t + 1>(x, tw, ls, hi, q, q2);
}

// fwd_radix with the first layer's twiddle w0 = Psi[2^ls + hi] already loaded by the
// caller (issued before a barrier so its latency is hidden).
template <int K>
__device__ __forceinline__ void fwd_radix_w0(uint32_t* x, uint2 w0, const uint2* __restrict__ tw, int ls,
                                             uint32_t hi, uint32_t q, uint32_t q2) {
#pragma unroll
    for (int r = 0; r < (1 << (K - 1)); ++r) ct_bfly(x[r], x[r + (1 << (K - 1))], w0, q, q2);
    if constexpr (K > 1) fwd_layer<K, 1>(x, tw, ls, hi, q, q2);   // layers ls+1..ls+K-1
}

template <int K>
__device__ __forceinline__ void fwd_radix(uint32_t* x, const uint2* __restrict__ tw, int ls,
                                          uint32_t hi, uint32_t q, uint32_t q2) {
    fwd_radix_w0<K>(x, __ldg(tw + (1u << ls) + hi), tw, ls, hi, q, q2);
}

// K inverse (GS) layers, mirror of fwd_radix: layers ls+K-1 down to ls.
// LAST: this block ends at global layer 0 (ls == 0), fold N^-1 there.
template <int K, int t>
__device__ __forceinline__ void inv_layer(uint32_t* x, const uint2* __restrict__ tw, int ls,
                                          uint32_t hi, uint32_t q, uint32_t q2) {
    constexpr int h = 1 << (K - 1 - t);
    const uint4* tp = reinterpret_cast<const uint4*>(tw + (1u << (ls + t)) + (hi << t));
#pragma unroll
    for (int g = 0; g < (1 << t); g += 2) {
        const uint4 v = __ldg(tp + g / 2);
        const uint2 wa = make_uint2(v.x, v.y), wb = make_uint2(v.z, v.w);
#pragma unroll
        for (int r = 0; r < h; ++r) gs_bfly(x[2 * g * h + r], x[2 * g * h + r + h], wa, q, q2);
#pragma unroll
        for (int r = 0; r < h; ++r) gs_bfly(x[2 * (g + 1) * h + r], x[2 * (g + 1) * h + r + h], wb, q, q2);
    }
    if constexpr (t > 1) inv_layer<K, t - 1>(x, tw, ls, hi, q, q2);
}

// The first (top, t = K-1) layer of an inverse radix-2^K block reads 2^(K-1) adjacent
// twiddles Psi[2^(ls+K-1) + (hi << (K-1)) ..]: InvTop holds them so a caller can
// issue the loads early (before a barrier / while other work is in flight).
template <int K>
struct InvTop { uint4 v[(1 << (K - 1)) / 2]; };

template <int K>
__device__ __forceinline__ void inv_top_load(InvTop<K>& p, const uint2* __restrict__ tw, int ls, uint32_t hi) {
    const uint4* tp = reinterpret_cast<const uint4*>(tw + (1u << (ls + K - 1)) + (hi << (K - 1)));
#pragma unroll
    for (int g = 0; g < (1 << (K - 1)) / 2; ++g) p.v[g] = __ldg(tp + g);
}

template <int K, bool LAST>
__device__ __forceinline__ void inv_radix_p(uint32_t* x, const InvTop<K>& p, const uint2* __restrict__ tw, int ls,
                                            uint32_t hi, const LimbConst& c) {
    static_assert(K >= 2, "top layer needs two groups");
#pragma unroll
    for (int g = 0; g < (1 << (K - 1)); g += 2) {      // layer ls+K-1, h = 1
        const uint4 v = p.v[g / 2];
        gs_bfly(x[2 * g], x[2 * g + 1], make_uint2(v.x, v.y), c.q, c.q2);
        gs_bfly(x[2 * g + 2], x[2 * g + 3], make_uint2(v.z, v.w), c.q, c.q2);
    }
    if constexpr (K > 2) inv_layer<K, K - 2>(x, tw, ls, hi, c.q, c.q2);
    if (LAST) {
#pragma unroll
        for (int r = 0; r < (1 << (K - 1)); ++r) gs_bfly_last(x[r], x[r + (1 << (K - 1))], c);
    } else {
        const uint2 w = __ldg(tw + (1u << ls) + hi);
#pragma unroll
        for (int r = 0; r < (1 << (K - 1)); ++r) gs_bfly(x[r], x[r + (1 << (K - 1))], w, c.q, c.q2);
    }
}

template <int K, bool LAST>
__device__ __forceinline__ void inv_radix(uint32_t* x, const uint2* __restrict__ tw, int ls,
                                          uint32_t hi, const LimbConst& c) {
    if constexpr (K >= 2) {
        InvTop<K> p;
        inv_top_load<K>(p, tw, ls, hi);
        inv_radix_p<K, LAST>(x, p, tw, ls, hi, c);
    } else if (LAST) {
        gs_bfly_last(x[0], x[1], c);
    } else {
        gs_bfly(x[0], x[1], __ldg(tw + (1u << ls) + hi), c.q, c.q2);
    }
}

}  // namespace wd
