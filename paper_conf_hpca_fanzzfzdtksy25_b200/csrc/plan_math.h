// plan_math.h -- host-side number theory for the plan precompute.
//
// PAPER.md:358 (section IV-D1): "selecting and generating moduli and
// precomputed values such as twiddle factors used in the NTT ... transferred
// to the GPU in advance".  Independent of oracle/ (which uses a linear scan
// for psi; here psi comes from a generator of Z_q^*, see plan_psi_min).
#pragma once
#include <cstdint>
#include <vector>

namespace wd {

inline uint32_t pm_mul(uint32_t a, uint32_t b, uint32_t q) { return (uint32_t)(((uint64_t)a * b) % q); }

inline uint32_t pm_pow(uint32_t a, uint64_t e, uint32_t q) {
    uint32_t r = 1 % q, b = a % q;
    for (; e; e >>= 1) {
        if (e & 1) r = pm_mul(r, b, q);
        b = pm_mul(b, b, q);
    }
    return r;
}

// Deterministic Miller-Rabin for 32-bit n with witnesses {2, 7, 61}.
inline bool pm_is_prime(uint32_t n) {
    if (n < 2) return false;
    for (uint32_t p : {2u, 3u, 5u, 7u, 11u, 13u, 61u}) {
        if (n == p) return true;
        if (n % p == 0) return false;
    }
    uint32_t d = n - 1;
    int s = 0;
    while (!(d & 1)) { d >>= 1; ++s; }
    for (uint32_t a : {2u, 7u, 61u}) {
        uint32_t x = pm_pow(a, d, n);
        if (x == 1 || x == n - 1) continue;
        bool witness = true;
        for (int i = 1; i < s && witness; ++i) {
            x = pm_mul(x, x, n);
            if (x == n - 1) witness = false;
        }
        if (witness) return false;
    }
    return true;
}

// Shoup companion floor(w * 2^32 / q), w < q.
inline uint32_t pm_shoup(uint32_t w, uint32_t q) { return (uint32_t)(((uint64_t)w << 32) / q); }

inline uint32_t pm_brv(uint32_t i, int logn) {
    uint32_t r = 0;
    for (int b = 0; b < logn; ++b, i >>= 1) r = (r << 1) | (i & 1);
    return r;
}

// Minimal primitive 2N-th root of unity (reading C-4): take a generator g0 of
// Z_q^*, psi0 = g0^((q-1)/2N), and the minimum over its odd powers (exactly
// the N primitive 2N-th roots).
inline uint32_t plan_psi_min(uint32_t q, uint32_t N) {
    const uint32_t phi = q - 1;
    std::vector<uint32_t> fac;
    uint32_t m = phi;
    for (uint32_t p = 2; (uint64_t)p * p <= m; ++p)
        if (m % p == 0) { fac.push_back(p); while (m % p == 0) m /= p; }
    if (m > 1) fac.push_back(m);
    uint32_t g0 = 2;
    for (;; ++g0) {
        bool gen = true;
        for (uint32_t p : fac) if (pm_pow(g0, phi / p, q) == 1) { gen = false; break; }
        if (gen) break;
    }
    const uint32_t psi0 = pm_pow(g0, phi / (2ull * N), q);
    const uint32_t step = pm_mul(psi0, psi0, q);
    uint32_t cur = psi0, best = psi0;
    for (uint32_t i = 1; i < N; ++i) {
        cur = pm_mul(cur, step, q);
        if (cur < best) best = cur;
    }
    return best;
}

}  // namespace wd
