// common.cuh -- launch arguments and small device helpers shared by the NTT kernels.
#pragma once
#include <cstdint>
#include "modarith.cuh"

namespace wd {

struct NttArgs {
    const uint32_t* in;
    const uint32_t* in2;      // inverse only: if set, transform in o in2 (pointwise product, row f1)
    uint32_t* out;
    const uint2* tw;          // [L][N] (psi^+-brv(i), Shoup) for this direction
    const LimbConst* lc;      // [L]
    uint32_t L;
    // RESCALE epilogue of the forward (ntt_v8<..., EPI = 1>): the phase-1
    // input row of row r is in + (r / L) * N (the last limb's coefficients c of polynomial r / L,
    // shared by its L output limbs), the output is (aux_i - NTT(c')) * q_last^-1 (ntt_rns.cuh)
    const uint32_t* aux = nullptr;   // the rescale input [batch][Lfull][N]
    const uint4* rs = nullptr;       // [L] {-q_last mod q_i, Shoup(1), q_last^-1 mod q_i, Shoup}
    uint32_t rs_thr = 0;             // q_last - floor(q_last / 2)
    uint32_t Lfull = 0;
    // v8 only: rows between consecutive polynomials in `in` / `out` (0 = L, contiguous); lets a
    // launch cover a limb SECTION of a wider [batch][Lfull][N] tensor (ModUp / ModDown, ntt_rns.cuh)
    uint32_t in_ls = 0, out_ls = 0;
    // v8 inverse only: if set, every input row is also copied unchanged to cpy (rows between
    // polynomials: cpy_ls) as it is staged -- ModUp's pass-through of the Q limbs (ntt_rns.cuh)
    uint32_t* cpy = nullptr;
    uint32_t cpy_ls = 0;
    uint32_t limb_major = 0;         // v8: walk rows limb by limb (rows must be a multiple of L)
    // a launch over a part of a bigger batch's schedule (tm + v8 tail, wd_ntt.cu launch_cuda_core): the
    // launch covers schedule slots slot0 .. slot0 + rows - 1 of a batch of nb_total polynomials (0: the
    // launch's own rows / L); the slot -> row map (limb-major) is the whole batch's
    uint32_t slot0 = 0;
    uint32_t nb_total = 0;
};

__device__ __forceinline__ uint32_t row_map(uint32_t row, uint32_t L, uint32_t ls) {
    return ls ? (row / L) * ls + row % L : row;
}

// ---------------------------------------------------------------- cp.async (16-byte, L2-only)
__device__ __forceinline__ void cp_async16(void* smem_dst, const void* gsrc) {
    const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem_dst);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" :: "n"(N) : "memory"); }

// ---------------------------------------------------------------- thread-block clusters
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

// ---------------------------------------------------------------- radix-16 blocks with explicit twiddles
// the 15 twiddles of one 16-point block, layers ls..ls+3, group hi: Psi[2^ls + hi], Psi[2^(ls+1) + 2hi ..],
// Psi[2^(ls+2) + 4hi ..], Psi[2^(ls+3) + 8hi ..], fetched as 16-byte vectors
__device__ __forceinline__ void load_tw16(uint2* w, const uint2* __restrict__ tw, int ls, uint32_t hi) {
    w[0] = __ldg(tw + (1u << ls) + hi);
    const uint4 a = __ldg(reinterpret_cast<const uint4*>(tw + (2u << ls) + 2 * hi));
    w[1] = make_uint2(a.x, a.y); w[2] = make_uint2(a.z, a.w);
#pragma unroll
    for (int k = 0; k < 2; ++k) {
        const uint4 b = __ldg(reinterpret_cast<const uint4*>(tw + (4u << ls) + 4 * hi) + k);
        w[3 + 2 * k] = make_uint2(b.x, b.y); w[4 + 2 * k] = make_uint2(b.z, b.w);
    }
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const uint4 b = __ldg(reinterpret_cast<const uint4*>(tw + (8u << ls) + 8 * hi) + k);
        w[7 + 2 * k] = make_uint2(b.x, b.y); w[8 + 2 * k] = make_uint2(b.z, b.w);
    }
}
// radix-16 forward block with explicit twiddles w[0..14] (layer t group g -> w[(1<<t)-1+g])
__device__ __forceinline__ void fwd16_tw(uint32_t* x, const uint2* w, uint32_t q, uint32_t q2) {
#pragma unroll
    for (int t = 0; t < 4; ++t) {
        const int h = 8 >> t;
#pragma unroll
        for (int g = 0; g < (1 << t); ++g)
#pragma unroll
            for (int r = 0; r < h; ++r) ct_bfly(x[2 * g * h + r], x[2 * g * h + r + h], w[(1 << t) - 1 + g], q, q2);
    }
}
__device__ __forceinline__ void inv16_tw(uint32_t* x, const uint2* w, uint32_t q, uint32_t q2) {
#pragma unroll
    for (int t = 3; t >= 0; --t) {
        const int h = 8 >> t;
#pragma unroll
        for (int g = 0; g < (1 << t); ++g)
#pragma unroll
            for (int r = 0; r < h; ++r) gs_bfly(x[2 * g * h + r], x[2 * g * h + r + h], w[(1 << t) - 1 + g], q, q2);
    }
}

}  // namespace wd
