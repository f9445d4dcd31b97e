// ntt_fused.cuh -- concurrent tensor-core + CUDA-core NTT/INTT for N = 2^16.
//
// WD-FUSE role of the paper (section IV-B, Fig. 3: tensor-core
// warps and CUDA-core warps in the SAME block so that every SM sub-partition
// holds both kinds of work; section IV-D3: the split follows the
// units' relative throughput; Fig. 6: WD-FUSE beats either unit).
// B200 design: one persistent CTA per SM with two warp groups --
//   warps  0..15 (512 threads): CUDA-core chunk worker (radix-16 butterflies,
//                                cp.async double-buffered chunks, ntt_persist.cuh)
//   warps 16..19 (128 threads): tcgen05 worker (ntt_tensor.cuh); warp 16 owns
//                                TMEM (its warp index is 0 mod 4, so warp 16+w
//                                reads TMEM lanes 32w..32w+31)
// Each group takes whole rows from the CTA's row list through a shared-memory
// counter, so the split between the units is decided at run time by their
// measured speed (a dynamic version of the paper's ratio knob).  If
// tensor_share is given (0..1), rows are instead assigned statically:
// row index i of the CTA goes to the tensor group iff frac(i*share) < share.
#pragma once
#include <algorithm>
#include "ntt_tensor.cuh"
#include "ntt_persist.cuh"

namespace wd {

constexpr int FU_CC = 512;
constexpr int FUP_TC = 256, FUP_T = FU_CC + FUP_TC;      // phase-split pipeline: 8 tensor warps
constexpr int FU_CC_BAR = 2;
constexpr int FUP_SMEM = PGeo<16>::SMEM_BYTES + TCC_SMEM + 64;

template <int BAR, int NT>
__device__ __forceinline__ void gbar() {
    if constexpr (BAR == 0) __syncthreads();
    else named_bar(BAR, NT);
}

// one whole row on the CUDA-core group (chunk pipeline of ntt_persist.cuh, named barrier BAR)
template <bool FWD, bool PW, int BAR>
__device__ __forceinline__ void cc_row(const NttArgs& a, uint32_t* smem, uint32_t row_id) {
    using G = PGeo<16>;
    constexpr int CA = FWD ? G::C1 : G::C2;
    constexpr int CH = G::C1 + G::C2;
    const uint32_t* in = a.in + ((size_t)row_id << 16);
    uint32_t* out = a.out + ((size_t)row_id << 16);
    const uint32_t limb = row_id % a.L;
    const LimbConst lc = a.lc[limb];
    const uint2* __restrict__ tw = a.tw + ((size_t)limb << 16);
    auto issue = [&](int kk, uint32_t* S) {
        if (FWD) {
            if (kk < G::C1) load_p1<16>(S, in, kk * G::W1);
            else load_p2<16>(S, out, (kk - G::C1) * G::W2);
        } else {
            if (kk < G::C2) load_p2<16>(S, in, kk * G::W2);
            else load_p1<16>(S, out, (kk - G::C2) * G::W1);
        }
        cp_async_commit();
    };
    issue(0, smem);
#pragma unroll 1
    for (int kk = 0; kk < CH; ++kk) {
        uint32_t* S = smem + (kk & 1) * G::BUF_WORDS;
        const bool dep = (kk + 1 == CA);
        if (kk + 1 < CH && !dep) {
            issue(kk + 1, smem + ((kk + 1) & 1) * G::BUF_WORDS);
            cp_async_wait<1>();
        } else {
            cp_async_wait<0>();
        }
        gbar<BAR, FU_CC>();
        if (FWD) {
            if (kk < G::C1) fwd_p1_chunk<16, BAR>(S, out, kk * G::W1, tw, lc.q, lc.q2);
            else fwd_p2_chunk<16, BAR>(S, out, (kk - G::C1) * G::W2, tw, lc.q, lc.q2);
        } else {
            const uint32_t* in2 = a.in2 + ((size_t)row_id << 16);
            if (kk < G::C2) inv_p2_chunk<16, PW, BAR>(S, out, in2, kk * G::W2, tw, lc);
            else inv_p1_chunk<16, BAR>(S, out, (kk - G::C2) * G::W1, tw, lc);
        }
        __threadfence_block();
        gbar<BAR, FU_CC>();
        if (dep) issue(kk + 1, smem + ((kk + 1) & 1) * G::BUF_WORDS);
    }
}

constexpr int FU_LEAD = 2;
// measured default tensor share of the pipeline (scripts/gpu_sweep.sh)
constexpr float FUSED_DEFAULT_SHARE = 1.0f;

__device__ __forceinline__ int ld_volatile(const int* p) { return *reinterpret_cast<const volatile int*>(p); }

// CUDA-core group: only phase 2 (forward) / phase 2' (inverse) of one row
template <bool FWD, int BAR>
__device__ __forceinline__ void cc_row_phase2(const NttArgs& a, uint32_t* smem, uint32_t row_id) {
    using G = PGeo<16>;
    const uint32_t* in = a.in + ((size_t)row_id << 16);
    uint32_t* out = a.out + ((size_t)row_id << 16);
    const uint32_t limb = row_id % a.L;
    const LimbConst lc = a.lc[limb];
    const uint2* __restrict__ tw = a.tw + ((size_t)limb << 16);
    const uint32_t* src = FWD ? out : in;
    load_p2<16>(smem, src, 0);
    cp_async_commit();
#pragma unroll 1
    for (int kk = 0; kk < G::C2; ++kk) {
        uint32_t* S = smem + (kk & 1) * G::BUF_WORDS;
        if (kk + 1 < G::C2) {
            load_p2<16>(smem + ((kk + 1) & 1) * G::BUF_WORDS, src, (kk + 1) * G::W2);
            cp_async_commit();
            cp_async_wait<1>();
        } else {
            cp_async_wait<0>();
        }
        gbar<BAR, FU_CC>();
        if (FWD) fwd_p2_chunk<16, BAR>(S, out, kk * G::W2, tw, lc.q, lc.q2);
        else inv_p2_chunk<16, false, BAR>(S, out, nullptr, kk * G::W2, tw, lc);
        gbar<BAR, FU_CC>();
    }
}

template <bool FWD>
// share: fraction of rows whose column phase runs on the tensor warps (interleaved); the
// CUDA-core warps run the remaining rows whole (the paper's tensor/CUDA ratio knob).
__global__ void __launch_bounds__(FUP_T, 1) ntt_fused16_pipe(TcArgs ta, const uint8_t* G, uint32_t rows, uint32_t per_cta,
                                                             float share) {
    constexpr int lead = FU_LEAD;
    extern __shared__ __align__(1024) uint8_t fsm[];
    uint32_t* ccbuf = reinterpret_cast<uint32_t*>(fsm);
    uint8_t* tcb = fsm + PGeo<16>::SMEM_BYTES;
    TccShared sh;
    sh.A0 = tcb;
    sh.B = tcb + TCC_NBUF * TC_TILE;
    sh.bar = reinterpret_cast<uint64_t*>(tcb + TCC_NBUF * TC_TILE + 17 * 4096);
    sh.tslot = reinterpret_cast<uint32_t*>(sh.bar + 4);
    uint32_t* loaded = sh.tslot + 1;
    int* ctl = reinterpret_cast<int*>(tcb + TCC_SMEM);          // [0] rows done by the leader, [1] by the follower
    const int tid = threadIdx.x;
    if (tid == 0) {
        ctl[0] = 0; ctl[1] = 0;
        for (int i = 0; i < 4; ++i) mbar_init(&sh.bar[i], 1);
        *loaded = 0xffffffffu;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (tid >= FU_CC && tid < FU_CC + 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(smem_addr(sh.tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t L = ta.a.L, Bp = rows / L;
    const uint32_t k0 = blockIdx.x * per_cta, k1 = min(rows, k0 + per_cta);
    const int nmine = k1 > k0 ? (int)(k1 - k0) : 0;
    const bool is_tc = tid >= FU_CC;
    const bool leader = FWD ? is_tc : !is_tc;                    // who runs the first phase of a row
    const int gtid = is_tc ? tid - FU_CC : tid;
    const int nthr = is_tc ? FUP_TC : FU_CC;
    const int bar = is_tc ? TC_BAR_ID : FU_CC_BAR;
    int* mine = &ctl[leader ? 0 : 1];
    const int* other = &ctl[leader ? 1 : 0];
    const uint32_t tmem = *sh.tslot;
    uint32_t ph[4] = {0, 0, 0, 0};
    for (int i = 0; i < nmine; ++i) {
        if (gtid == 0) {
            if (leader) { while (i - ld_volatile(other) >= lead) __nanosleep(256); }
            else { while (ld_volatile(other) <= i) __nanosleep(128); }
        }
        named_bar(bar, nthr);
        __threadfence_block();
        const uint32_t k = k0 + (uint32_t)i;
        const uint32_t limb = k / Bp, row = (k % Bp) * L + limb;
        const bool tc_row = floorf((float)(i + 1) * share) > floorf((float)i * share);
        if (is_tc) {
            if (tc_row)
                tcc_columns<FWD, false, FUP_TC>(ta, sh, tmem, ph, row, G + ((size_t)limb * 2 + (FWD ? 0 : 1)) * 17 * 4096,
                                                loaded, TC_BAR_ID);
        } else {
            if (tc_row) cc_row_phase2<FWD, FU_CC_BAR>(ta.a, ccbuf, row);
            else cc_row<FWD, false, FU_CC_BAR>(ta.a, ccbuf, row);
        }
        __threadfence_block();
        named_bar(bar, nthr);
        if (gtid == 0) atomicExch(mine, i + 1);
    }
    if (is_tc) {
        tc_fence_before();
        named_bar(TC_BAR_ID, FUP_TC);
        if (gtid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tmem));
    }
}

inline int prepare_fused_kernels(uint32_t logN) {
    if (logN != 16) return 0;
    for (auto k : {ntt_fused16_pipe<true>, ntt_fused16_pipe<false>})
        if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, FUP_SMEM) != cudaSuccess ||
            cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, 100) != cudaSuccess)
            return 4;
    return 0;
}

// FUSED: one persistent CTA per SM; rows split evenly over the CTAs (limb-major), the share of
// rows whose column phase goes to the tensor warps is `share` (< 0: FUSED_DEFAULT_SHARE)
inline int launch_fused(uint32_t logN, bool fwd, const NttArgs& a, const TensorTables& tc, uint32_t rows,
                        int sm_count, float share, cudaStream_t s) {
    if (logN != 16 || !tc.ok || a.in2) return -1;
    TcArgs ta;
    ta.a = a;
    ta.B = tc.d_B;
    ta.t1 = fwd ? tc.d_tw1 : tc.d_sg1;
    ta.t2 = fwd ? tc.d_tw2 : tc.d_sg2;
    ta.t3 = fwd ? tc.d_tw3 : tc.d_sg3;
    ta.c16 = tc.d_c16;
    const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)sm_count);
    const uint32_t per = (rows + grid - 1) / grid;
    const float sh = share < 0.0f ? FUSED_DEFAULT_SHARE : share;
    if (fwd) ntt_fused16_pipe<true><<<grid, FUP_T, FUP_SMEM, s>>>(ta, tc.d_G, rows, per, sh);
    else ntt_fused16_pipe<false><<<grid, FUP_T, FUP_SMEM, s>>>(ta, tc.d_G, rows, per, sh);
    return 1;
}

}  // namespace wd
