// ntt_tmt.cuh -- "tm" for N = 2^13: one team per row, TMEM-resident rows (
// DESIGN.md 5.1a).
//
// v8's decomposition with A = 1 (ntt_v8.cuh): N = 2 x 4096, layer 0 on the 4096 columns of 2 elements,
// layers 1..12 as three radix-16 stages on the 2 sub-rows.  A row is 2^13 words = 32 cells per (TMEM
// lane, column half), so every team of the CTA can own its rows outright: team tau is a virtual CTA that
// processes schedule slots 4 blockIdx + tau + k (4 gridDim), with two row slots of its own in TMEM,
//   cell (column pass p, element k) -> lane t % 128, column 256 h + 64 tau + 32 (j & 1) + 2 p + k,
// and no synchronisation with the other teams at all (team barriers only).  Per row and team:
//   forward, step i = 0, 1:  R1(j, i) [stage 1 of sub-row i from TMEM]  C(j+1, passes 8i..8i+7) [one
//                            3-D TMA box of 8 passes -> layer 0 -> TMEM]  team barrier  R23(j, i)
//   inverse:                 team barrier (row j in TMEM), then for i = 0, 1: C'(j, passes 8i..8i+7)
//                            [TMEM -> layer 0 with N^-1 -> out]  R'(j+1, i) [cp.async -> stages 3', 2' ->
//                            team barrier -> stage 1' -> TMEM]
// Every team barrier that orders TMEM accesses of different warps is bracketed by tcgen05.wait::st +
// fence::before_thread_sync and fence::after_thread_sync.
#pragma once
#include "ntt_tms.cuh"

namespace wd {
namespace tmt {

using tmr::TEAMS; using tmr::TT; using tmr::NT; using tmr::SUBW; using tmr::TWW; using tmr::TEAM_W;
constexpr int SMEM = TEAMS * TEAM_W * 4 + 256;   // + 3 mbarriers per team + the TMEM base slot

template <bool FWD>
__global__ void __launch_bounds__(NT, 1) ntt_tmt13(NttArgs a, uint32_t rows, const __grid_constant__ CUtensorMap tm_in) {
    constexpr int LOGN = 13, A = 1, R = 2;
    constexpr int SLOT = 32;                     // TMEM columns of one row per (lane, half) and team
    extern __shared__ __align__(1024) uint32_t smem[];
    const int team = (int)(threadIdx.x >> 8), t = (int)(threadIdx.x & (TT - 1));
    const int w = t >> 5, h = w >> 2, hi4 = t >> 4, lo4 = t & 15;
    uint32_t* TS = smem + team * TEAM_W;
    uint32_t* const B0 = TS;                     // forward: sub-row exchange; inverse: input buffer 0
    uint32_t* const B1 = TS + SUBW;              // inverse: input buffer 1; forward: staging of even steps
    auto SB = [&](uint32_t m) { return TS + SUBW + (m & 1) * SUBW; };   // forward staging of step m
    auto TWB = [&](int b) { return reinterpret_cast<uint2*>(TS + 3 * SUBW + b * TWW); };
    // per team: tbar[0..1] the forward TMA stagings, tbar[2] "B0 free"
    uint64_t* tbar = reinterpret_cast<uint64_t*>(smem + TEAMS * TEAM_W) + 3 * team;
    uint32_t* tslot = reinterpret_cast<uint32_t*>(reinterpret_cast<uint64_t*>(smem + TEAMS * TEAM_W) + 3 * TEAMS);

    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(smem_u32(tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (t == 0) {
        mb_init(tbar, 1); mb_init(tbar + 1, 1); mb_init(tbar + 2, TT / 32);
        mb_init_fence();
    }
    tmr::tfence_before();
    __syncthreads();
    tmr::tfence_after();
    // lane quadrant of the warp, column half, the team's 64 columns
    const uint32_t tl = *tslot + ((uint32_t)(32 * (w & 3)) << 16) + 256u * h + 64u * team;
    auto team_sync_tmem = [&]() {                // TMEM accesses of the team's warps ordered across it
        tmr::tm_wait_st();
        tmr::tfence_before();
        tmr::team_bar(team);
        tmr::tfence_after();
    };

    // the team as a virtual CTA: schedule slots v + j G4 (recomputed from the special registers where
    // needed, so they need not stay live in registers)
    auto vslot = [&](uint32_t j) { return 4 * blockIdx.x + (threadIdx.x >> 8) + j * 4 * gridDim.x; };
    const uint32_t nrow = rows > vslot(0) ? (rows - vslot(0) + 4 * gridDim.x - 1) / (4 * gridDim.x) : 0;
    auto limb_of = [&](uint32_t j) {
        const uint32_t sr = vslot(j), nb = a.nb_total ? a.nb_total : rows / a.L;
        return a.limb_major ? sr / nb : sr % a.L;
    };
    auto row_of = [&](uint32_t j) {
        const uint32_t sr = vslot(j), nb = a.nb_total ? a.nb_total : rows / a.L;
        TM_ASSERT(sr < nb * a.L);                // a schedule slot of the batch
        if (!a.limb_major) return sr;
        const uint32_t lb = sr / nb;
        return (sr - lb * nb) * a.L + lb;
    };

    if (nrow > 0) {
        uint32_t lbc = limb_of(0), rwc = row_of(0);
        uint32_t lbn = nrow > 1 ? limb_of(1) : 0, rwn = nrow > 1 ? row_of(1) : 0;
        uint32_t u = 0;                              // the team's sub-row counter (twiddle / buffer parity)
        if constexpr (FWD) {
            const uint32_t mtot = 2 * nrow;          // column steps of the team (8 passes each)
            // step m: row m / 2, passes 8 (m & 1) .. + 7 -- one 3-D box {256 columns, 8 passes, 2 lines}
            auto issue_step = [&](uint32_t m, uint32_t prow) {   // team thread 0
                fence_proxy_async();
                mb_expect(tbar + (m & 1), 8 * R * TT * 4);
                tma3_load_hint(SB(m), &tm_in, 0, 8 * (int)(m & 1), (int)(prow * R), tbar + (m & 1),
                               l2_evict_first_policy());
            };
            // qv = (q, 2q) of the limb, loaded once per row by the caller (as in ntt_tmr.cuh)
            auto colstep = [&](uint32_t m, uint32_t limb, uint2 qv) {   // layer 0 of 8 passes into slot (m / 2) & 1
                LimbConst lc;
                lc.q = qv.x; lc.q2 = qv.y;
                const uint2 w0 = __ldg(a.tw + ((size_t)limb << LOGN) + 1);
                mb_wait(tbar + (m & 1), (m >> 1) & 1);
                const uint32_t* B = SB(m);
                uint32_t x[16];                          // cells 2p + k of the 8 passes: 16 contiguous columns
#pragma unroll
                for (int q = 0; q < 8; ++q) {
                    x[2 * q] = B[q * TT + t];
                    x[2 * q + 1] = B[8 * TT + q * TT + t];
                    ct_bfly(x[2 * q], x[2 * q + 1], w0, lc.q, lc.q2);
                }
                tmr::tm_st16(tl + SLOT * ((m >> 1) & 1) + 16 * (m & 1), x);
            };

            if (t == 0) {
                issue_step(0, rwc);
                if (1 < mtot) issue_step(1, rwc);
            }
            tmr::tw_fwd<A>(TWB(0), a.tw + ((size_t)lbc << LOGN), 0, t);
            cp_async_commit();
#pragma unroll 1
            for (uint32_t m = 0; m < 2; ++m) {       // prologue: row 0's column passes
                colstep(m, lbc, __ldg(reinterpret_cast<const uint2*>(a.lc + lbc)));
                team_sync_tmem();
                if (t == 0 && m + 2 < mtot) issue_step(m + 2, rwn);
            }
#pragma unroll 1
            for (uint32_t j = 0; j < nrow; ++j) {
                const bool more = j + 1 < nrow;
                const uint32_t r2 = j + 2 < nrow ? row_of(j + 2) : 0;
                const uint2 qc = __ldg(reinterpret_cast<const uint2*>(a.lc + lbc));   // (q, 2q) of rows j, j + 1
                const uint2 qn = __ldg(reinterpret_cast<const uint2*>(a.lc + lbn));
#pragma unroll 1
                for (int s = 0; s < R; ++s, ++u) {
                    LimbConst lc;                        // the row stages use q, 2q only
                    lc.q = qc.x; lc.q2 = qc.y;
                    const uint2* __restrict__ tw = a.tw + ((size_t)lbc << LOGN);
                    uint32_t* S = B0;
                    // ---- R1(j, s): stage 1 (layers 1..4, thread (b, c), elements a) from slot j & 1
                    cp_async_wait<0>();
                    __syncwarp();                        // this warp's stage-1 twiddles landed
                    uint32_t x[16];
                    tms::ld16_stride<R>(tl + SLOT * (j & 1) + s, x);
                    {
                        const uint2* W = TWB(u & 1) + 16 * w;
                        fwd16_sp(x, W, W + 2, W + 4, W + 8, lc.q, lc.q2);
                        if (u > 0) mb_wait(tbar + 2, (u - 1) & 1);   // every warp done with sub-row u - 1
#pragma unroll
                        for (int k = 0; k < 16; ++k) S[v8_phys(k, hi4, lo4)] = x[k];
                    }
                    // ---- C(j+1, passes 8s .. 8s+7)
                    const uint32_t m = 2 * (j + 1) + s;
                    if (more) colstep(m, lbn, qn);
                    team_sync_tmem();                    // stage 1, the step's passes done team-wide
                    if (t == 0 && more && m + 2 < mtot) issue_step(m + 2, r2);
                    {   // the team's next sub-row's twiddles
                        const uint32_t nj = s + 1 < R ? j : j + 1, ns = s + 1 < R ? s + 1 : 0;
                        if (nj < nrow) tmr::tw_fwd<A>(TWB((u + 1) & 1), a.tw + ((size_t)(nj == j ? lbc : lbn) << LOGN), ns, t);
                        cp_async_commit();
                    }
                    // ---- R23(j, s)
                    const uint32_t qq = lc.q, q2 = lc.q2;
                    uint32_t* out = a.out + ((size_t)rwc << LOGN) + s * SUBW;
                    uint2 w3[15];
                    load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                    tmr::fwd_stages23(S, x, TWB(u & 1) + 128, w3, qq, q2, out, t, tbar + 2);
                }
                lbc = lbn; rwc = rwn;
                if (j + 2 < nrow) { lbn = limb_of(j + 2); rwn = r2; }
            }
        } else {
            // sub-row s of row jr: stages 3', 2' (team barrier) stage 1' into slot jr & 1
            auto rowpass = [&](uint32_t jr, int s, uint32_t limb, uint32_t row_self, uint32_t limb_next,
                               uint32_t row_next) {
                const LimbConst lc = a.lc[limb];
                const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
                uint32_t* S = (u & 1) ? B1 : B0;
                uint2 w3[15];
                load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                cp_async_wait<0>();
                __syncwarp();                            // this warp's slice of the sub-row landed
                uint32_t x[16];
                tmr::inv_stages32(S, x, w3, TWB(u & 1), lc, t);
                tmr::team_bar(team);                     // stage 2' done team-wide; the other buffer is free
                {   // the team's next sub-row: data and twiddles into the other buffer
                    uint32_t nj = jr, ns = (uint32_t)s + 1, nl = limb, nr = row_self;
                    if (ns >= (uint32_t)R) { nj = jr + 1; ns = 0; nl = limb_next; nr = row_next; }
                    if (nj < nrow) {
                        tmr::tw_inv<A>(TWB((u + 1) & 1), a.tw + ((size_t)nl << LOGN), ns, t);
                        tmr::load_inv_slice((u & 1) ? B0 : B1, a.in + ((size_t)nr << LOGN) + ns * SUBW, t);
                    }
                    cp_async_commit();
                }
                {   // stage 1': layers A+3..A, thread (b, c), elements a -> TMEM (lazy, in [0, 2q))
                    tmr::inv_stage1(S, x, TWB(u & 1), lc, t);
                    tms::st16_stride<R>(tl + SLOT * (jr & 1) + s, x);
                }
                ++u;
            };
            // passes 8i .. 8i+7 of row j: layer 0 with N^-1, canonical output
            auto colstep = [&](uint32_t j, int i, uint32_t limb, uint32_t row) {
                const LimbConst lc = a.lc[limb];
                uint32_t* o = a.out + ((size_t)row << LOGN) + 8 * i * TT + t;
                uint32_t x[16];                          // cells 2p + k of the 8 passes: 16 contiguous columns
                tmr::tm_ld16(tl + SLOT * (j & 1) + 16 * i, x);
#pragma unroll
                for (int q = 0; q < 8; ++q) {
                    gs_bfly_last(x[2 * q], x[2 * q + 1], lc);
                    __stcs(o + q * TT, canon2(x[2 * q], lc.q));
                    __stcs(o + SUBW + q * TT, canon2(x[2 * q + 1], lc.q));
                }
            };

            tmr::tw_inv<A>(TWB(0), a.tw + ((size_t)lbc << LOGN), 0, t);
            tmr::load_inv_slice(B0, a.in + ((size_t)rwc << LOGN), t);
            cp_async_commit();
#pragma unroll 1
            for (int s = 0; s < R; ++s) rowpass(0, s, lbc, rwc, lbn, rwn);
#pragma unroll 1
            for (uint32_t j = 0; j < nrow; ++j) {
                const bool more = j + 1 < nrow;
                const uint32_t lb2 = j + 2 < nrow ? limb_of(j + 2) : 0, rw2 = j + 2 < nrow ? row_of(j + 2) : 0;
                team_sync_tmem();                        // row j in TMEM (every warp's stage 1')
#pragma unroll 1
                for (int i = 0; i < R; ++i) {
                    colstep(j, i, lbc, rwc);
                    if (more) rowpass(j + 1, i, lbn, rwn, lb2, rw2);   // refills slot (j + 1) & 1
                }
                lbc = lbn; rwc = rwn; lbn = lb2; rwn = rw2;
            }
        }
    }
    cp_async_wait<0>();
    tmr::tfence_before();
    __syncthreads();
    if (threadIdx.x < 32) {
        tmr::tfence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(*tslot));
    }
}

}  // namespace tmt
}  // namespace wd
