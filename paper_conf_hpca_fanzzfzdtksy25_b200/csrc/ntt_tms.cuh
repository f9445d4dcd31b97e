// ntt_tms.cuh -- "tm" for N = 2^14 and 2^15: TMEM-resident rows with two row slots (SURVEY.md 8 rows
// a2-a4, a6-a8).
//
// The N = 2^16 kernel (ntt_tmr.cuh) fills the whole tensor memory with one row and therefore recycles
// cells through a two-layout ping-pong.  A row of N = R x 4096 with R = 4 or 8 takes 16 R cells per
// (lane, column half), so two rows fit side by side: row j lives in slot j & 1 with one fixed layout,
//   cell (column pass p, element k) of thread t -> TMEM lane t % 128, column 256 h + 16 R (j & 1) + R p + k,
// (h = t / 128).  A column pass writes its R elements as one contiguous tcgen05.st (.x4 / .x8); stage 1 of
// sub-row s reads its 16 elements (a, s), a = 0..15, with 16 strided .x1 loads, as in the N = 2^16 kernel.
// Everything else is v8's decomposition with A = log2 R column layers (ntt_v8.cuh) and the team scheme
// of ntt_tmr.cuh: one CTA per SM, four teams of 256 threads; team tau owns sub-rows tau + 4 i (R / 4 of
// them per row) and column passes tau + 4 i (four per row, in steps of 16 / R passes per sub-row).
//   forward, row j:  R1(j, s) [stage 1 from slot j & 1]  C(j+1, ...) [TMA staging -> layers 0..A-1 ->
//                    slot (j+1) & 1]  team barrier  R23(j, s) [stages 2, 3 -> out]
//   inverse, row j:  C'(j, ...) [slot j & 1 -> layers A-1..0 with N^-1 -> out]  R'(j+1, s) [cp.async ->
//                    stages 3', 2' -> team barrier -> stage 1' -> slot (j+1) & 1]
// Two CTA mbarriers order the row handoff (every column pass / sub-row of row j is in TMEM before it is
// read) and the slot reuse (every warp has read row j - 1 before row j + 1 overwrites its slot), so
// teams may drift apart by up to a row.
#pragma once
#include "ntt_tmr.cuh"

namespace wd {
namespace tms {

using tmr::TEAMS; using tmr::TT; using tmr::NT; using tmr::SUBW; using tmr::TWW; using tmr::TEAM_W;
constexpr int SMEM = TEAMS * TEAM_W * 4 + 320;   // + 9 mbarriers per team, 2 CTA mbarriers, the TMEM slot

// 16 cells at column offsets ta + R a, a = 0..15 (complete on return: the wait carries x as in/out
// operands, so no use of x is scheduled before it)
// (the column offset is an immediate of each access: one template instance per cell)
template <int R, int I>
__device__ __forceinline__ void ld1_at(uint32_t ta, uint32_t* x) {
    if constexpr (I < 16) {
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1+%2];" : "=r"(x[I]) : "r"(ta), "n"(R * I));
        ld1_at<R, I + 1>(ta, x);
    }
}
template <int R, int I>
__device__ __forceinline__ void st1_at(uint32_t ta, const uint32_t* x) {
    if constexpr (I < 16) {
        asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+%1], {%2};" :: "r"(ta), "n"(R * I), "r"(x[I]) : "memory");
        st1_at<R, I + 1>(ta, x);
    }
}
template <int R>
__device__ __forceinline__ void ld16_stride(uint32_t ta, uint32_t* x) {
    tmr::tm_check(ta, 15 * R + 1);
    ld1_at<R, 0>(ta, x);
    asm volatile("tcgen05.wait::ld.sync.aligned;"
                 : "+r"(x[0]), "+r"(x[1]), "+r"(x[2]), "+r"(x[3]), "+r"(x[4]), "+r"(x[5]), "+r"(x[6]), "+r"(x[7]),
                   "+r"(x[8]), "+r"(x[9]), "+r"(x[10]), "+r"(x[11]), "+r"(x[12]), "+r"(x[13]), "+r"(x[14]), "+r"(x[15])
                 :: "memory");
}
template <int R>
__device__ __forceinline__ void st16_stride(uint32_t ta, const uint32_t* x) {
    tmr::tm_check(ta, 15 * R + 1);
    st1_at<R, 0>(ta, x);
}
// R contiguous cells
template <int R>
__device__ __forceinline__ void stR(uint32_t ta, const uint32_t* x) {
    tmr::tm_check(ta, R);
    if constexpr (R == 8)
        asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
                     :: "r"(ta), "r"(x[0]), "r"(x[1]), "r"(x[2]), "r"(x[3]), "r"(x[4]), "r"(x[5]), "r"(x[6]), "r"(x[7])
                     : "memory");
    else
        asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1,%2,%3,%4};"
                     :: "r"(ta), "r"(x[0]), "r"(x[1]), "r"(x[2]), "r"(x[3]) : "memory");
}
template <int R>
__device__ __forceinline__ void ldR(uint32_t ta, uint32_t* x) {
    tmr::tm_check(ta, R);
    if constexpr (R == 8)
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n\t"
                     "tcgen05.wait::ld.sync.aligned;"
                     : "=r"(x[0]), "=r"(x[1]), "=r"(x[2]), "=r"(x[3]), "=r"(x[4]), "=r"(x[5]), "=r"(x[6]), "=r"(x[7])
                     : "r"(ta) : "memory");
    else
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0,%1,%2,%3}, [%4];\n\t"
                     "tcgen05.wait::ld.sync.aligned;"
                     : "=r"(x[0]), "=r"(x[1]), "=r"(x[2]), "=r"(x[3]) : "r"(ta) : "memory");
}

template <int A, bool FWD>
__global__ void __launch_bounds__(NT, 1) ntt_tms(NttArgs a, uint32_t rows, const __grid_constant__ CUtensorMap tm_in) {
    constexpr int LOGN = 12 + A, R = 1 << A;
    static_assert(A == 2 || A == 3, "N = 2^14, 2^15");
    constexpr int NST = R / 4;                   // sub-rows per team and row
    constexpr int PPS = 16 / R;                  // column passes per sub-row step (4 per team and row)
    constexpr int NB = 2 * PPS;                  // forward staging buffers per team (R KB each, 32 KB)
    constexpr int SLOT = 16 * R;                 // TMEM columns of one row per (lane, half)
    extern __shared__ __align__(1024) uint32_t smem[];
    const int team = (int)(threadIdx.x >> 8), t = (int)(threadIdx.x & (TT - 1));
    const int w = t >> 5, h = w >> 2, hi4 = t >> 4, lo4 = t & 15, lane = t & 31;
    uint32_t* TS = smem + team * TEAM_W;
    uint32_t* const B0 = TS;                     // forward: sub-row exchange; inverse: input buffer 0
    uint32_t* const B1 = TS + SUBW;              // inverse: input buffer 1
    auto SB = [&](uint32_t m) { return TS + SUBW + (m % NB) * (R * TT); };   // forward staging of pass m
    auto TWB = [&](int b) { return reinterpret_cast<uint2*>(TS + 3 * SUBW + b * TWW); };
    // per team: tbar[0..NB-1] the forward TMA stagings, tbar[8] "B0 free"
    uint64_t* tbar = reinterpret_cast<uint64_t*>(smem + TEAMS * TEAM_W) + 9 * team;
    // CTA: rowbar "every warp's part of row r is in TMEM", slotbar "every warp has read row r's slot"
    uint64_t* rowbar = reinterpret_cast<uint64_t*>(smem + TEAMS * TEAM_W) + 9 * TEAMS;
    uint64_t* slotbar = rowbar + 1;
    uint32_t* tslot = reinterpret_cast<uint32_t*>(rowbar + 2);

    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(smem_u32(tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (t == 0) {
        for (int i = 0; i < NB; ++i) mb_init(tbar + i, 1);
        mb_init(tbar + 8, TT / 32);
        if (team == 0) { mb_init(rowbar, NT / 32); mb_init(slotbar, NT / 32); }
        mb_init_fence();
    }
    tmr::tfence_before();
    __syncthreads();
    tmr::tfence_after();
    const uint32_t tl = *tslot + ((uint32_t)(32 * (w & 3)) << 16) + 256u * h;   // lane quadrant, column half
    // this warp's earlier TMEM accesses are complete and ordered before its arrival on b
    auto warp_arrive_tmem = [&](uint64_t* b) {
        tmr::tm_wait_st();
        tmr::tfence_before();
        __syncwarp();
        if (lane == 0) mb_arrive(b);
    };
    auto wait_tmem = [&](uint64_t* b, uint32_t r) {   // phase r of b completed; later TMEM accesses after it
        mb_wait(b, r & 1);
        tmr::tfence_after();
    };

    const uint32_t G = gridDim.x;
    const uint32_t nrow = rows > blockIdx.x ? (rows - blockIdx.x + G - 1) / G : 0;
    const uint32_t nb = a.nb_total ? a.nb_total : rows / a.L;   // polynomials of the schedule
    auto limb_of = [&](uint32_t j) {
        const uint32_t sr = blockIdx.x + j * G;
        return a.limb_major ? sr / nb : sr % a.L;
    };
    auto row_of = [&](uint32_t j) {
        const uint32_t sr = blockIdx.x + j * G;
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
            const uint32_t mtot = 4 * nrow;          // column passes of the team
            // pass m of the team: row m / 4, column pass p = team + 4 (m % 4); staging m % NB, mbarrier m % NB
            auto issue_col = [&](uint32_t m, uint32_t prow) {   // team thread 0
                fence_proxy_async();
                mb_expect(tbar + m % NB, R * TT * 4);
                tma2_load_hint(SB(m), &tm_in, (team + 4 * (int)(m & 3)) * TT, (int)(prow * R), tbar + m % NB,
                               l2_evict_first_policy());
            };
            // qv = (q, 2q) of the limb, loaded once per row by the caller (as in ntt_tmr.cuh)
            auto colpass = [&](uint32_t m, uint32_t limb, uint2 qv) {   // layers 0..A-1 of pass m into slot (m / 4) & 1
                const int p = team + 4 * (int)(m & 3);
                LimbConst lc;
                lc.q = qv.x; lc.q2 = qv.y;
                const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
                mb_wait(tbar + m % NB, (m / NB) & 1);
                const uint32_t* B = SB(m);
                uint32_t x[R];
#pragma unroll
                for (int k = 0; k < R; ++k) x[k] = B[k * TT + t];
                fwd_radix<A>(x, tw, 0, 0, lc.q, lc.q2);
                stR<R>(tl + SLOT * ((m >> 2) & 1) + R * p, x);
            };
            // the TMAs of the team's first 2 PPS passes, then row 0's passes in PPS-pass steps
            if (t == 0)
                for (uint32_t m = 0; m < (uint32_t)NB && m < mtot; ++m) issue_col(m, (m >> 2) == 0 ? rwc : rwn);
            tmr::tw_fwd<A>(TWB(0), a.tw + ((size_t)lbc << LOGN), team, t);
            cp_async_commit();
#pragma unroll 1
            for (uint32_t m0 = 0; m0 < 4; m0 += PPS) {
#pragma unroll 1
                for (uint32_t q = 0; q < (uint32_t)PPS; ++q) colpass(m0 + q, lbc, __ldg(reinterpret_cast<const uint2*>(a.lc + lbc)));
                tmr::team_bar(team);
                if (t == 0)
                    for (uint32_t q = 0; q < (uint32_t)PPS; ++q) {
                        const uint32_t mm = m0 + NB + q;
                        if (mm < mtot) issue_col(mm, (mm >> 2) == 0 ? rwc : (mm >> 2) == 1 ? rwn : row_of(mm >> 2));
                    }
            }
            warp_arrive_tmem(rowbar);                    // this warp's passes of row 0 are in TMEM
#pragma unroll 1
            for (uint32_t j = 0; j < nrow; ++j) {
                const bool more = j + 1 < nrow;
                const uint32_t r2 = j + 2 < nrow ? row_of(j + 2) : 0;
                const uint32_t r3 = j + 3 < nrow ? row_of(j + 3) : 0;
                const uint2 qc = __ldg(reinterpret_cast<const uint2*>(a.lc + lbc));   // (q, 2q) of rows j, j + 1
                const uint2 qn = __ldg(reinterpret_cast<const uint2*>(a.lc + lbn));
#pragma unroll 1
                for (int i = 0; i < NST; ++i, ++u) {
                    const int s = team + 4 * i;
                    LimbConst lc;                        // the row stages use q, 2q only
                    lc.q = qc.x; lc.q2 = qc.y;
                    const uint2* __restrict__ tw = a.tw + ((size_t)lbc << LOGN);
                    uint32_t* S = B0;
                    // ---- R1(j, s): stage 1 (layers A..A+3, thread (b, c), elements a) from slot j & 1
                    cp_async_wait<0>();
                    __syncwarp();                        // this warp's stage-1 twiddles landed
                    uint32_t x[16];
                    if (i == 0) wait_tmem(rowbar, j);    // every column pass of row j is in TMEM
                    ld16_stride<R>(tl + SLOT * (j & 1) + s, x);
                    {
                        const uint2* W = TWB(u & 1) + 16 * w;
                        fwd16_sp(x, W, W + 2, W + 4, W + 8, lc.q, lc.q2);
                        if (u > 0) mb_wait(tbar + 8, (u - 1) & 1);   // every warp done with sub-row u - 1
#pragma unroll
                        for (int k = 0; k < 16; ++k) S[v8_phys(k, hi4, lo4)] = x[k];
                    }
                    // ---- C(j+1, ...): the step's PPS column passes of the next row
                    const uint32_t m0 = 4 * (j + 1) + i * PPS;
                    if (more) {
                        // slot (j + 1) & 1 last held row j - 1: every warp has read it
                        if (i == 0 && j > 0) wait_tmem(slotbar, j - 1);
#pragma unroll 1
                        for (uint32_t q = 0; q < (uint32_t)PPS; ++q) colpass(m0 + q, lbn, qn);
                        if (i == NST - 1) warp_arrive_tmem(rowbar);   // this warp's passes of row j + 1
                    }
                    tmr::team_bar(team);                 // stage 1 (and the step's passes) done team-wide
                    // this warp's reads of row j's slot are done (arrived only after this row's slot wait,
                    // so a waiter never sees the barrier two phases ahead)
                    if (i == NST - 1) warp_arrive_tmem(slotbar);
                    if (t == 0 && more)
                        for (uint32_t q = 0; q < (uint32_t)PPS; ++q) {
                            const uint32_t mm = m0 + NB + q;
                            if (mm < mtot) {
                                const uint32_t rr = mm >> 2;
                                issue_col(mm, rr == j + 1 ? rwn : rr == j + 2 ? r2 : r3);
                            }
                        }
                    {   // the team's next sub-row's twiddles
                        uint32_t nj = j, ns = (uint32_t)s + TEAMS;
                        if (i + 1 >= NST) { nj = j + 1; ns = team; }
                        if (nj < nrow) tmr::tw_fwd<A>(TWB((u + 1) & 1), a.tw + ((size_t)(nj == j ? lbc : lbn) << LOGN), ns, t);
                        cp_async_commit();
                    }
                    // ---- R23(j, s)
                    const uint32_t qq = lc.q, q2 = lc.q2;
                    uint32_t* out = a.out + ((size_t)rwc << LOGN) + s * SUBW;
                    uint2 w3[15];
                    load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                    tmr::fwd_stages23(S, x, TWB(u & 1) + 128, w3, qq, q2, out, t, tbar + 8);
                }
                lbc = lbn; rwc = rwn;
                if (j + 2 < nrow) { lbn = limb_of(j + 2); rwn = r2; }
            }
        } else {
            // sub-row s of row jr: stages 3', 2' (team barrier) stage 1' into slot jr & 1
            auto rowpass = [&](uint32_t jr, int s, uint32_t limb, uint32_t row_self, uint32_t limb_next,
                               uint32_t row_next, int i) {
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
                    uint32_t nj = jr, ns = (uint32_t)s + TEAMS, nl = limb, nr = row_self;
                    if (i + 1 >= NST) { nj = jr + 1; ns = team; nl = limb_next; nr = row_next; }
                    if (nj < nrow) {
                        tmr::tw_inv<A>(TWB((u + 1) & 1), a.tw + ((size_t)nl << LOGN), ns, t);
                        tmr::load_inv_slice((u & 1) ? B0 : B1, a.in + ((size_t)nr << LOGN) + ns * SUBW, t);
                    }
                    cp_async_commit();
                }
                {   // stage 1': layers A+3..A, thread (b, c), elements a -> TMEM (lazy, in [0, 2q))
                    tmr::inv_stage1(S, x, TWB(u & 1), lc, t);
                    st16_stride<R>(tl + SLOT * (jr & 1) + s, x);
                }
                ++u;
            };
            // column pass p of row j: layers A-1..0 with N^-1, canonical output
            auto colpass = [&](uint32_t j, int p, uint32_t limb, uint32_t row) {
                const LimbConst lc = a.lc[limb];
                const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
                uint32_t x[R];
                ldR<R>(tl + SLOT * (j & 1) + R * p, x);
                inv_radix<A, true>(x, tw, 0, 0, lc);
                uint32_t* o = a.out + ((size_t)row << LOGN) + p * TT + t;
#pragma unroll
                for (int k = 0; k < R; ++k) __stcs(o + k * SUBW, canon2(x[k], lc.q));
            };

            tmr::tw_inv<A>(TWB(0), a.tw + ((size_t)lbc << LOGN), team, t);
            tmr::load_inv_slice(B0, a.in + ((size_t)rwc << LOGN) + team * SUBW, t);
            cp_async_commit();
#pragma unroll 1
            for (int i = 0; i < NST; ++i) rowpass(0, team + 4 * i, lbc, rwc, lbn, rwn, i);
            warp_arrive_tmem(rowbar);                    // this warp's sub-rows of row 0 are in TMEM
#pragma unroll 1
            for (uint32_t j = 0; j < nrow; ++j) {
                const bool more = j + 1 < nrow;
                const uint32_t lb2 = j + 2 < nrow ? limb_of(j + 2) : 0, rw2 = j + 2 < nrow ? row_of(j + 2) : 0;
#pragma unroll 1
                for (int i = 0; i < NST; ++i) {
                    if (i == 0) wait_tmem(rowbar, j);    // every sub-row of row j is in TMEM
#pragma unroll 1
                    for (int q = 0; q < PPS; ++q) colpass(j, team + 4 * (i * PPS + q), lbc, rwc);
                    if (more) {
                        // slot (j + 1) & 1 last held row j - 1: every warp has read it
                        if (i == 0 && j > 0) wait_tmem(slotbar, j - 1);
                        rowpass(j + 1, team + 4 * i, lbn, rwn, lb2, rw2, i);
                    }
                }
                // this warp's sub-rows of row j + 1 are in TMEM, and its reads of row j are done (both
                // arrivals after this row's waits, so a waiter never sees a barrier two phases ahead)
                if (more) warp_arrive_tmem(rowbar);
                warp_arrive_tmem(slotbar);
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

}  // namespace tms
}  // namespace wd
