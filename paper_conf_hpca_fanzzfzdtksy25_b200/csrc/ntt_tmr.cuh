// ntt_tmr.cuh -- "tm": the TMEM-resident CUDA-core NTT, N = 2^16.
//
// Same butterfly network and decomposition as v8 (ntt_v8.cuh: N = 16 x 4096, layers 0..3 on the 4096
// columns of 16 elements, layers 4..15 as three radix-16 register stages on the 16 contiguous 4096-word
// sub-rows; merged-psi CT, PAPER.md:85-91 with reading C-1), but the phase-1 <-> phase-2 intermediate
// never leaves the SM: a whole row (2^16 words = 256 KB) sits in the SM's tensor memory (TMEM, 128
// lanes x 512 columns x 32 bit), which the CUDA-core NTT otherwise leaves idle.  v8 keeps it in the
// row's output slot in L2 instead, with a 2-CTA cluster per row and a cluster barrier between the
// phases; here there is no L2 round trip, no cluster and no excess DRAM traffic.
//
// One persistent CTA per SM (1024 threads = 4 teams of 256).  Team tau owns sub-rows / column passes
// s = tau, tau+4, tau+8, tau+12 of every row.  Team thread t (warp w = t/32, h = t/128) uses TMEM lane
// t % 128 -- its own warp's lane quadrant (w % 4) -- and half h of the lane's columns:
//   column pass p, thread t: column c = 256 p + t, elements k = 0..15 (x[k*4096 + c])
//   sub-row s, stage 1, thread t: elements a*256 + t of sub-row s, a = 0..15, i.e. (k = s, c = 256 a + t)
// so stage 1 of sub-row s reads exactly what column pass a = 0..15 of the same thread index t wrote:
// TMEM cell (lane t % 128, column col(p, k, h)).  Two layouts alternate from row to row,
//   A: col(p, k, h) = 32 k + 16 h + p          B: col(p, k, h) = 32 p + 16 h + k,
// so that the 32 cells sub-row s of row j has consumed are exactly the cells column pass s of row j+1
// writes, by the same thread (forward; the inverse mirrors it).  A team therefore interleaves, for its
// four s,
//   forward:  R1(j, s) [stage 1 from TMEM]  C(j+1, s) [column pass into the cells R1 just read]  team
//             barrier  R23(j, s); rows hand over through a CTA mbarrier (arrive after a warp's last
//             column pass of row j+1, wait before its first stage-1 read of that row),
//   inverse:  C'(j, s) R'(j+1, s) [stages 3', 2', team barrier, stage 1' into the cells C' read], then
//             one CTA barrier per row,
// the classic in-place ping-pong.  In each row one of the two accesses is 16 contiguous columns (one
// tcgen05.ld/st .x16), the other 16 strided ones (.x1).  The column pass between stage 1 and the
// stage-1 barrier covers that barrier's wait.
// Forward column passes are fed by TMA (one 256 x 16 box per pass, two staging buffers per team, issued
// two passes ahead); inverse sub-rows by 16-byte cp.async, double-buffered as in v8; forward outputs
// leave by coalesced 512-byte STG from the sub-row buffer, inverse outputs straight from registers
// (128-byte lines per warp).  Ablations and measurements: DESIGN.md 5.1a.
#pragma once
#include "ntt_v8.cuh"

namespace wd {
namespace tmr {

constexpr int TEAMS = 4, TT = 256, NT = TEAMS * TT;
constexpr int SUBW = 4096;
constexpr int TWW = 768;                        // words per twiddle area (<= 384 (w, w') pairs)
// per team: three sub-row buffers (forward: the sub-row exchange and two TMA column stagings; inverse:
// two input buffers), two twiddle areas
constexpr int TEAM_W = 3 * SUBW + 2 * TWW;
constexpr int SMEM = TEAMS * TEAM_W * 4 + 128;  // + 3 mbarriers per team, the row mbarrier, the TMEM slot

// ---------------------------------------------------------------- debug checks (compute-sanitizer is closed
// on the GPU pool this round): a -DWD_TM_DEBUG build traps on a TMEM access outside the warp's lane
// quadrant or the 512 allocated columns, on a row index outside the batch, and on an mbarrier wait that
// does not complete (tma.cuh); tests/test_gpu_parity.py runs the tm shapes against it
#ifdef WD_TM_DEBUG
#define TM_ASSERT(c) do { if (!(c)) __trap(); } while (0)
#else
#define TM_ASSERT(c) do { } while (0)
#endif
// a TMEM access of `span` consecutive columns from ta by this thread's warp
__device__ __forceinline__ void tm_check(uint32_t ta, uint32_t span) {
    TM_ASSERT((ta >> 16) == 32u * ((threadIdx.x >> 5) & 3));
    TM_ASSERT((ta & 0xFFFFu) + span <= 512u);
    (void)ta; (void)span;
}

// ---------------------------------------------------------------- tensor memory
__device__ __forceinline__ void tfence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tfence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tm_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
// 16 consecutive columns of the warp's lanes -> x[0..15]; complete on return (wait::ld in the same asm,
// so no use of x can be scheduled before it)
__device__ __forceinline__ void tm_ld16(uint32_t ta, uint32_t* x) {
    tm_check(ta, 16);
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 "
                 "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];\n\t"
                 "tcgen05.wait::ld.sync.aligned;"
                 : "=r"(x[0]), "=r"(x[1]), "=r"(x[2]), "=r"(x[3]), "=r"(x[4]), "=r"(x[5]), "=r"(x[6]), "=r"(x[7]),
                   "=r"(x[8]), "=r"(x[9]), "=r"(x[10]), "=r"(x[11]), "=r"(x[12]), "=r"(x[13]), "=r"(x[14]), "=r"(x[15])
                 : "r"(ta) : "memory");
}
// columns ta, ta + 32, ..., ta + 480 -> x[0..15]
__device__ __forceinline__ void tm_ld16s(uint32_t ta, uint32_t* x) {
    tm_check(ta, 481);
    asm volatile("{\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%16];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%1}, [%16+32];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%2}, [%16+64];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%3}, [%16+96];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%4}, [%16+128];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%5}, [%16+160];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%6}, [%16+192];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%7}, [%16+224];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%8}, [%16+256];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%9}, [%16+288];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%10}, [%16+320];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%11}, [%16+352];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%12}, [%16+384];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%13}, [%16+416];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%14}, [%16+448];\n\t"
                 "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%15}, [%16+480];\n\t"
                 "tcgen05.wait::ld.sync.aligned;\n\t}"
                 : "=r"(x[0]), "=r"(x[1]), "=r"(x[2]), "=r"(x[3]), "=r"(x[4]), "=r"(x[5]), "=r"(x[6]), "=r"(x[7]),
                   "=r"(x[8]), "=r"(x[9]), "=r"(x[10]), "=r"(x[11]), "=r"(x[12]), "=r"(x[13]), "=r"(x[14]), "=r"(x[15])
                 : "r"(ta) : "memory");
}
__device__ __forceinline__ void tm_st16(uint32_t ta, const uint32_t* x) {
    tm_check(ta, 16);
    asm volatile("tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
                 "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};"
                 :: "r"(ta), "r"(x[0]), "r"(x[1]), "r"(x[2]), "r"(x[3]), "r"(x[4]), "r"(x[5]), "r"(x[6]), "r"(x[7]),
                    "r"(x[8]), "r"(x[9]), "r"(x[10]), "r"(x[11]), "r"(x[12]), "r"(x[13]), "r"(x[14]), "r"(x[15])
                 : "memory");
}
__device__ __forceinline__ void tm_st16s(uint32_t ta, const uint32_t* x) {
    tm_check(ta, 481);
    asm volatile("{\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+32], {%2};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+64], {%3};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+96], {%4};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+128], {%5};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+160], {%6};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+192], {%7};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+224], {%8};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+256], {%9};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+288], {%10};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+320], {%11};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+352], {%12};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+384], {%13};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+416], {%14};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+448], {%15};\n\t"
                 "tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+480], {%16};\n\t}"
                 :: "r"(ta), "r"(x[0]), "r"(x[1]), "r"(x[2]), "r"(x[3]), "r"(x[4]), "r"(x[5]), "r"(x[6]), "r"(x[7]),
                    "r"(x[8]), "r"(x[9]), "r"(x[10]), "r"(x[11]), "r"(x[12]), "r"(x[13]), "r"(x[14]), "r"(x[15])
                 : "memory");
}

__device__ __forceinline__ void team_bar(int team) {
    asm volatile("bar.sync %0, %1;" :: "r"(team + 1), "n"(TT) : "memory");
}
// every TMEM store of this thread done and ordered before the CTA barrier; TMEM reads after it ordered
// after it (PTX tcgen05 memory-consistency rules)
__device__ __forceinline__ void cta_sync_tmem() {
    tm_wait_st();
    tfence_before();
    __syncthreads();
    tfence_after();
}

// twiddles of one sub-row, staged by cp.async (team thread t; no commit): v8_tw_fwd / v8_tw_inv with
// the team-local thread index
template <int A>
__device__ __forceinline__ void tw_fwd(uint2* TW, const uint2* __restrict__ tw, uint32_t s, int t) {
    const int w = t >> 5, l = t & 31;
    if (l < 15) {
        const int k = 31 - __clz(l + 1), g = l - ((1 << k) - 1);
        cp_async8(TW + 16 * w + (k ? (1 << k) : 0) + g, tw + (1u << (A + k)) + (s << k) + g);
    }
    if (t < 240) {
        const int k = 31 - __clz((t >> 4) + 1), g = t - 16 * ((1 << k) - 1);
        cp_async8(TW + 128 + 16 * ((1 << k) - 1) + g, tw + (16u << (A + k)) + ((s * 16) << k) + g);
    }
}
template <int A>
__device__ __forceinline__ void tw_inv(uint2* TW, const uint2* __restrict__ tw, uint32_t s, int t) {
    const int w = t >> 5, l = t & 31;
    if (l < 30) {
        const int k = 31 - __clz((l >> 1) + 1), g = l - 2 * ((1 << k) - 1);
        cp_async8(TW + 32 * w + 2 * ((1 << k) - 1) + g, tw + (16u << (A + k)) + ((s * 16 + 2 * w) << k) + g);
    }
    if (t < 15) {
        const int k = 31 - __clz(t + 1), g = t - ((1 << k) - 1);
        cp_async8(TW + 256 + (k ? (1 << k) : 0) + g, tw + (1u << (A + k)) + (s << k) + g);
    }
}
// inverse sub-row slice (stage 3' reads of warp w: words 512w .. 512w+511), no commit
__device__ __forceinline__ void load_inv_slice(uint32_t* S, const uint32_t* src, int t) {
    const int w = t >> 5, l = t & 31;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const int e = 512 * w + 4 * (32 * k + l);
        cp_async16(S + v8_phys(e >> 8, (e >> 4) & 15, e & 15), src + e);
    }
}

// the forward twiddle areas / stage bodies shared by the two directions are written out in each branch
// ---------------------------------------------------------------- row-phase stages shared by the tm kernels
// v8's sub-row layout (ntt_v8.cuh v8_phys) in a 4096-word shared-memory buffer S; team thread t.
// Forward stages 2 (twiddles T2 = the sub-row's stage-2 area) and 3 (twiddles w3), then the coalesced
// canonical store of the sub-row to out and this warp's arrival on b0free (its last read of S).
__device__ __forceinline__ void fwd_stages23(uint32_t* S, uint32_t* x, const uint2* T2, const uint2* w3, uint32_t q,
                                             uint32_t q2, uint32_t* out, int t, uint64_t* b0free) {
    const int hi4 = t >> 4, lo4 = t & 15, w = t >> 5, lane = t & 31;
    {   // stage 2: thread (a, c), elements b
        const int aa = hi4, c = lo4;
#pragma unroll
        for (int k = 0; k < 16; ++k) x[k] = S[v8_phys(aa, k, c)];
        fwd16_sp(x, T2 + aa, T2 + 16 + 2 * aa, T2 + 48 + 4 * aa, T2 + 112 + 8 * aa, q, q2);
#pragma unroll
        for (int k = 0; k < 16; ++k) S[v8_phys(aa, k, c)] = x[k];
    }
    __syncwarp();
    {   // stage 3: thread (a, b), 16 contiguous elements; coalesced store through the warp's own slots
        const int aa = hi4, b = lo4;
        uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
        const int sw = (b >> 1) & 3;
#pragma unroll
        for (int v = 0; v < 4; ++v) {
            const uint4 r = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
            x[4 * v] = r.x; x[4 * v + 1] = r.y; x[4 * v + 2] = r.z; x[4 * v + 3] = r.w;
        }
        fwd16_tw(x, w3, q, q2);
#pragma unroll
        for (int v = 0; v < 4; ++v)
            *reinterpret_cast<uint4*>(base + ((v ^ sw) << 2)) = make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
        __syncwarp();
        const int wbase = w * 512 + 4 * lane;
#pragma unroll
        for (int v = 0; v < 4; ++v) {
            const int e = wbase + 128 * v;
            const uint4 r = *reinterpret_cast<const uint4*>(S + v8_phys(e >> 8, (e >> 4) & 15, e & 15));
            __stcs(reinterpret_cast<uint4*>(out + e),
                   make_uint4(canon4(r.x, q, q2), canon4(r.y, q, q2), canon4(r.z, q, q2), canon4(r.w, q, q2)));
        }
        __syncwarp();
        if (lane == 0) mb_arrive(b0free);
    }
}
// Inverse stages 3' (twiddles w3) and 2' (this warp's twiddle copies in TW, tw_inv's layout) in S
__device__ __forceinline__ void inv_stages32(uint32_t* S, uint32_t* x, const uint2* w3, const uint2* TW, const LimbConst& lc,
                                             int t) {
    const int hi4 = t >> 4, lo4 = t & 15, w = t >> 5;
    {   // stage 3': thread (a, b), 16 contiguous elements
        const int aa = hi4, b = lo4;
        uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
        const int sw = (b >> 1) & 3;
#pragma unroll
        for (int v = 0; v < 4; ++v) {
            const uint4 r = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
            x[4 * v] = r.x; x[4 * v + 1] = r.y; x[4 * v + 2] = r.z; x[4 * v + 3] = r.w;
        }
        inv16_tw(x, w3, lc.q, lc.q2);
#pragma unroll
        for (int v = 0; v < 4; ++v)
            *reinterpret_cast<uint4*>(base + ((v ^ sw) << 2)) = make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
    }
    __syncwarp();
    {   // stage 2': thread (a, c), elements b
        const int aa = hi4, c = lo4;
#pragma unroll
        for (int k = 0; k < 16; ++k) x[k] = S[v8_phys(aa, k, c)];
        const uint2* W = TW + 32 * w + (aa & 1);
        inv16_sp<false>(x, W, W + 2 + (aa & 1), W + 6 + 3 * (aa & 1), W + 14 + 7 * (aa & 1), lc);
#pragma unroll
        for (int k = 0; k < 16; ++k) S[v8_phys(aa, k, c)] = x[k];
    }
}
// Inverse stage 1' (twiddles TW + 256): x <- thread (b, c)'s 16 elements a, lazy in [0, 2q)
__device__ __forceinline__ void inv_stage1(const uint32_t* S, uint32_t* x, const uint2* TW, const LimbConst& lc, int t) {
#pragma unroll
    for (int k = 0; k < 16; ++k) x[k] = S[v8_phys(k, t >> 4, t & 15)];
    const uint2* T1 = TW + 256;
    inv16_sp<false>(x, T1, T1 + 2, T1 + 4, T1 + 8, lc);
}

// H17 (forward only): N = 2^17 as two independent 2^16 halves.  After the first merged-psi layer (pairs j,
// j + 2^16, twiddle Psi17[1]) the halves never interact again, and half h is the 2^16 network whose layer-l
// group-g twiddle is Psi17[2^(l+1) + h 2^l + g].  The host passes a virtual plan: 2 L limbs (limb' = 2 l + h,
// re-indexed twiddle tables, LimbConst with (Psi17[1], Shoup) in pad_[0..1]) and 2 rows per 2^17 row, so
// one CTA holds one half in TMEM.  Only the column pass differs: it loads both halves' lines of its columns
// (two TMA boxes, 32 KB, single-buffered, issued one pass ahead) and applies layer 0 before layers 1..4.
template <bool FWD, bool H17 = false>
__global__ void __launch_bounds__(NT, 1) ntt_tmr16(NttArgs a, uint32_t rows, const __grid_constant__ CUtensorMap tm_in) {
    static_assert(FWD || !H17, "H17: forward only");
    constexpr int LOGN = 16, A = 4;
    extern __shared__ __align__(1024) uint32_t smem[];
    const int team = (int)(threadIdx.x >> 8), t = (int)(threadIdx.x & (TT - 1));
    const int w = t >> 5, h = w >> 2, hi4 = t >> 4, lo4 = t & 15, lane = t & 31;
    uint32_t* TS = smem + team * TEAM_W;
    uint32_t* const B0 = TS;                     // forward: sub-row exchange; inverse: input buffer 0
    uint32_t* const B1 = TS + SUBW;              // forward: TMA column staging 0; inverse: input buffer 1
    uint32_t* const B2 = TS + 2 * SUBW;          // forward: TMA column staging 1
    auto TWB = [&](int b) { return reinterpret_cast<uint2*>(TS + 3 * SUBW + b * TWW); };
    // per team: tbar[0..1] the forward TMA stagings, tbar[2] "B0 free" (the team's 8 warps are done with
    // the previous sub-row's exchange buffer); rowbar (CTA): every warp's TMEM writes of a row are done
    uint64_t* tbar = reinterpret_cast<uint64_t*>(smem + TEAMS * TEAM_W) + 3 * team;
    uint64_t* rowbar = reinterpret_cast<uint64_t*>(smem + TEAMS * TEAM_W) + 3 * TEAMS;
    uint32_t* tslot = reinterpret_cast<uint32_t*>(rowbar + 1);

    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(smem_u32(tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (t == 0) { mb_init(tbar, 1); mb_init(tbar + 1, 1); mb_init(tbar + 2, TT / 32); }
    if (threadIdx.x == 0) mb_init(rowbar, NT / 32);
    if (t == 0) mb_init_fence();
    tfence_before();
    __syncthreads();
    tfence_after();
    // this thread's TMEM lane (its warp's quadrant) and column half
    const uint32_t tl = *tslot + ((uint32_t)(32 * (w & 3)) << 16) + 16u * h;
    // the warp's TMEM writes of a row are complete and ordered before the row barrier's arrival
    auto row_arrive = [&]() {
        tm_wait_st();
        tfence_before();
        __syncwarp();
        if (lane == 0) mb_arrive(rowbar);
    };
    // every warp's TMEM writes of row r are visible to this thread's later TMEM reads
    auto row_wait = [&](uint32_t r) {
        mb_wait(rowbar, r & 1);
        tfence_after();
    };

    const uint32_t G = gridDim.x;
    const uint32_t nrow = rows > blockIdx.x ? (rows - blockIdx.x + G - 1) / G : 0;
    const uint32_t nb = a.nb_total ? a.nb_total : rows / a.L;   // polynomials of the schedule
    // limb-major schedule as in v8: the CTA's j-th row is schedule slot blockIdx.x + j G
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
        // (limb, physical row) of the CTA's rows j (lbc, rwc) and j + 1 (lbn, rwn): one division per row
        uint32_t lbc = limb_of(0), rwc = row_of(0);
        uint32_t lbn = nrow > 1 ? limb_of(1) : 0, rwn = nrow > 1 ? row_of(1) : 0;
        uint32_t u = 0;                              // the team's sub-row counter (twiddle / buffer parity)
        if constexpr (FWD) {
            // Schedule per team and row j: for its four s,
            //   R1(j, s)  [TMEM -> stage 1 -> B0]   C(j+1, s) [TMA staging -> layers 0..3 -> TMEM]
            //   team barrier   R23(j, s) [stage 2, stage 3 -> out]
            // The column pass sits between stage 1 and the barrier that stage 2 needs, so the barrier wait
            // is covered by a whole pass of work; it overwrites exactly the TMEM cells R1 just read.
            // Column pass m (= 4 j + i: row j, s = team + 4 i) lands in staging buffer m & 1 (B1 / B2) and
            // completes on mbarrier m & 1; its TMA is issued right after the team barrier that follows
            // column pass m - 2, the previous reader of that buffer (two passes ahead).
            uint32_t tph = 0;                        // bit b: parity of mbarrier b's next completion
            const uint32_t mtot = 4 * nrow;          // column passes of the CTA
            auto issue_col = [&](uint32_t m, uint32_t prow) {   // team thread 0
                fence_proxy_async();
                if constexpr (H17) {                 // both halves' lines of the 2^17 row prow / 2 -> B1, B2
                    mb_expect(tbar, 32 * TT * 4);
                    const int line = (int)((prow >> 1) * 32), c0 = (team + 4 * (int)(m & 3)) * TT;
                    tma2_load_hint(B1, &tm_in, c0, line, tbar, l2_evict_first_policy());
                    tma2_load_hint(B2, &tm_in, c0, line + 16, tbar, l2_evict_first_policy());
                } else {
                    mb_expect(tbar + (m & 1), 16 * TT * 4);
                    tma2_load_hint((m & 1) ? B2 : B1, &tm_in, (team + 4 * (int)(m & 3)) * TT, (int)(prow * 16),
                                   tbar + (m & 1), l2_evict_first_policy());
                }
            };
            // column pass m (row m / 4): layers 0..3, into TMEM (layout (m / 4) & 1)
            // qv = (q, 2q) of the limb, loaded once per row by the caller: a LimbConst load per pass
            // (re-issued after every asm volatile TMEM access) stalls the first butterfly on its latency
            auto colpass = [&](uint32_t m, uint32_t limb, uint2 qv) {
                const int s = team + 4 * (int)(m & 3);
                LimbConst lc;
                if constexpr (H17) lc = a.lc[limb];  // + (Psi17[1], Shoup) in pad_
                else { lc.q = qv.x; lc.q2 = qv.y; }
                const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
                uint32_t x[16];
                if constexpr (H17) {
                    mb_wait(tbar, m & 1);            // one staging buffer, one completion per pass
                    const uint2 w0 = make_uint2(lc.pad_[0], lc.pad_[1]);
                    const bool upper = limb & 1;     // half h = limb' & 1
#pragma unroll
                    for (int k = 0; k < 16; ++k) {   // layer 0 of 2^17: (x_j, x_j+2^16) -> this half's value
                        const uint32_t lo = umin32(B1[k * TT + t], B1[k * TT + t] - lc.q2);
                        const uint32_t tt = shoup_mul(B2[k * TT + t], w0.x, w0.y, lc.q);
                        x[k] = upper ? lo - tt + lc.q2 : lo + tt;
                    }
                } else {
                    const uint32_t b = m & 1;
                    mb_wait(tbar + b, (tph >> b) & 1);
                    tph ^= 1u << b;
                    const uint32_t* SB = b ? B2 : B1;
#pragma unroll
                    for (int k = 0; k < 16; ++k) x[k] = SB[k * TT + t];
                }
                fwd_radix<A>(x, tw, 0, 0, lc.q, lc.q2);
                if ((m >> 2) & 1) tm_st16(tl + 32 * s, x);   // B: 32 s + 16 h + k
                else tm_st16s(tl + s, x);                    // A: 32 k + 16 h + s
            };

            // prologue: the column passes of row 0 (TMA 0, 1 up front, m + 2 after pass m's team barrier)
            constexpr uint32_t AHEAD = H17 ? 1 : 2;  // passes a TMA runs ahead (staging buffers)
            if (t == 0) {
                issue_col(0, rwc);
                if (!H17 && 1 < mtot) issue_col(1, rwc);
            }
            tw_fwd<A>(TWB(0), a.tw + ((size_t)lbc << LOGN), team, t);
            cp_async_commit();
#pragma unroll 1
            for (uint32_t m = 0; m < 4; ++m) {
                colpass(m, lbc, __ldg(reinterpret_cast<const uint2*>(a.lc + lbc)));
                team_bar(team);
                if (t == 0 && m + AHEAD < mtot) issue_col(m + AHEAD, m + AHEAD < 4 ? rwc : rwn);
            }
            row_arrive();
#pragma unroll 1
            for (uint32_t j = 0; j < nrow; ++j) {
                const bool more = j + 1 < nrow;
                const uint32_t r2 = j + 2 < nrow ? row_of(j + 2) : 0;
                const uint2 qc = __ldg(reinterpret_cast<const uint2*>(a.lc + lbc));   // (q, 2q) of rows j, j + 1
                const uint2 qn = __ldg(reinterpret_cast<const uint2*>(a.lc + lbn));
#pragma unroll 1
                for (int i = 0; i < 4; ++i, ++u) {
                    const int s = team + 4 * i;
                    LimbConst lc;                        // the row stages use q, 2q only
                    lc.q = qc.x; lc.q2 = qc.y;
                    const uint2* __restrict__ tw = a.tw + ((size_t)lbc << LOGN);
                    uint32_t* S = B0;
                    // ---- R1(j, s): stage 1 (layers 4..7, thread (b, c), elements a) from TMEM
                    if (i == 0) row_wait(j);             // every column pass of row j is in TMEM
                    cp_async_wait<0>();
                    __syncwarp();                        // this warp's stage-1 twiddles landed
                    uint32_t x[16];
                    if (j & 1) tm_ld16s(tl + s, x);      // B: element 256 a + t at 32 a + 16 h + s
                    else tm_ld16(tl + 32 * s, x);        // A: 32 s + 16 h + a
                    {
                        const uint2* W = TWB(u & 1) + 16 * w;
                        fwd16_sp(x, W, W + 2, W + 4, W + 8, lc.q, lc.q2);
                        if (u > 0) mb_wait(tbar + 2, (u - 1) & 1);   // every warp done with sub-row u - 1
#pragma unroll
                        for (int k = 0; k < 16; ++k) S[v8_phys(k, hi4, lo4)] = x[k];
                    }
                    // ---- C(j+1, s): overwrites exactly the TMEM cells R1 read
                    const uint32_t m = 4 * (j + 1) + i;
                    if (more) {
                        colpass(m, lbn, qn);
                        if (i == 3) row_arrive();        // this warp's part of row j + 1 is in TMEM
                    }
                    team_bar(team);                      // stage 1 (and column pass m) done team-wide
                    if (t == 0 && more && m + AHEAD < mtot)
                        issue_col(m + AHEAD, ((m + AHEAD) >> 2) == j + 1 ? rwn : r2);
                    {   // the team's next sub-row's twiddles
                        uint32_t nj = j, ns = (uint32_t)s + TEAMS;
                        if (ns >= 16) { nj = j + 1; ns = team; }
                        if (nj < nrow) tw_fwd<A>(TWB((u + 1) & 1), a.tw + ((size_t)(nj == j ? lbc : lbn) << LOGN), ns, t);
                        cp_async_commit();
                    }
                    // ---- R23(j, s)
                    const uint32_t qq = lc.q, q2 = lc.q2;
                    uint32_t* out = a.out + ((size_t)rwc << LOGN) + s * SUBW;
                    uint2 w3[15];
                    load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                    fwd_stages23(S, x, TWB(u & 1) + 128, w3, qq, q2, out, t, tbar + 2);
                }
                lbc = lbn; rwc = rwn;
                if (j + 2 < nrow) { lbn = limb_of(j + 2); rwn = r2; }
            }
        } else {
            // sub-row s of row j: layers 15..4 (input bit-reversed), stage 1' into TMEM (layout j & 1)
            auto rowpass = [&](uint32_t j, int s, uint32_t u, uint32_t limb, uint32_t row_self, uint32_t limb_next,
                               uint32_t row_next) {
                const LimbConst lc = a.lc[limb];
                const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
                uint32_t* S = (u & 1) ? B1 : B0;
                uint2 w3[15];
                load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                cp_async_wait<0>();
                __syncwarp();                            // this warp's slice of sub-row s landed
                uint32_t x[16];
                inv_stages32(S, x, w3, TWB(u & 1), lc, t);
                team_bar(team);                          // stage 2' done team-wide; the other buffer is free
                {   // the team's next sub-row: data and twiddles into the other buffer
                    uint32_t nj = j, ns = (uint32_t)s + TEAMS, nl = limb, nr = row_self;
                    if (ns >= 16) { nj = j + 1; ns = team; nl = limb_next; nr = row_next; }
                    if (nj < nrow) {
                        tw_inv<A>(TWB((u + 1) & 1), a.tw + ((size_t)nl << LOGN), ns, t);
                        load_inv_slice((u & 1) ? B0 : B1, a.in + ((size_t)nr << LOGN) + ns * SUBW, t);
                    }
                    cp_async_commit();
                }
                {   // stage 1': layers A+3..A, thread (b, c), elements a -> TMEM (lazy, in [0, 2q))
                    inv_stage1(S, x, TWB(u & 1), lc, t);
                    if (j & 1) tm_st16s(tl + s, x);      // B: element 256 a + t at 32 a + 16 h + s
                    else tm_st16(tl + 32 * s, x);        // A: 32 s + 16 h + a
                }
            };
            // column pass s of row j: layers 3..0 with N^-1, canonical output
            auto colpass = [&](int s, uint32_t limb, uint32_t row, bool jpar) {
                const LimbConst lc = a.lc[limb];
                const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
                uint32_t x[16];
                if (jpar) tm_ld16(tl + 32 * s, x);       // B: 32 s + 16 h + k
                else tm_ld16s(tl + s, x);                // A: 32 k + 16 h + s
                inv_radix<A, true>(x, tw, 0, 0, lc);
                uint32_t* o = a.out + ((size_t)row << LOGN) + s * TT + t;
#pragma unroll
                for (int k = 0; k < 16; ++k) __stcs(o + k * SUBW, canon2(x[k], lc.q));
            };

            tw_inv<A>(TWB(0), a.tw + ((size_t)lbc << LOGN), team, t);
            load_inv_slice(B0, a.in + ((size_t)rwc << LOGN) + team * SUBW, t);
            cp_async_commit();
            bool jpar = false;                           // layout of row j (j & 1)
#pragma unroll 1
            for (int s = team; s < 16; s += TEAMS, ++u) rowpass(0, s, u, lbc, rwc, lbn, rwn);
            cta_sync_tmem();
#pragma unroll 1
            for (uint32_t j = 0; j < nrow; ++j) {
                const bool more = j + 1 < nrow;
                const uint32_t lb2 = j + 2 < nrow ? limb_of(j + 2) : 0, rw2 = j + 2 < nrow ? row_of(j + 2) : 0;
#pragma unroll 1
                for (int s = team; s < 16; s += TEAMS) {
                    colpass(s, lbc, rwc, jpar);
                    if (more) { rowpass(j + 1, s, u, lbn, rwn, lb2, rw2); ++u; }   // refills the cells colpass read
                }
                lbc = lbn; rwc = rwn; lbn = lb2; rwn = rw2;
                jpar = !jpar;
                cta_sync_tmem();
            }
        }
    }
    cp_async_wait<0>();
    tfence_before();
    __syncthreads();
    if (threadIdx.x < 32) {
        tfence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(*tslot));
    }
}

}  // namespace tmr
}  // namespace wd
