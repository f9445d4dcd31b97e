// ntt_tc4.cuh -- warp-specialised 4-step tcgen05 NTT for N = 2^16.
//
// The paper's WD-FUSE idea (Fig. 3: tensor-core and CUDA-core work of different
// tiles at the same time on one SM; Alg. 2: inner DFTs as u8 GEMMs with the
// twiddles in the matrices) re-derived for sm_100a.  One persistent CTA per SM, 20 warps (<= 96
// registers each):
//   warp 0  producers: lane 0 streams the input / intermediate tiles HBM/L2 -> shared memory
//           (cp.async.bulk.tensor, mbarrier complete_tx), lane 1 the per-group stage matrices
//           (cp.async.bulk) one tile ahead of their MMA
//   warps 1, 3  MMA issuers (one thread each, even / odd tiles): tcgen05.mma.cta_group::1.kind::i8,
//           accumulators in TMEM, completion by tcgen05.commit -> mbarrier; warp 1 owns the TMEM
//           allocation (512 columns)
//   warp 2  TMA store issuer: shared-memory staging tiles -> global (cp.async.bulk.tensor store)
//   warps 4..19  CUDA-core workers, two groups of 8 (in a group, two warps per TMEM lane quarter,
//           one per output half): operand transposition, the accumulator epilogues (byte-plane
//           recombination, Shoup fold), the 4-step twist
// The units overlap through rings (8 input slots, 4 A-operand slots, 4 TMEM accumulators, 6 staging
// slots, 8 matrix slots): the tensor pipe runs the next tiles while the workers finish tile t.
//
// Decomposition (reading C-1 negacyclic, C-3 bit-reversed output).  Row x[j],
// j = 256 j1 + j2.  With psi of order 2N, zeta = psi^256, omega = psi^512:
//   X[k1 + 256 k2] = sum_j2 omega^(k2 j2) psi^((2k1+1) j2) sum_j1 zeta^((2k1+1) j1) x[256 j1 + j2]
// column phase (per column j2; j1 = 16a + b, k1 = c + 16d):
//   stage A  U[c][b]    = sum_a MA[c][a] x[16a+b],        MA[c][a]   = psi^(4096 a (2c+1))   (shared)
//   stage B  Y[c+16d]   = sum_b MB_c[d][b] U[c][b],       MB_c[d][b] = psi^(256 b (2c+1+32d)) (group c)
//   twist    Z[k1][j2]  = Y[k1] psi^((2k1+1) j2)                                      (per element)
// row phase (per k1; j2 = 16f + e, k2 = g + 16h):
//   stage C  V[g][e]    = sum_f MC[g][f] Z[16f+e],        MC[g][f]   = psi^(8192 g f)          (shared)
//   stage D  X[k1+256(g+16h)] = sum_e MD_g[h][e] V[g][e], MD_g[h][e] = psi^(512 e (g + 16 h)) (group g)
// Output index brv16(k1 + 256 g + 4096 h) = 256 brv8(k1) + 16 brv4(g) + brv4(h): every stage-D
// instance writes 16 contiguous words (MD_g's rows are taken in brv4 order).
// Every stage is a radix-16 u8 x u8 -> s32 GEMM over the byte view of the u32 data (the byte-plane
// identity of tensor_tables.h: K = 16 coefficients x 4 bytes, N = 16 outputs x 4 planes): 4 MMA
// stages + ONE per-element twist, against 8 Shoup butterflies per element on the CUDA-core path.
//
// A CTA takes a contiguous range of limb-major rows.  Each row is 4 passes of 32 tiles (16 stage-1
// + 16 stage-2, M = 128 instances each): column passes h = 0,1 (columns [128h, 128h+128)) and row
// passes hh = 0,1 (rows r in [128hh, 128hh+128), r = brv8(k1)).  Passes of consecutive rows are
// interleaved (C(i+1,0) R(i,0) C(i+1,1) R(i,1)) so a row's intermediate is in L2 before its row
// passes load it.  The intermediate lives in the row's own output slot; every pass writes only
// the region it has already read, so in == out is safe.
#pragma once
#include <cuda.h>
#include <cstdint>
#include "modarith.cuh"

namespace wd {
namespace tc4 {

constexpr int NT = 640;                          // 20 warps (5 per SM sub-partition at <= 96 registers)
constexpr int W_LOAD = 0, W_MMA = 1, W_STORE = 2, W_MMA2 = 3, W_WORK0 = 4, NWW = 16;
constexpr int NIN = 8, NOPA = 4, NACC = 4, NSTG = 6, NB = 8;
constexpr uint32_t TILE = 8192;                  // one operand / staging tile: 128 x 64 bytes
constexpr uint32_t MAT = 4096;                   // one 16x16 stage matrix as 64 x 64 byte planes
constexpr uint32_t MATSET = 17 * MAT;            // MA + MB[16]  (or MC + MD[16]) in global memory
// shared memory: the two shared-matrix stages (MA, MC) resident; the 16 per-group matrices of a
// pass (MB_c / MD_g) stream through a ring of NB slots one tile ahead of their MMA
constexpr uint32_t SM_MATC = 0, SM_MATR = MAT, SM_BR = 2 * MAT, SM_IN = SM_BR + NB * MAT,
                   SM_OPA = SM_IN + NIN * TILE, SM_STG = SM_OPA + NOPA * TILE, SM_BAR = SM_STG + NSTG * TILE;
constexpr uint32_t SMEM = SM_BAR + 1024;
constexpr uint32_t TM_OP2 = 0, TM_ACC = 256;     // TMEM columns: stage-2 operands, 4 accumulators
static_assert(SMEM <= 232448, "shared memory");

struct Args {
    const uint8_t* mat;      // [L][2 sets][17][MAT] byte planes of this direction (set 0: MA, MB_c; set 1: MC, MD_g)
    const uint2* tw;         // [L][2 h][16 c][16 d][128 lane] twist (w, w') in worker-lane order
    const uint4* lq;         // [L] {q, Shoup(2^16), Shoup(1), 0}
    uint32_t rows, L, nb;
    unsigned long long* trace;   // diagnostics: CTA 0 event timestamps (clock64), or nullptr
};
// trace slots: [0, 4096) loads issued, [4096, 8192) MMAs issued, [8192, 12288) worker 0 accumulator
// ready, [12288, 16384) worker 0 staging handed over, [16384, 20480) stores issued
constexpr int TR_LOAD = 0, TR_MMA = 4096, TR_ACC = 8192, TR_STG = 12288, TR_STORE = 16384, TR_DET = 20480, TR_N = 53248;
#define TC4_TRACE(slot) do { if (a.trace && blockIdx.x == 0 && (slot) < TR_N) a.trace[(slot)] = clock64(); } while (0)

// ------------------------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void bar_init(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(sa(b)), "r"(n));
}
__device__ __forceinline__ void bar_wait(uint64_t* b, uint32_t parity) {
    asm volatile("{\n\t.reg .pred P1;\n\tTC4W_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
                 "@!P1 bra TC4W_%=;\n\t}\n" :: "r"(sa(b)), "r"(parity) : "memory");
}
// with a suspend-time hint the waiting thread sleeps in hardware until the phase completes: for the
// producer / store / matrix threads, whose waits are long and whose schedulers host epilogue warps
__device__ __forceinline__ void bar_wait_sleep(uint64_t* b, uint32_t parity) {
    asm volatile("{\n\t.reg .pred P1;\n\tTC4S_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n\t"
                 "@!P1 bra TC4S_%=;\n\t}\n" :: "r"(sa(b)), "r"(parity), "r"(1000000) : "memory");
}
__device__ __forceinline__ void bar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(sa(b)) : "memory");
}
__device__ __forceinline__ void bar_expect(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(sa(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_load4(void* dst, const CUtensorMap* m, int c0, int c1, int c2, int c3, uint64_t* b) {
    asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
                 " [%0], [%1, {%2, %3, %4, %5}], [%6];"
                 :: "r"(sa(dst)), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(sa(b)) : "memory");
}
__device__ __forceinline__ void tma_load5(void* dst, const CUtensorMap* m, int c0, int c1, int c2, int c3, int c4,
                                          uint64_t* b) {
    asm volatile("cp.async.bulk.tensor.5d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
                 " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 :: "r"(sa(dst)), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "r"(sa(b)) : "memory");
}
__device__ __forceinline__ void tma_store2(const CUtensorMap* m, int c0, int c1, const void* src) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.tile.bulk_group [%0, {%1, %2}], [%3];"
                 :: "l"(m), "r"(c0), "r"(c1), "r"(sa(src)) : "memory");
}
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(sa(dst)), "l"(src), "r"(bytes), "r"(sa(b)) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read1() { asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tfence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tfence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void prefetch_map(const CUtensorMap* m) {
    asm volatile("prefetch.tensormap [%0];" :: "l"(m) : "memory");
}

// K-major SWIZZLE_NONE smem descriptor: 8-row x 16-byte core matrices, LBO 128 B (K), SBO 512 B (M)
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)(128 >> 4) << 16) | ((uint64_t)(512 >> 4) << 32) |
           ((uint64_t)1 << 46);
}
// kind::i8: D s32 (bits 4-5 = 2), A/B u8, both K-major, N = 64 (bits 17-22 = N/8), M = 128 (bits 24-28 = M/16)
constexpr uint32_t IDESC = (2u << 4) | ((uint32_t)(64 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);

__device__ __forceinline__ void mma_ss(uint32_t d, uint64_t a, uint64_t b, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
                 :: "r"(d), "l"(a), "l"(b), "r"(IDESC), "r"(acc));
}
__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t}\n"
                 :: "r"(d), "r"(a_tmem), "l"(b), "r"(IDESC), "r"(acc));
}
__device__ __forceinline__ void mma_commit(uint64_t* b) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(sa(b)) : "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t* r) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 "
                 "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                 "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
                   "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
                   "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                 : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld64(uint32_t taddr, uint32_t* r) {   // 64 columns: two x32 loads
    tmem_ld32(taddr, r);
    tmem_ld32(taddr + 32, r + 32);
}
__device__ __forceinline__ void tmem_st2(uint32_t taddr, uint32_t a, uint32_t b) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1, %2};" :: "r"(taddr), "r"(a), "r"(b) : "memory");
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_st4(uint32_t taddr, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};"
                 :: "r"(taddr), "r"(a), "r"(b), "r"(c), "r"(d) : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ uint32_t brv4(uint32_t x) { return __brev(x) >> 28; }

// ---------------------------------------------------------------------------- epilogue arithmetic
// Byte shifts as PRMT (ALU pipe): ptxas turns every plain shift-add of this kernel into an IMAD on
// the fma pipe, which the Shoup products already load.  shl8(a) = a << 8 for a < 2^24, shl16(a) =
// a << 16 mod 2^32 (byte permutes with a zero source).
__device__ __forceinline__ uint32_t shl8(uint32_t a) {
    uint32_t r;
    asm("prmt.b32 %0, %1, 0, 0x2104;" : "=r"(r) : "r"(a));
    return r;
}
__device__ __forceinline__ uint32_t shl16(uint32_t a) {
    uint32_t r;
    asm("prmt.b32 %0, %1, 0, 0x1044;" : "=r"(r) : "r"(a));
    return r;
}
// Sum_b 2^(8b) D_b mod q, lazily: lo = D0 + 2^8 D1 < 2^30, hi = D2 + 2^8 D3; hi * 2^16 by Shoup in
// [0, 2q); the sum < 2^30 + 2^31 < 2^32 is a valid input of the next byte-plane GEMM (any u32 is).
// D_b < 2^22, so the byte shifts of D1, D3 lose nothing.  nq = -q mod 2^32.
__device__ __forceinline__ uint32_t fold(const uint32_t* d, uint32_t nq, uint32_t c16s) {
    const uint32_t lo = d[0] + shl8(d[1]);
    const uint32_t hi = d[2] + shl8(d[3]);
    const uint32_t t = __umulhi(hi, c16s);
    return t * nq + (lo + shl16(hi));
}
// the same value, fully reduced to [0, q) (last stage): lo by Shoup with w = 1, both parts < 2q
__device__ __forceinline__ uint32_t fold_canon(const uint32_t* d, uint32_t q, uint32_t nq, uint32_t c16s, uint32_t ones) {
    const uint32_t lo = d[0] + shl8(d[1]);
    const uint32_t hi = d[2] + shl8(d[3]);
    const uint32_t a = __umulhi(lo, ones) * nq + lo;                    // [0, 2q)
    uint32_t v = __umulhi(hi, c16s) * nq + (a + shl16(hi));             // [0, 4q)
    v = umin32(v, v - 2 * q);
    return umin32(v, v - q);
}

// worker lane m (0..127) of a column pass -> column offset pi(m) in [0, 128) of the pass's half.
// pi(m) = 16 f + e with (l = m & 31, w = m >> 5):  e = 4 l[3:5) + l[0:2),  f = 4 f2 + 2 f1 + l[2],
// (f2 f1) = l[3:5) ^ w.  Both shared-memory patterns of the column pass are then conflict-free:
// the input gather [a][pi(m)] (banks 16 l[2] + e) and the intermediate staging [row][8e + f]
// (banks 8 l[0:2) + f).
__host__ __device__ __forceinline__ uint32_t col_pi(uint32_t m) {
    const uint32_t l = m & 31, w = m >> 5;
    const uint32_t e = 4 * ((l >> 3) & 3) + (l & 3);
    const uint32_t f = 4 * ((((l >> 3) & 3) ^ w) >> 1) + 2 * ((((l >> 3) & 3) ^ w) & 1) + ((l >> 2) & 1);
    return 16 * f + e;
}

// pass p of a CTA with n rows: row index i, column (true) or row pass, half h
__device__ __forceinline__ void pass_info(uint32_t p, uint32_t n, uint32_t& i, bool& col, uint32_t& h) {
    if (p < 2) { i = 0; col = true; h = p; return; }
    if (p >= 4 * n - 2) { i = n - 1; col = false; h = p - (4 * n - 2); return; }
    const uint32_t q = p - 2, k = q & 3;
    i = q / 4 + 1;
    col = (k & 1) == 0;
    h = k >> 1;
    if (!col) i -= 1;
}

struct Bars {
    uint64_t in_full[NIN], in_empty[NIN], opa_full[NOPA], opa_empty[NOPA], acc_full[NACC], acc_empty[NACC];
    uint64_t stg_full[NSTG], stg_empty[NSTG];
    uint64_t br_full[NB], br_empty[NB];
    uint64_t op2_full, op2_empty, inter_done, matc_full, matr_full, colset_free, rowset_free;
    uint32_t tmem;
};

// --------------------------------------------------------------------------------- forward kernel
__global__ void __launch_bounds__(NT, 1) ntt_tc4_fwd(const __grid_constant__ CUtensorMap tm_x,
                                                     const __grid_constant__ CUtensorMap tm_c,
                                                     const __grid_constant__ CUtensorMap tm_i,
                                                     const __grid_constant__ CUtensorMap tm_o, Args a) {
    extern __shared__ __align__(1024) uint8_t sm[];
    Bars& B = *reinterpret_cast<Bars*>(sm + SM_BAR);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t r0 = (uint32_t)((uint64_t)blockIdx.x * a.rows / gridDim.x);
    const uint32_t r1 = (uint32_t)((uint64_t)(blockIdx.x + 1) * a.rows / gridDim.x);
    if (r0 >= r1) return;
    const uint32_t n = r1 - r0;
    const uint32_t npass = 4 * n;

    if (threadIdx.x == 0) {
        for (int i = 0; i < NIN; ++i) { bar_init(&B.in_full[i], 1); bar_init(&B.in_empty[i], 1); }
        for (int i = 0; i < NOPA; ++i) { bar_init(&B.opa_full[i], NWW / 2); bar_init(&B.opa_empty[i], 1); }
        for (int i = 0; i < NACC; ++i) { bar_init(&B.acc_full[i], 1); bar_init(&B.acc_empty[i], NWW / 2); }
        for (int i = 0; i < NSTG; ++i) { bar_init(&B.stg_full[i], NWW / 2); bar_init(&B.stg_empty[i], 1); }
        for (int i = 0; i < NB; ++i) { bar_init(&B.br_full[i], 1); bar_init(&B.br_empty[i], 1); }
        bar_init(&B.op2_full, NWW); bar_init(&B.op2_empty, 2); bar_init(&B.inter_done, 1);
        bar_init(&B.matc_full, 1); bar_init(&B.matr_full, 1); bar_init(&B.colset_free, 2); bar_init(&B.rowset_free, 2);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        prefetch_map(&tm_x); prefetch_map(&tm_c); prefetch_map(&tm_i); prefetch_map(&tm_o);
    }
    if (warp == W_MMA) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(sa(&B.tmem)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tfence_before();
    __syncthreads();
    tfence_after();
    const uint32_t tmem = B.tmem;

    auto limb_of = [&](uint32_t i) { return (r0 + i) / a.nb; };
    auto row_of = [&](uint32_t i) { const uint32_t s = r0 + i, l = s / a.nb; return (s - l * a.nb) * a.L + l; };

    if (warp == W_LOAD && lane == 0) {
        // ===================================================================== TMA producer (inputs)
        {
            uint32_t nin = 0;
            for (uint32_t p = 0; p < npass; ++p) {
                uint32_t i, h; bool col;
                pass_info(p, n, i, col, h);
                const uint32_t row = row_of(i);
                if (!col && h == 0) bar_wait_sleep(&B.inter_done, i & 1);     // row i's intermediate is in global memory
                for (uint32_t k = 0; k < 16; ++k, ++nin) {
                    const uint32_t s = nin % NIN;
                    bar_wait_sleep(&B.in_empty[s], ((nin / NIN) & 1) ^ 1);
                    bar_expect(&B.in_full[s], TILE);
                    uint8_t* dst = sm + SM_IN + s * TILE;
                    TC4_TRACE(TR_LOAD + nin);
                    if (col) tma_load4(dst, &tm_x, (int)(128 * h), (int)k, 0, (int)row, &B.in_full[s]);   // x piece b = k
                    else tma_load5(dst, &tm_c, (int)(8 * k), 0, 0, 0, (int)(row * 32 + 16 * h), &B.in_full[s]);  // C tile e = k
                }
            }
        }
    } else if (warp == W_LOAD && lane == 1) {
        // ===================================================================== matrix producer
        {
            uint32_t nb = 0;
            uint32_t lc = 0xffffffffu, lr = 0xffffffffu;
            for (uint32_t p = 0; p < npass; ++p) {
                uint32_t i, h; bool col;
                pass_info(p, n, i, col, h);
                const uint32_t limb = limb_of(i);
                const uint8_t* set = a.mat + ((size_t)limb * 2 + (col ? 0 : 1)) * MATSET;
                if (h == 0 && limb != (col ? lc : lr)) {            // this limb's shared stage matrix
                    if (i > 0) bar_wait_sleep(col ? &B.colset_free : &B.rowset_free, (i - 1) & 1);
                    uint64_t* fb = col ? &B.matc_full : &B.matr_full;
                    bar_expect(fb, MAT);
                    bulk_load(sm + (col ? SM_MATC : SM_MATR), set, MAT, fb);
                    if (col) lc = limb; else lr = limb;
                }
                for (uint32_t k = 0; k < 16; ++k, ++nb) {           // the pass's per-group matrices
                    const uint32_t s = nb % NB;
                    bar_wait_sleep(&B.br_empty[s], ((nb / NB) & 1) ^ 1);
                    bar_expect(&B.br_full[s], MAT);
                    bulk_load(sm + SM_BR + s * MAT, set + (1 + k) * MAT, MAT, &B.br_full[s]);
                }
            }
        }
    } else if (warp == W_LOAD) {
        // lanes 2..31 of the producer warp: idle
    } else if (warp == W_MMA || warp == W_MMA2) {
        // ===================================================================== MMA issuers
        // two threads in two warps, even and odd tiles: the per-tile chain of mbarrier waits, MMA
        // dispatch and commits (~0.4 us) is the serial limit of a single issuer at these tile sizes
        if (lane == 0) {
            const uint32_t par = warp == W_MMA ? 0 : 1;
            uint32_t nin = 0, nopa = 0, t = 0, nmc = 0, nmr = 0, nb = 0;
            uint32_t lc = 0xffffffffu, lr = 0xffffffffu;
            const uint32_t matc = sa(sm + SM_MATC), matr = sa(sm + SM_MATR);
            for (uint32_t p = 0; p < npass; ++p) {
                uint32_t i, h; bool col;
                pass_info(p, n, i, col, h);
                const uint32_t limb = limb_of(i);
                if (col && h == 0 && limb != lc) { bar_wait(&B.matc_full, nmc & 1); lc = limb; ++nmc; }
                if (!col && h == 0 && limb != lr) { bar_wait(&B.matr_full, nmr & 1); lr = limb; ++nmr; }
                const uint32_t mbase = col ? matc : matr;
                // ---- stage 1 (A or C): operand in shared memory
                for (uint32_t k = 0; k < 16; ++k, ++nin, ++t) {
                    if (col) ++nopa;
                    if ((k & 1) != par) continue;
                    const uint32_t s = nin % NIN, as = t % NACC;
                    uint32_t abase;
                    if (col) {
                        const uint32_t o = (nopa - 1) % NOPA;
                        bar_wait(&B.opa_full[o], ((nopa - 1) / NOPA) & 1);
                        bar_arrive(&B.in_empty[s]);              // the workers have consumed the x piece
                        abase = sa(sm + SM_OPA + o * TILE);
                    } else {
                        bar_wait(&B.in_full[s], (nin / NIN) & 1);
                        abase = sa(sm + SM_IN + s * TILE);
                    }
                    TC4_TRACE(TR_DET + 8 * t + 6);
                    bar_wait(&B.acc_empty[as], ((t / NACC) & 1) ^ 1);
                    tfence_after();
                    const uint32_t d = tmem + TM_ACC + 64 * as;
                    mma_ss(d, sdesc(abase), sdesc(mbase), 0);
                    mma_ss(d, sdesc(abase + 256), sdesc(mbase + 256), 1);
                    TC4_TRACE(TR_MMA + t);
                    mma_commit(&B.acc_full[as]);
                    if (col) mma_commit(&B.opa_empty[(nopa - 1) % NOPA]);
                    else mma_commit(&B.in_empty[s]);
                }
                // ---- stage 2 (B or D): operand in TMEM (written by the stage-1 epilogues)
                bar_wait(&B.op2_full, p & 1);
                tfence_after();
                for (uint32_t k = 0; k < 16; ++k, ++t, ++nb) {
                    if ((k & 1) != par) continue;
                    const uint32_t as = t % NACC, bs = nb % NB;
                    bar_wait(&B.br_full[bs], (nb / NB) & 1);
                    TC4_TRACE(TR_DET + 8 * t + 6);
                    bar_wait(&B.acc_empty[as], ((t / NACC) & 1) ^ 1);
                    tfence_after();
                    const uint32_t d = tmem + TM_ACC + 64 * as;
                    const uint32_t bm = sa(sm + SM_BR + bs * MAT);
                    mma_ts(d, tmem + TM_OP2 + 16 * k, sdesc(bm), 0);
                    mma_ts(d, tmem + TM_OP2 + 16 * k + 8, sdesc(bm + 256), 1);
                    TC4_TRACE(TR_MMA + t);
                    mma_commit(&B.acc_full[as]);
                    mma_commit(&B.br_empty[bs]);
                }
                mma_commit(&B.op2_empty);
                if (h == 1) mma_commit(col ? &B.colset_free : &B.rowset_free);
            }
        }
    } else if (warp == W_STORE) {
        // ===================================================================== TMA store issuer
        if (lane == 0) {
            // staging slots are released in order, SLAG stores behind the newest (their smem reads done)
            constexpr uint32_t SLAG = 3;
            static_assert(SLAG < NSTG, "staging ring");
            uint32_t ns = 0, rel = 0;
            for (uint32_t p = 0; p < npass; ++p) {
                uint32_t i, h; bool col;
                pass_info(p, n, i, col, h);
                const uint32_t row = row_of(i);
                for (uint32_t k = 0; k < 16; ++k, ++ns) {
                    const uint32_t s = ns % NSTG;
                    bar_wait_sleep(&B.stg_full[s], (ns / NSTG) & 1);
                    const uint8_t* src = sm + SM_STG + s * TILE;
                    TC4_TRACE(TR_STORE + ns);
                    if (col) tma_store2(&tm_i, (int)(128 * h), (int)(row * 256 + 16 * brv4(k)), src);
                    else tma_store2(&tm_o, (int)(16 * brv4(k)), (int)(row * 256 + 128 * h), src);
                    bulk_commit();
                    if (ns + 1 > rel + SLAG) {
                        asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(SLAG) : "memory");
                        for (; rel + SLAG < ns + 1; ++rel) bar_arrive(&B.stg_empty[rel % NSTG]);
                    }
                }
                if (col && h == 1) {                              // row i's intermediate complete in global
                    bulk_wait0();
                    for (; rel < ns; ++rel) bar_arrive(&B.stg_empty[rel % NSTG]);
                    bar_arrive(&B.inter_done);
                }
            }
            bulk_wait0();
        }
    } else {
        // ===================================================================== CUDA-core workers
        // Two groups of eight warps take alternate tiles (stage 1: alternate tile pairs); inside a group
        // the two warps of a TMEM lane quarter split a tile's 16 outputs (8 each).  While one group
        // waits on a barrier or a TMEM load the other computes; four epilogue warps per sub-partition.
        const uint32_t wi = warp - W_WORK0;                       // 0..15
        const uint32_t quad = warp & 3, hf = (wi >> 2) & 1, grp = wi >> 3;
        const uint32_t m = 32 * quad + lane;                      // this thread's TMEM lane / instance
        const uint32_t pim = col_pi(m);
        const uint32_t lrow = 32 * quad;
        const bool w0 = (wi == 0 || wi == 8) && lane == 0;        // trace: first warp of each group
        uint32_t nin = 0, nopa = 0, t = 0, ns = 0;
        auto acc_get = [&](uint32_t tt, uint32_t* d) {            // this warp's 32 accumulator columns of tile tt
            const uint32_t as = tt % NACC;
            bar_wait(&B.acc_full[as], (tt / NACC) & 1);
            if (w0) TC4_TRACE(TR_ACC + tt);
            tfence_after();
            tmem_ld32(tmem + (lrow << 16) + TM_ACC + 64 * as + 32 * hf, d);
            tmem_wait_ld();
            tfence_before();
            __syncwarp();
            if (lane == 0) bar_arrive(&B.acc_empty[as]);
        };
        for (uint32_t p = 0; p < npass; ++p) {
            uint32_t i, h; bool col;
            pass_info(p, n, i, col, h);
            const uint32_t limb = limb_of(i);
            const uint4 lq = __ldg(a.lq + limb);
            const uint32_t q = lq.x, nq = 0u - lq.x, c16s = lq.y, ones = lq.z;
            const uint32_t nin0 = nin, nopa0 = nopa, t1 = t, t2 = t + 16, ns0 = ns;
            // stage-1 prologue of tile b (column passes): x piece [a][128 words] -> OPA row m (K-major)
            auto pro = [&](uint32_t b) {
                const uint32_t s = (nin0 + b) % NIN, o = (nopa0 + b) % NOPA;
                bar_wait(&B.in_full[s], ((nin0 + b) / NIN) & 1);
                bar_wait(&B.opa_empty[o], (((nopa0 + b) / NOPA) & 1) ^ 1);
                const uint32_t* X = reinterpret_cast<const uint32_t*>(sm + SM_IN + s * TILE);
                uint32_t v[8];
#pragma unroll
                for (int k = 0; k < 8; ++k) v[k] = X[(8 * hf + k) * 128 + pim];
                uint8_t* A = sm + SM_OPA + o * TILE + (m & 7) * 16 + (m >> 3) * 512 + (2 * hf) * 128;
                *reinterpret_cast<uint4*>(A) = make_uint4(v[0], v[1], v[2], v[3]);
                *reinterpret_cast<uint4*>(A + 128) = make_uint4(v[4], v[5], v[6], v[7]);
                fence_async_smem();
                __syncwarp();
                if (lane == 0) bar_arrive(&B.opa_full[o]);
            };
            // ---- stage 1: pairs j = grp, grp + 2, ... (tiles 2j, 2j + 1) -> OP2 (TMEM)
            if (col) { pro(2 * grp); pro(2 * grp + 1); }
#pragma unroll 1
            for (uint32_t j = grp; j < 8; j += 2) {
                uint32_t u[2][8];
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    const uint32_t k = 2 * j + e;
                    uint32_t d[32];
                    acc_get(t1 + k, d);
                    if (col && k + NOPA < 16) pro(k + NOPA);
#pragma unroll
                    for (int c = 0; c < 8; ++c) u[e][c] = fold(d + 4 * c, nq, c16s);
                }
                if (j == grp && p > 0) { bar_wait(&B.op2_empty, (p - 1) & 1); tfence_after(); }
#pragma unroll
                for (int c = 0; c < 8; ++c)
                    tmem_st2(tmem + (lrow << 16) + TM_OP2 + 16 * (8 * hf + c) + 2 * j, u[0][c], u[1][c]);
            }
            tmem_wait_st();
            tfence_before();
            __syncwarp();
            if (lane == 0) bar_arrive(&B.op2_full);
            // ---- stage 2: tiles k = grp, grp + 2, ... -> staging -> TMA store
#pragma unroll 1
            for (uint32_t k = grp; k < 16; k += 2) {
                uint2 tw[8];
                if (col) {
                    const uint2* T = a.tw + ((((size_t)limb * 2 + h) * 16 + k) * 16 + 8 * hf) * 128 + m;
#pragma unroll
                    for (int c = 0; c < 8; ++c) tw[c] = __ldg(T + c * 128);
                }
                uint32_t d[32];
                acc_get(t2 + k, d);
                const uint32_t nsk = ns0 + k, ss = nsk % NSTG;
                bar_wait(&B.stg_empty[ss], ((nsk / NSTG) & 1) ^ 1);
                uint8_t* S = sm + SM_STG + ss * TILE;
                if (col) {
                    // Z[k1 = c + 16 d][j2] -> staging row brv4(d), word 8 e + f (pi(m) = 16 f + e)
                    uint32_t* Sw = reinterpret_cast<uint32_t*>(S) + 8 * (pim & 15) + (pim >> 4);
#pragma unroll
                    for (int dd = 0; dd < 8; ++dd)
                        Sw[brv4(8 * hf + dd) * 128] = shoup_mul(fold(d + 4 * dd, nq, c16s), tw[dd].x, tw[dd].y, q);
                } else {
                    // final outputs h' = 8 hf .. 8 hf + 7 of row m -> 64-byte swizzled staging row m
#pragma unroll
                    for (int cc = 0; cc < 2; ++cc) {
                        uint32_t y[4];
#pragma unroll
                        for (int e = 0; e < 4; ++e) y[e] = fold_canon(d + 16 * cc + 4 * e, q, nq, c16s, ones);
                        const uint32_t chunk = 2 * hf + cc;
                        *reinterpret_cast<uint4*>(S + m * 64 + ((chunk ^ ((m >> 1) & 3)) << 4)) = make_uint4(y[0], y[1], y[2], y[3]);
                    }
                }
                fence_async_smem();
                __syncwarp();
                if (lane == 0) bar_arrive(&B.stg_full[ss]);
                if (w0) TC4_TRACE(TR_STG + nsk);
            }
            t += 32;
            nin += 16;
            ns += 16;
            if (col) nopa += 16;
        }
    }
    tfence_before();
    __syncthreads();
    if (warp == W_MMA) {
        tfence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tmem));
    }
}

}  // namespace tc4
}  // namespace wd
