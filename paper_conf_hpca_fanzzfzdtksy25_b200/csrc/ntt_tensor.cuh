// ntt_tensor.cuh -- tcgen05 int8 tensor-core NTT/INTT for N = 2^16.
//
// WD-Tensor role of the paper (Alg.2 "OneStageNTTKernel";
// 4-step decomposition PAPER.md:93-100, 272-290 with inner dimension 16),
// re-derived for sm_100a:
//   * N = 2^16 = 256 columns x 256 rows; phase 1 = two radix-16 stages on
//     32-column chunks, phase 2 = two radix-16 stages on 32-row chunks
//     (intermediate through the row's own output slot, L2-resident).
//   * a radix-16 stage over 512 instances = 4 MMA tiles of M = 128 rows; one
//     row = one 16-point inner NTT whose 16 u32 inputs are 64 bytes along K
//     (the u8 view of the words, SURVEY H-3: no bit-splitting pass);
//     B = 64 x 64 byte planes of the stage matrix (tensor_tables.h);
//     D = 128 x 64 s32 in TMEM: 4 byte-plane partial sums per output.
//   * tcgen05.mma.cta_group::1.kind::i8 (u8 x u8 -> s32) issued by one thread,
//     operands in shared memory (K-major, no swizzle), accumulators in TMEM,
//     completion via tcgen05.commit -> mbarrier; two TMEM regions ping-pong so
//     the MMA of tile t+2 overlaps the epilogue of tile t.
//   * CUDA-core epilogue (tcgen05.ld 32x32b): Y = D0 + 2^8 D1 + 2^16 (D2 + 2^8 D3)
//     mod q (one Shoup multiply by 2^16), then the per-group twist of the next
//     stage (forward) / of this stage (inverse), then a conflict-free scalar
//     st.shared into the next stage's operand tile, or global stores.
//   * stage 0 (forward) / stage 0' (inverse, with N^-1) have a single group,
//     so their twist is folded into the matrix; the other stages use the fixed
//     DFT16 F (F') and a CUDA-core twist -- the paper's Hadamard step
//     (steps 2/4/6 of Fig. 2).
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include <vector>
#include <cstring>
#include "modarith.cuh"
#include "ntt_cuda_core.cuh"
#include "ntt_persist.cuh"
#include "tensor_tables.h"

namespace wd {

struct TcArgs {
    NttArgs a;
    const uint8_t* B;
    const uint2 *t1, *t2, *t3;
    const uint2* c16;
};


// ------------------------------------------------------------------ device helpers
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr) {       // K-major, SWIZZLE_NONE, LBO 128, SBO 512
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)(128 >> 4) << 16) | ((uint64_t)(512 >> 4) << 32) |
           ((uint64_t)1 << 46);
}
constexpr uint32_t IDESC_I8_128x64 = (2u << 4) | ((uint32_t)(64 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);

__device__ __forceinline__ void tc_mma(uint32_t d, uint64_t a, uint64_t b, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
                 :: "r"(d), "l"(a), "l"(b), "r"(IDESC_I8_128x64), "r"(acc));
}
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                 :: "r"(smem_addr(bar)) : "memory");
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_addr(bar)), "r"(n));
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t ph) {
    asm volatile("{\n\t.reg .pred P1;\n\tTCW_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
                 "@!P1 bra TCW_%=;\n\t}\n" :: "r"(smem_addr(bar)), "r"(ph) : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" :: "r"(id), "r"(n) : "memory"); }

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t* r) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ void cp_async4(void* smem_dst, const void* gsrc) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"(smem_addr(smem_dst)), "l"(gsrc) : "memory");
}

// byte offset of (row m, coefficient j) inside one 128 x 64-byte operand tile
__device__ __forceinline__ uint32_t aoff_w(int m, int j) {
    return (uint32_t)((m & 7) * 16 + (m >> 3) * 512 + (j >> 2) * 128 + (j & 3) * 4);
}

// Y = sum_b 2^(8b) D_b mod-ish: result < 2^32, congruent mod q
__device__ __forceinline__ uint32_t combine(const uint32_t* d, uint32_t q, uint32_t c16s) {
    const uint32_t lo = d[0] + (d[1] << 8);
    const uint32_t hi = d[2] + (d[3] << 8);
    return lo + shoup_mul(hi, 65536u, c16s, q);
}

// ------------------------------------------------------------------ the kernel
constexpr int TC_T = 128;                 // threads (4 warps; warp w owns TMEM lanes 32w..32w+31)
constexpr int TC_TILE = 128 * 64;         // bytes per operand tile
constexpr int TC_SMEM = 2 * 4 * TC_TILE   // A_in (also the inverse stage-2' staging), A_mid
                        + 2 * 4096        // B images of the current limb (folded stage, fixed DFT16)
                        + 64;             // mbarriers + TMEM address
constexpr int TC_BAR_ID = 1;              // named barrier used by the tensor group
constexpr int TC_CTAS_PER_SM = 3;         // 3 x 73 KB smem, 3 x 128 TMEM columns, 3 x 128 threads per SM

struct TcShared {
    uint8_t* Ain; uint8_t* Amid; uint8_t* B; uint64_t* bar; uint32_t* tslot;
};

// One radix-16 stage over the 4 tiles of Abuf with B image Bimg.  epi(t, half, d[32]) consumes
// outputs k = 8*half .. 8*half+7 of tile t (TMEM columns 32*half .. 32*half+31).
template <typename Epi>
__device__ __forceinline__ void tc_stage(const TcShared& sh, uint32_t tmem, const uint8_t* Abuf, const uint8_t* Bimg,
                                         uint32_t* ph, Epi&& epi) {
    const int tid = threadIdx.x % TC_T, w = tid >> 5;
    const uint32_t a0 = smem_addr(Abuf), b0 = smem_addr(Bimg);
    auto issue = [&](int t) {
        const uint32_t d = tmem + (t & 1) * 64;
        tc_fence_after();
        tc_mma(d, umma_desc(a0 + t * TC_TILE), umma_desc(b0), 0);
        tc_mma(d, umma_desc(a0 + t * TC_TILE + 256), umma_desc(b0 + 256), 1);
        tc_commit(&sh.bar[t & 1]);
    };
    if (tid == 0) { issue(0); issue(1); }
#pragma unroll 1
    for (int t = 0; t < 4; ++t) {
        const int r = t & 1;
        mbar_wait(&sh.bar[r], ph[r]);
        ph[r] ^= 1;
        tc_fence_after();
        const uint32_t ta = tmem + ((uint32_t)(32 * w) << 16) + r * 64;
        uint32_t d[32];
        tmem_ld32(ta, d);
        tmem_wait_ld();
        epi(t, 0, d);
        tmem_ld32(ta + 32, d);
        tmem_wait_ld();
        tc_fence_before();
        named_bar(TC_BAR_ID, TC_T);
        if (tid == 0 && t + 2 < 4) issue(t + 2);
        epi(t, 1, d);
    }
}

// PH = 0: the whole row; PH = 1: only the column phase (chunks of phase 1);
// PH = 2: only the row phase.  (The fused kernel splits a row's phases between the units.)
// PLAIN_MID (forward, PH = 1): store the plain merged-CT intermediate instead of pre-twisting
// it by tau2 for the tensor stage 2, so the CUDA-core butterflies can take phase 2 over.
template <bool FWD, int PH = 0, bool PLAIN_MID = false>
__device__ __forceinline__ void tc_transform(const TcArgs& ta, const TcShared& sh, uint32_t tmem, uint32_t* ph,
                                             uint32_t row_id) {
    const NttArgs& a = ta.a;
    const int tid = threadIdx.x % TC_T, w = tid >> 5, lane = tid & 31;
    const uint32_t limb = row_id % a.L;
    const LimbConst lc = a.lc[limb];
    const uint32_t q = lc.q;
    const uint2 cc = ta.c16[limb];
    const uint32_t c16s = cc.x, one_s = cc.y;
    const uint32_t* in = a.in + ((size_t)row_id << 16);
    uint32_t* out = a.out + ((size_t)row_id << 16);
    const uint8_t* Bl = ta.B + (size_t)limb * 4 * 4096 + (FWD ? 0 : 2 * 4096);
    const uint2* T1 = ta.t1 + (size_t)limb * 256;
    const uint2* T2 = ta.t2 + (size_t)limb * 4096;
    const uint2* T3 = ta.t3 + (size_t)limb * 65536;
    uint32_t* stg = reinterpret_cast<uint32_t*>(sh.Ain);      // inverse stage-2' staging (32 x 256, XOR-swizzled)

    // B images: [0] = folded single-group matrix (M0 or MI0), [1] = fixed DFT16 (F or F')
    for (int i = tid; i < 2 * 4096 / 16; i += TC_T) cp_async16(sh.B + 16 * i, Bl + 16 * i);
    cp_async_commit();

#pragma unroll 1
    for (int ch = 0; ch < 16; ++ch) {
        const bool phase1 = FWD ? (ch < 8) : (ch >= 8);
        if ((PH == 1 && !phase1) || (PH == 2 && phase1)) continue;
        const int c0 = 32 * (ch & 7), r0 = 32 * (ch & 7);
        // ---------------- chunk -> operand tiles of the first stage.  Lane maps put 8 distinct
        // (row & 7) x 4 distinct (coefficient & 3) in a warp: conflict-free 4-byte smem writes
        // and 32-byte global sectors.
        if (FWD && phase1) {                       // F-S0: (c, i0), coeff r, p = i0 + 16 r
            const int c = (lane & 7) + 8 * w, r3 = lane >> 3;
            const uint32_t* src = in + (16 * r3) * 256 + c0 + c;
            uint8_t* dst = sh.Ain + (lane & 7) * 16 + (4 * w) * 512 + r3 * 4;
#pragma unroll
            for (int i0 = 0; i0 < 16; ++i0)
#pragma unroll
                for (int rh = 0; rh < 4; ++rh)
                    cp_async4(dst + (i0 >> 2) * TC_TILE + (i0 & 3) * 512 + rh * 128, src + (i0 + 64 * rh) * 256);
        } else if (FWD) {                          // F-S2: (rho, clo), coeff chi, col = clo + 16 chi
            const int rho = (lane >> 2) + 8 * w, cl3 = lane & 3;
            const uint32_t* src = out + (r0 + rho) * 256 + cl3;
            uint8_t* dst = sh.Ain + (rho & 7) * 16 + (cl3 + 4 * w) * 512;
#pragma unroll
            for (int ch2 = 0; ch2 < 4; ++ch2)
#pragma unroll
                for (int chi = 0; chi < 16; ++chi)
                    cp_async4(dst + ch2 * TC_TILE + (chi >> 2) * 128 + (chi & 3) * 4, src + 4 * ch2 + 16 * chi);
        } else if (!phase1) {                      // I-S3: (rho, chi), coeff clo (16-byte runs)
            const int rho = (lane & 7) + 8 * w, v = lane >> 3;
            const uint32_t* src = in + (r0 + rho) * 256 + 4 * v;
            uint8_t* dst = sh.Ain + (lane & 7) * 16 + (4 * w) * 512 + v * 128;
#pragma unroll
            for (int chi = 0; chi < 16; ++chi)
                cp_async16(dst + (chi >> 2) * TC_TILE + (chi & 3) * 512, src + 16 * chi);
        } else {                                   // I-S1: (c, i1), coeff j, p = 16 i1 + j
            const int c = (lane & 7) + 8 * w, j3 = lane >> 3;
            const uint32_t* src = out + j3 * 256 + c0 + c;
            uint8_t* dst = sh.Ain + (lane & 7) * 16 + (4 * w) * 512 + j3 * 4;
#pragma unroll
            for (int i1 = 0; i1 < 16; ++i1)
#pragma unroll
                for (int jh = 0; jh < 4; ++jh)
                    cp_async4(dst + (i1 >> 2) * TC_TILE + (i1 & 3) * 512 + jh * 128, src + (16 * i1 + 4 * jh) * 256);
        }
        cp_async_commit();
        cp_async_wait<0>();
        fence_async_smem();
        named_bar(TC_BAR_ID, TC_T);

        if (FWD && phase1) {
            // stage 0 (folded M0) -> twist tau1 -> A_mid (F-S1 layout: m = 32 (k&3) + c, coeff i0)
            tc_stage(sh, tmem, sh.Ain, sh.B, ph, [&](int t, int hf, const uint32_t* d) {
                const int c = (lane & 7) + 8 * w, i0 = 4 * t + (lane >> 3);
                uint8_t* dst = sh.Amid + (c & 7) * 16 + (c >> 3) * 512 + (i0 >> 2) * 128 + (i0 & 3) * 4;
#pragma unroll
                for (int kk = 0; kk < 8; ++kk) {
                    const int k = 8 * hf + kk;
                    const uint2 tw = __ldg(T1 + k * 16 + i0);
                    const uint32_t z = shoup_mul(combine(d + 4 * kk, q, c16s), tw.x, tw.y, q);
                    *reinterpret_cast<uint32_t*>(dst + (k >> 2) * TC_TILE + (k & 3) * 2048) = z;
                }
            });
            fence_async_smem();
            named_bar(TC_BAR_ID, TC_T);
            // stage 1 (F) -> twist tau2 -> intermediate (lanes walk c: coalesced)
            tc_stage(sh, tmem, sh.Amid, sh.B + 4096, ph, [&](int t, int hf, const uint32_t* d) {
                const int i1 = 4 * t + w, c = lane;
                const uint2* t2 = T2 + (16 * i1) * 16 + ((c0 + c) >> 4);
                uint32_t* o = out + (16 * i1) * 256 + c0 + c;
#pragma unroll
                for (int kk = 0; kk < 8; ++kk) {
                    const int k = 8 * hf + kk;
                    if (PLAIN_MID) {
                        o[k * 256] = shoup_mul(combine(d + 4 * kk, q, c16s), 1u, one_s, q);   // [0, 2q)
                    } else {
                        const uint2 tw = __ldg(t2 + 16 * k);
                        o[k * 256] = shoup_mul(combine(d + 4 * kk, q, c16s), tw.x, tw.y, q);
                    }
                }
            });
        } else if (FWD) {
            // stage 2 (F) -> twist tau3 -> A_mid (F-S3 layout: m = 32 (k&3) + rho, coeff clo)
            tc_stage(sh, tmem, sh.Ain, sh.B + 4096, ph, [&](int t, int hf, const uint32_t* d) {
                const int rho = (lane & 7) + 8 * w, clo = 4 * t + (lane >> 3);
                const uint2* t3 = T3 + (size_t)(r0 + rho) * 256 + clo;        // group (row*16 + k), j = clo
                uint8_t* dst = sh.Amid + (rho & 7) * 16 + (rho >> 3) * 512 + (clo >> 2) * 128 + (clo & 3) * 4;
#pragma unroll
                for (int kk = 0; kk < 8; ++kk) {
                    const int k = 8 * hf + kk;
                    const uint2 tw = __ldg(t3 + 16 * k);
                    const uint32_t z = shoup_mul(combine(d + 4 * kk, q, c16s), tw.x, tw.y, q);
                    *reinterpret_cast<uint32_t*>(dst + (k >> 2) * TC_TILE + (k & 3) * 2048) = z;
                }
            });
            fence_async_smem();
            named_bar(TC_BAR_ID, TC_T);
            // stage 3 (F) -> canonical -> final rows (lane = row, 8 consecutive words per half)
            tc_stage(sh, tmem, sh.Amid, sh.B + 4096, ph, [&](int t, int hf, const uint32_t* d) {
                const int chi = 4 * t + w, rho = lane;
                uint4* o = reinterpret_cast<uint4*>(out + (r0 + rho) * 256 + 16 * chi + 8 * hf);
#pragma unroll
                for (int v = 0; v < 2; ++v) {
                    uint32_t y[4];
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        const uint32_t yy = shoup_mul(combine(d + 4 * (4 * v + e), q, c16s), 1u, one_s, q);
                        y[e] = umin32(yy, yy - q);
                    }
                    __stcs(o + v, make_uint4(y[0], y[1], y[2], y[3]));
                }
            });
        } else if (!phase1) {
            // stage 3' (F') -> sigma3 -> A_mid (I-S2 layout: m = 32 (k&3) + rho, coeff chi)
            tc_stage(sh, tmem, sh.Ain, sh.B + 4096, ph, [&](int t, int hf, const uint32_t* d) {
                const int rho = (lane & 7) + 8 * w, chi = 4 * t + (lane >> 3);
                const uint4* s3 = reinterpret_cast<const uint4*>(T3 + ((size_t)(r0 + rho) * 16 + chi) * 16 + 8 * hf);
                uint8_t* dst = sh.Amid + (rho & 7) * 16 + (rho >> 3) * 512 + (chi >> 2) * 128 + (chi & 3) * 4;
#pragma unroll
                for (int k2 = 0; k2 < 4; ++k2) {
                    const uint4 sg = __ldg(s3 + k2);
#pragma unroll
                    for (int e = 0; e < 2; ++e) {
                        const int kk = 2 * k2 + e, k = 8 * hf + kk;
                        const uint32_t z = shoup_mul(combine(d + 4 * kk, q, c16s), e ? sg.z : sg.x, e ? sg.w : sg.y, q);
                        *reinterpret_cast<uint32_t*>(dst + (k >> 2) * TC_TILE + (k & 3) * 2048) = z;
                    }
                }
            });
            fence_async_smem();
            named_bar(TC_BAR_ID, TC_T);
            // stage 2' (F') -> sigma2 -> staging (col XOR row swizzle) -> coalesced intermediate
            tc_stage(sh, tmem, sh.Amid, sh.B + 4096, ph, [&](int t, int hf, const uint32_t* d) {
                const int clo = 4 * t + w, rho = lane;
                const uint4* s2 = reinterpret_cast<const uint4*>(T2 + (size_t)(r0 + rho) * 16 + 8 * hf);
#pragma unroll
                for (int k2 = 0; k2 < 4; ++k2) {
                    const uint4 sg = __ldg(s2 + k2);
#pragma unroll
                    for (int e = 0; e < 2; ++e) {
                        const int kk = 2 * k2 + e, k = 8 * hf + kk;
                        const int col = clo + 16 * k;
                        stg[rho * 256 + (col ^ rho)] = shoup_mul(combine(d + 4 * kk, q, c16s), e ? sg.z : sg.x,
                                                                 e ? sg.w : sg.y, q);
                    }
                }
            });
            named_bar(TC_BAR_ID, TC_T);
#pragma unroll 4
            for (int e = tid; e < 8192; e += TC_T) {
                const int rho = e >> 8, col = e & 255;
                out[(r0 + rho) * 256 + col] = stg[rho * 256 + (col ^ rho)];
            }
        } else {
            // stage 1' (F') -> sigma1 -> A_mid (I-S0 layout: m = 32 (k&3) + c, coeff i1)
            tc_stage(sh, tmem, sh.Ain, sh.B + 4096, ph, [&](int t, int hf, const uint32_t* d) {
                const int c = (lane & 7) + 8 * w, i1 = 4 * t + (lane >> 3);
                const uint4* s1 = reinterpret_cast<const uint4*>(T1 + i1 * 16 + 8 * hf);
                uint8_t* dst = sh.Amid + (c & 7) * 16 + (c >> 3) * 512 + (i1 >> 2) * 128 + (i1 & 3) * 4;
#pragma unroll
                for (int k2 = 0; k2 < 4; ++k2) {
                    const uint4 sg = __ldg(s1 + k2);
#pragma unroll
                    for (int e = 0; e < 2; ++e) {
                        const int kk = 2 * k2 + e, k = 8 * hf + kk;
                        const uint32_t z = shoup_mul(combine(d + 4 * kk, q, c16s), e ? sg.z : sg.x, e ? sg.w : sg.y, q);
                        *reinterpret_cast<uint32_t*>(dst + (k >> 2) * TC_TILE + (k & 3) * 2048) = z;
                    }
                }
            });
            fence_async_smem();
            named_bar(TC_BAR_ID, TC_T);
            // stage 0' (folded MI0 incl. N^-1) -> canonical -> final columns (lanes walk c)
            tc_stage(sh, tmem, sh.Amid, sh.B, ph, [&](int t, int hf, const uint32_t* d) {
                const int i0 = 4 * t + w, c = lane;
                uint32_t* o = out + i0 * 256 + c0 + c;
#pragma unroll
                for (int kk = 0; kk < 8; ++kk) {
                    const int k = 8 * hf + kk;
                    uint32_t y = shoup_mul(combine(d + 4 * kk, q, c16s), 1u, one_s, q);
                    __stcs(o + 16 * k * 256, umin32(y, y - q));
                }
            });
        }
        // chunk boundary: global intermediate visible to this group's later loads; buffers free
        __threadfence_block();
        named_bar(TC_BAR_ID, TC_T);
    }
}

// ------------------------------------------------------------------ column phase with TMEM operands
// Both column stages of N = 2^16 (layers 0-7) with every twist folded: a 128-column chunk is
// processed as 16 stage-a tiles (one per value of the stage-a instance digit, all 128 columns)
// and 16 stage-b tiles (one per stage-b GROUP, all 128 columns), so every stage-b tile uses the
// single matrix of its group (M1_g / MI1_g) and no CUDA-core twist is needed.  The stage-a
// epilogue writes its outputs straight into TMEM (tcgen05.st), which is where the stage-b MMA
// takes its A operand from: the inter-stage exchange (steps 2/6 of PAPER.md Fig. 2) never
// touches shared memory.  TMEM: cols [0,256) stage-b A tiles (16 x 16 columns = 64 bytes of K
// per lane), [256,384) stage-a accumulators (ping-pong), [384,512) stage-b accumulators.
//   forward (PH1 of the row): stage a = stage 0 (instance (c, i0), coeff r, p = i0 + 16 r,
//            matrix M0), stage b = stage 1 (instance (c, i1), coeff i0, p = 16 i1 + k, M1_{i1});
//            output = plain merged-CT intermediate (or pre-twisted by tau2 for the tensor P2).
//   inverse (PH1' of the row): stage a = stage 1' (instance (c, i1), coeff j, p = 16 i1 + j,
//            MI1_{i1}), stage b = stage 0' (instance (c, i0), coeff i1, p = i0 + 16 k, MI0).
constexpr int TCC_NBUF = 6;                                  // stage-a operand ring depth
constexpr int TCC_SMEM = TCC_NBUF * TC_TILE + 17 * 4096 + 64;  // stage-a A ring + 17 B images
constexpr uint32_t TCC_A1 = 0, TCC_D0 = 256;          // D pool: 4 regions x 64 columns

struct TccShared { uint8_t* A0; uint8_t* B; uint64_t* bar; uint32_t* tslot; };

__device__ __forceinline__ void tmem_st1(uint32_t taddr, uint32_t v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" :: "r"(taddr), "r"(v) : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tc_mma_ts(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t}\n"
                 :: "r"(d), "r"(a_tmem), "l"(b), "r"(IDESC_I8_128x64), "r"(acc));
}

// one row's column phase.  TWIST2 (forward only): pre-twist the output by tau2 for tc P2.
// bar[0..1] stage-a accumulators, bar[2..3] stage-b accumulators; ph[4] their phases.
// NT = 128: each warp owns TMEM lanes 32w..32w+31 and all 64 accumulator columns of a tile;
// NT = 256: warps w and w+4 share lanes 32(w&3).. and split the columns (outputs k 0-7 / 8-15),
// halving every epilogue.
template <bool FWD, bool TWIST2, int NT = TC_T>
__device__ __forceinline__ void tcc_columns(const TcArgs& ta, const TccShared& sh, uint32_t tmem, uint32_t* ph,
                                            uint32_t row_id, const uint8_t* Gl, uint32_t* loaded_limb, int bar_id) {
    const NttArgs& a = ta.a;
    const int tid = threadIdx.x % NT, w = tid >> 5, lane = tid & 31;
    const int wq = w & 3;                        // TMEM lane quarter
    const int h0 = NT == 256 ? (w >> 2) : 0;     // first accumulator half handled by this warp
    const uint32_t limb = row_id % a.L;
    const LimbConst lc = a.lc[limb];
    const uint32_t q = lc.q, q2 = lc.q2;
    const uint2 cc = ta.c16[limb];
    const uint32_t c16s = cc.x, one_s = cc.y;
    const uint32_t* src = FWD ? a.in + ((size_t)row_id << 16) : a.out + ((size_t)row_id << 16);
    uint32_t* out = a.out + ((size_t)row_id << 16);
    const uint2* T2 = ta.t2 + (size_t)limb * 4096;
    const uint32_t lane_base = (uint32_t)(32 * wq) << 16;
    if (*loaded_limb != limb) {                  // 17 B images of this limb (68 KB), once per limb
        named_bar(bar_id, NT);
        for (int i = tid; i < 17 * 4096 / 16; i += NT) cp_async16(sh.B + 16 * i, Gl + 16 * i);
        cp_async_commit();
        cp_async_wait<0>();
        fence_async_smem();
        named_bar(bar_id, NT);
        if (tid == 0) *loaded_limb = limb;
    }
    const uint32_t b_single = smem_addr(sh.B);
    auto b_group = [&](int g) { return smem_addr(sh.B + 4096 * (1 + g)); };
    // stage-a tile t loader: element (coefficient j, row m) at p = FWD ? t + 16 j : 16 t + j
    auto load_a = [&](int t, int c0, uint8_t* buf) {
#pragma unroll
        for (int mq = 0; mq < 16 / (NT / 32); ++mq)
#pragma unroll
            for (int jh = 0; jh < 4; ++jh) {
                const int mh = w + (NT / 32) * mq, m = 8 * mh + (lane & 7), j = 4 * jh + (lane >> 3);
                const int p = FWD ? t + 16 * j : 16 * t + j;
                cp_async4(buf + (lane & 7) * 16 + mh * 512 + jh * 128 + (lane >> 3) * 4, src + p * 256 + c0 + m);
            }
        cp_async_commit();
    };
    // Both stages run as a distance-3 software pipeline over a pool of 4 TMEM accumulator
    // regions (cols [256,512), region = tile & 3, mbarrier bar[region]): iteration t first makes
    // sure operand tile t+3 is ready, issues MMA(t+3) into the region freed by epilogue t-1, then
    // runs epilogue t.  Stage-a operands come through a ring of NB shared-memory tiles; tile t+NB
    // is loaded into the buffer of tile t once epilogue t has seen MMA t complete.  At the top of
    // iteration t the issued stage-a tiles are 0 .. t+NB-1, so <= NB-4 groups may stay pending.
    constexpr int NB = TCC_NBUF;
    constexpr int PD = 3;                                  // MMA issue distance
    auto issue_a = [&](int t) {
        const uint32_t ab = smem_addr(sh.A0 + (t % NB) * TC_TILE);
        const uint32_t bb = FWD ? b_single : b_group(t);
        const uint32_t d = tmem + TCC_D0 + (t & 3) * 64;
        tc_fence_after();
        tc_mma(d, umma_desc(ab), umma_desc(bb), 0);
        tc_mma(d, umma_desc(ab + 256), umma_desc(bb + 256), 1);
        tc_commit(&sh.bar[t & 3]);
    };
    auto issue_b = [&](int k) {
        const uint32_t bb = FWD ? b_group(k) : b_single;
        const uint32_t d = tmem + TCC_D0 + (k & 3) * 64;
        tc_fence_after();
        tc_mma_ts(d, tmem + TCC_A1 + 16 * k, umma_desc(bb), 0);
        tc_mma_ts(d, tmem + TCC_A1 + 16 * k + 8, umma_desc(bb + 256), 1);
        tc_commit(&sh.bar[k & 3]);
    };
    for (int t = 0; t < NB; ++t) load_a(t, 0, sh.A0 + t * TC_TILE);
#pragma unroll 1
    for (int c0 = 0; c0 < 256; c0 += 128) {
        // ---------------- stage a: 16 tiles, A from smem, outputs -> TMEM stage-b operand tiles
        cp_async_wait<NB - PD>();                     // tiles 0..PD-1 landed
        fence_async_smem();
        tc_fence_before();
        named_bar(bar_id, NT);
        if (tid == 0) for (int t = 0; t < PD; ++t) issue_a(t);
#pragma unroll 1
        for (int t = 0; t < 16; ++t) {
            const int tn = t + PD;                    // tile whose MMA is issued in this iteration
            if (tn < 16) {
                if (t + NB - 1 <= 15) cp_async_wait<NB - PD - 1>(); else cp_async_wait<0>();
                fence_async_smem();
            }
            tc_fence_before();
            named_bar(bar_id, NT);                    // operand tile tn visible; epilogue t-1 done with its region
            if (tid == 0 && tn < 16) issue_a(tn);
            const int r = t & 3;
            mbar_wait(&sh.bar[r], (ph[0] >> r) & 1);
            ph[0] ^= 1u << r;
            tc_fence_after();
            uint32_t d[32];
#pragma unroll
            for (int hh = 0; hh < (NT == 256 ? 1 : 2); ++hh) {
                const int hf = h0 + hh;
                tmem_ld32(tmem + lane_base + TCC_D0 + r * 64 + 32 * hf, d);
                tmem_wait_ld();
#pragma unroll
                for (int kk = 0; kk < 8; ++kk) {
                    const int k = 8 * hf + kk;
                    tmem_st1(tmem + lane_base + TCC_A1 + 16 * k + t, combine(d + 4 * kk, q, c16s));
                }
            }
            if (t + NB <= 15) load_a(t + NB, c0, sh.A0 + (t % NB) * TC_TILE);   // MMA t is done
        }
        if (c0 == 0)                                  // next chunk's first tiles overlap this stage b
            for (int t = 0; t < NB; ++t) load_a(t, 128, sh.A0 + t * TC_TILE);
        tmem_wait_st();
        tc_fence_before();
        named_bar(bar_id, NT);
        // ---------------- stage b: 16 tiles, A from TMEM, outputs -> global
        if (tid == 0) for (int k = 0; k < PD; ++k) issue_b(k);
#pragma unroll 1
        for (int k = 0; k < 16; ++k) {
            const int kn = k + PD;
            if (k > 0) { tc_fence_before(); named_bar(bar_id, NT); }   // epilogue k-1 done with region (k+3)&3
            if (tid == 0 && kn < 16) issue_b(kn);
            const int r = k & 3;
            mbar_wait(&sh.bar[r], (ph[0] >> r) & 1);
            ph[0] ^= 1u << r;
            tc_fence_after();
            uint32_t d[32];
            const int m = 32 * wq + lane;
#pragma unroll
            for (int hh = 0; hh < (NT == 256 ? 1 : 2); ++hh) {
                const int hf = h0 + hh;
                tmem_ld32(tmem + lane_base + TCC_D0 + r * 64 + 32 * hf, d);
                tmem_wait_ld();
#pragma unroll
                for (int kk = 0; kk < 8; ++kk) {
                    const int ko = 8 * hf + kk;
                    const int p = FWD ? 16 * k + ko : k + 16 * ko;
                    uint32_t y = combine(d + 4 * kk, q, c16s);
                    if (FWD) {
                        if (TWIST2) {
                            const uint2 tw = __ldg(T2 + p * 16 + ((c0 + m) >> 4));
                            y = shoup_mul(y, tw.x, tw.y, q);
                        } else {
                            y = shoup_mul(y, 1u, one_s, q);                  // [0, 2q) for the butterflies
                        }
                        out[p * 256 + c0 + m] = y;
                    } else {
                        y = shoup_mul(y, 1u, one_s, q);
                        __stcs(out + p * 256 + c0 + m, umin32(y, y - q));
                    }
                }
            }
        }
        tc_fence_before();
        named_bar(bar_id, NT);                        // all stage-b epilogues done before A1 / D reuse
    }
    (void)q2;
}

// Column phase over all rows (TENSOR mode launch 1 of 2; one CTA per SM, whole TMEM).
template <bool FWD>
__global__ void __launch_bounds__(TC_T, 1) ntt_tcc16(TcArgs ta, const uint8_t* G, uint32_t rows, uint32_t per_cta) {
    extern __shared__ __align__(1024) uint8_t tsm[];
    TccShared sh;
    sh.A0 = tsm;
    sh.B = tsm + TCC_NBUF * TC_TILE;
    sh.bar = reinterpret_cast<uint64_t*>(tsm + TCC_NBUF * TC_TILE + 17 * 4096);
    sh.tslot = reinterpret_cast<uint32_t*>(sh.bar + 4);
    uint32_t* loaded = sh.tslot + 1;
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int i = 0; i < 4; ++i) mbar_init(&sh.bar[i], 1);
        *loaded = 0xffffffffu;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (tid < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(smem_addr(sh.tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *sh.tslot;
    uint32_t ph[4] = {0, 0, 0, 0};
    // contiguous (limb-major) work ranges so the 68 KB of B images are reloaded only when the limb changes
    const uint32_t L = ta.a.L, B = rows / L;
    const uint32_t k0 = blockIdx.x * per_cta, k1 = min(rows, k0 + per_cta);
    for (uint32_t k = k0; k < k1; ++k) {
        const uint32_t limb = k / B, poly = k % B, row = poly * L + limb;
        tcc_columns<FWD, true>(ta, sh, tmem, ph, row, G + ((size_t)limb * 2 + (FWD ? 0 : 1)) * 17 * 4096, loaded, TC_BAR_ID);
    }
    tc_fence_before();
    __syncthreads();
    if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tmem));
}

// Standalone tensor-core kernel: persistent CTAs of 128 threads (TENSOR mode).
template <bool FWD, int PH = 0>
__global__ void __launch_bounds__(TC_T, TC_CTAS_PER_SM) ntt_tc16(TcArgs ta, uint32_t rows) {
    extern __shared__ __align__(1024) uint8_t tsm[];
    TcShared sh;
    sh.Ain = tsm;
    sh.Amid = tsm + 4 * TC_TILE;
    sh.B = tsm + 8 * TC_TILE;
    sh.bar = reinterpret_cast<uint64_t*>(tsm + 8 * TC_TILE + 8192);
    sh.tslot = reinterpret_cast<uint32_t*>(sh.bar + 2);
    const int tid = threadIdx.x;
    if (tid == 0) {
        mbar_init(&sh.bar[0], 1);
        mbar_init(&sh.bar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (tid < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" :: "r"(smem_addr(sh.tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *sh.tslot;
    uint32_t ph[2] = {0, 0};
    for (uint32_t row = blockIdx.x; row < rows; row += gridDim.x) tc_transform<FWD, PH>(ta, sh, tmem, ph, row);
    tc_fence_before();
    __syncthreads();
    if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" :: "r"(tmem));
}

}  // namespace wd
