// ntt_v8.cuh -- CUDA-core kernel generation v8, N = 2^12 .. 2^17.
//
// Decomposition N = 2^A x 4096 (A = logN - 12), i.e. the merged-psi Cooley-Tukey network
// (Eq.(1); reading C-1) cut after its first A layers:
//   phase 1 (A layers, 0..A-1): 4096 independent columns of 2^A elements at stride 4096.
//            Register-only: a warp's 32 lanes take 32 consecutive columns, so each of a
//            thread's 2^A loads/stores is one fully used 128-byte line per warp -- no
//            shared memory, no barrier.  Output (lazy, in [0,4q)) goes to the row's out slot.
//   phase 2 (12 layers, A..A+11): 2^A contiguous 4096-word sub-rows.  A sub-row is staged
//            in shared memory by cp.async (double-buffered: sub-row s+1 loads while s
//            computes) and runs three radix-16 register stages (element strides 256, 16, 1)
//            with two in-place exchanges through a swizzled layout that is conflict-free
//            for all three access patterns; the last stage stores 16 contiguous words per
//            thread straight to global (128-bit, streaming).
// The inverse is the mirror image (phase 2' then phase 1', N^-1 folded into layer 0).
// Barriers: 1 per 4096-word sub-row and 2 per row, none in phase 1 (v6 has 6 per 4096 words):
// each warp stages its own first-stage slice, and one exchange stays inside a half-warp.
//
// Sub-row element e = a*256 + b*16 + c (a, b, c in [0,16)) lives at word
//   phys(a,b,c) = a*256 + ((b ^ (a&1)) << 4) + (c ^ (((b >> 1) & 3) << 2)):
//   stage 1 (thread (b,c), loops a), stage 2 (thread (a,c), loops b): 32 lanes hit 32
//   distinct banks; stage 3 (thread (a,b), 4 x 128-bit loads of its 16 c's): every
//   8-lane phase hits 8 distinct 16-byte bank groups.  The XOR only permutes 16-byte
//   granules, so 16-byte cp.async fills stay aligned.
#pragma once
#include "ntt_persist.cuh"
#include "ntt_smem.cuh"     // cluster_sync
#include "ntt_tensor.cuh"   // tcgen05 helpers, byte-plane tables (v10)

namespace wd {

constexpr int V8_T = 256;                    // threads per CTA (4 CTAs per SM at 64 registers)
constexpr int V8_SUBW = 4096;                // words per phase-2 sub-row
constexpr int V8_SMEM = 2 * V8_SUBW * 4;     // two sub-row buffers = 32 KB

__device__ __forceinline__ int v8_phys(int a, int b, int c) {
    return a * 256 + ((b ^ (a & 1)) << 4) + (c ^ (((b >> 1) & 3) << 2));
}

// Sub-row loads read data for the LAST time (the input, or the L2-resident intermediate); an L2
// evict-first hint would keep them from pushing other rows' intermediates out of L2 (see below).
__device__ __forceinline__ uint64_t l2_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void cp_async16_ef(void* smem_dst, const void* gsrc, uint64_t pol) {
    // NOTE: the .L2::cache_hint form of cp.async (createpolicy evict_first) faulted with an
    // illegal instruction on B200 (ptxas packs the policy into the odd UR of the memory
    // descriptor), so the hint is dropped here; pol is unused.
    (void)pol;
    cp_async16(smem_dst, gsrc);
}

// Per-warp slices: in phase 2 each warp cp.asyncs exactly the words its own FIRST stage reads,
// so the first stage needs only the warp's own wait + __syncwarp, and the stage pair that stays
// inside a half-warp (forward 2->3, inverse 3'->2') needs only __syncwarp: one CTA barrier per
// sub-row instead of three.
// forward (stage 1, thread (b,c) loops a): warp w reads words a*256 + 32w .. +31, a = 0..15
__device__ __forceinline__ void v8_load_fwd_slice(uint32_t* S, const uint32_t* src) {
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    const uint64_t pol = l2_evict_first();
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const int a = 4 * k + (l >> 3), g = l & 7;           // 128-byte segment a, granule g
        cp_async16_ef(S + v8_phys(a, 2 * w + (g >> 2), (g & 3) << 2), src + a * 256 + 32 * w + 4 * g, pol);
    }
    cp_async_commit();
}
// inverse (stage 3', thread (a,b) reads 16 contiguous c): warp w reads words 512w .. 512w + 511
__device__ __forceinline__ void v8_load_inv_slice(uint32_t* S, const uint32_t* src) {
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    const uint64_t pol = l2_evict_first();
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const int e = 512 * w + 4 * (32 * k + l);
        cp_async16_ef(S + v8_phys(e >> 8, (e >> 4) & 15, e & 15), src + e, pol);
    }
    cp_async_commit();
}

// cp.async one 4096-word sub-row (contiguous in global) into the swizzled layout
__device__ __forceinline__ void v8_load_sub(uint32_t* S, const uint32_t* src) {
    const uint64_t pol = l2_evict_first();
#pragma unroll
    for (int k = 0; k < V8_SUBW / 4 / V8_T; ++k) {
        const int G = threadIdx.x + k * V8_T;               // 16-byte granule: words 4G..4G+3
        cp_async16_ef(S + v8_phys(G >> 6, (G >> 2) & 15, (G & 3) << 2), src + 4 * G, pol);
    }
    cp_async_commit();
}

// Coalesced forward store of a sub-row's stage-3 results (v8 and the kernels sharing its layout):
// stage 3 of warp w holds words 512w .. 512w+511 (thread (aa, b): 16 contiguous words), the same
// words its stages 2 and 3 read, so the warp writes them back to its own slots of S, syncs, and
// each lane re-reads granules 128v + 4*lane: every STG.128 writes 512 contiguous bytes instead of
// 32 scattered 16-byte pieces (4x fewer L1 wavefronts).
template <typename F>
__device__ __forceinline__ void v8_store_sub(uint32_t* S, int aa, int b, const uint32_t* x, uint32_t* osub, F fin) {
    uint32_t* wb = S + aa * 256 + ((b ^ (aa & 1)) << 4);
    const int sw = (b >> 1) & 3;
#pragma unroll
    for (int v = 0; v < 4; ++v)
        *reinterpret_cast<uint4*>(wb + ((v ^ sw) << 2)) = make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
    __syncwarp();
    const int wbase = (threadIdx.x >> 5) * 512 + 4 * (threadIdx.x & 31);
#pragma unroll
    for (int v = 0; v < 4; ++v) {
        const int e = wbase + 128 * v;
        const uint4 u = *reinterpret_cast<const uint4*>(S + v8_phys(e >> 8, (e >> 4) & 15, e & 15));
        __stcs(reinterpret_cast<uint4*>(osub + e), make_uint4(fin(u.x), fin(u.y), fin(u.z), fin(u.w)));
    }
}

// MINB: resident CTAs per SM the register budget is cut for (4 -> 64 registers; 5, 6 -> 48, 40
// with per-layer just-in-time stage-3 twiddles instead of 15 preloaded pairs).
// ONLY: 1 = phase 1 only, 2 = phase 2 only, 3..8 other timing experiments (results are wrong); 9 = v8
// with the column-pass prefetch PF (correct; A/B runs).
// CL > 1: a cluster of CL CTAs shares each row -- CTA rank r takes column passes and sub-rows
// [r, r+1) * (16|R)/CL, with ONE cluster barrier (release/acquire) between the phases.  Rows
// in flight, hence the L2 footprint of the intermediate, shrink by CL.
// RESCALE input map (EPI = 1): c in [0, q_last) -> a representative in [0, 2q) of the centred
// residue v = c - q_last [c >= q_last - floor(q_last/2)] of the coefficient mod q_last, mod q
// (oracle/rns.py steps 2-4)
// c + (-q_last mod q) < 2^31 is already a valid lazy input (< 4q) when q >= 2^29 (uniform branch)
__device__ __forceinline__ uint32_t rs_in(uint32_t c, uint32_t thr, const uint4& r, uint32_t q) {
    const uint32_t v = c + (c >= thr ? r.x : 0u);
    return q >= (1u << 29) ? v : shoup_mul(v, 1u, r.y, q);
}
// RESCALE output map: y = NTT_q(v) in [0, 2q) -> (a - y) * q_last^-1 mod q, canonical (step 5)
__device__ __forceinline__ uint32_t rs_out(uint32_t aval, uint32_t y, const uint4& r, uint32_t q) {
    return canon2(shoup_mul(aval + 2 * q - y, r.z, r.w, q), q);
}

// EPI (forward only): 0 = plain NTT; 1 = RESCALE (shared last-limb input row through rs_in, output
// through rs_out against aux); 2 = ModDown (plain input rows, output through rs_out against aux)
template <int LOGN, bool FWD, bool PW, int ONLY = 0, int MINB = 4, int CL = 1, int EPI = 0>
__global__ void __launch_bounds__(V8_T, MINB) ntt_v8(NttArgs a, uint32_t rows) {
    constexpr bool JIT3 = MINB > 4;
    constexpr int A = LOGN - 12;             // phase-1 layers (radix 2^A columns)
    constexpr int R = 1 << A;                // column length = number of sub-rows
    static_assert(A >= 0 && A <= 5, "N = 2^12 .. 2^17");
    static_assert(R % CL == 0 && (V8_SUBW / V8_T) % CL == 0, "cluster splits passes and sub-rows evenly");
    constexpr int NP = V8_SUBW / V8_T / CL;  // phase-1 column passes per CTA
    constexpr int NS = R / CL;               // phase-2 sub-rows per CTA
    // PF: column passes pipelined two deep (needs 2 x 2^A data registers: A <= 4).  Opt-in
    // experiment (ONLY = 9, WD_NTT_KERNEL=v89): same-box A/B at config 3 puts it 1-2% BEHIND the
    // plain passes (forward 1.050 vs 1.040 ms, inverse 1.073 vs 1.048 ms; the inverse spills)
    constexpr bool PF = R <= 16 && NP % 2 == 0 && NP >= 2 && ONLY == 9;
    const int rank = CL > 1 ? (int)(blockIdx.x % CL) : 0;
    const int p0 = rank * NP, s0 = rank * NS, s1 = s0 + NS;
    extern __shared__ __align__(16) uint32_t smem[];
    const int t = threadIdx.x;
    const int hi4 = t >> 4, lo4 = t & 15;
    if (a.stagger_ns) {                          // experiment: start the grid's quarters staggered
        const uint32_t k = blockIdx.x * 4 / gridDim.x;
        for (uint32_t i = 0; i < k * a.stagger_ns / 1000; ++i) __nanosleep(1000);
    }

    const uint32_t nb = rows / a.L;              // polynomials in the launch
#pragma unroll 1
    for (uint32_t srow = blockIdx.x / CL; srow < rows; srow += gridDim.x / CL) {
        // limb-major schedule (a.limb_major): the rows in flight at any time share a few limbs,
        // so their twiddle tables (N x 8 bytes per limb and direction) stay a small part of L2
        // next to the L2-resident intermediates; the data layout is unchanged
        const uint32_t limb = a.limb_major ? srow / nb : srow % a.L;
        const uint32_t row = a.limb_major ? (srow - limb * nb) * a.L + limb : srow;
        const LimbConst lc = a.lc[limb];
        // the last inverse layer's constants: with the pointwise product (PW, Montgomery, which
        // leaves a factor 2^-32) they carry an extra 2^32 (N^-1 * 2^32, wn * 2^32)
        LimbConst lcl = lc;
        if constexpr (PW) { lcl.ninv = lc.ninv_r; lcl.ninv_sh = lc.ninv_r_sh; lcl.wn = lc.wn_r; lcl.wn_sh = lc.wn_r_sh; }
        const uint32_t q = lc.q, q2 = lc.q2;
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        const uint32_t* in = a.in + ((size_t)(EPI == 1 ? row / a.L : row_map(row, a.L, a.in_ls)) << LOGN);
        uint32_t* out = a.out + ((size_t)row_map(row, a.L, a.out_ls) << LOGN);
        uint4 rsc = make_uint4(0, 0, 0, 0);
        const uint32_t* ain = nullptr;
        if constexpr (EPI) {
            rsc = a.rs[limb];
            ain = a.aux + (((size_t)(row / a.L) * a.Lfull + limb) << LOGN);
        }

        if constexpr (FWD) {
            // ---- phase 1: layers 0..A-1 on columns c (elements c + 4096 k) ----
            if constexpr (A > 0 && ONLY != 2 && (ONLY < 3 || ONLY >= 7) && PF) {
                // column passes software-pipelined by two register sets: pass p+1's 2^A loads are
                // in flight while pass p computes (ncu: the first use of the column loads was the
                // top stall site, long scoreboard, with one pass in flight per thread)
                uint32_t xa[R], xb[R];
                auto ldp = [&](uint32_t (&v)[R], int pass) {
                    const int c = pass * V8_T + t;
#pragma unroll
                    for (int k = 0; k < R; ++k) v[k] = EPI == 1 ? __ldg(in + k * V8_SUBW + c) : __ldcs(in + k * V8_SUBW + c);
                };
                auto cmp = [&](uint32_t (&v)[R], int pass) {
                    const int c = pass * V8_T + t;
                    if constexpr (EPI == 1) {
#pragma unroll
                        for (int k = 0; k < R; ++k) v[k] = rs_in(v[k], a.rs_thr, rsc, q);
                    }
                    fwd_radix<A>(v, tw, 0, 0, q, q2);
#pragma unroll
                    for (int k = 0; k < R; ++k) out[k * V8_SUBW + c] = v[k];
                };
                ldp(xa, p0);
#pragma unroll 1
                for (int pass = p0; pass < p0 + NP; pass += 2) {
                    ldp(xb, pass + 1);
                    cmp(xa, pass);
                    if (pass + 2 < p0 + NP) ldp(xa, pass + 2);
                    cmp(xb, pass + 1);
                }
                if constexpr (CL > 1) cluster_sync();    // the whole intermediate is written
                else __syncthreads();
            } else if constexpr (A > 0 && ONLY != 2 && (ONLY < 3 || ONLY >= 7)) {
#pragma unroll 1
                for (int pass = p0; pass < p0 + NP; ++pass) {
                    const int c = pass * V8_T + t;
                    uint32_t x[R];
#pragma unroll
                    for (int k = 0; k < R; ++k) {
                        if constexpr (EPI == 1) x[k] = rs_in(__ldg(in + k * V8_SUBW + c), a.rs_thr, rsc, q);
                        else x[k] = __ldcs(in + k * V8_SUBW + c);
                    }
                    fwd_radix<A>(x, tw, 0, 0, q, q2);
#pragma unroll
                    for (int k = 0; k < R; ++k) out[k * V8_SUBW + c] = x[k];
                }
                if constexpr (CL > 1) cluster_sync();    // the whole intermediate is written
                else __syncthreads();
            }
            // ---- phase 2: layers A..A+11 on sub-rows s ----
            if constexpr (ONLY != 1) {
            const uint32_t* src = A > 0 ? out : in;
            if constexpr (ONLY < 3 || ONLY >= 7) v8_load_fwd_slice(smem, src + s0 * V8_SUBW);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                if constexpr (ONLY < 3 || ONLY >= 7) cp_async_wait<0>();
                __syncwarp();                            // this warp's stage-1 slice of sub-row s landed
                // ONLY 3..5 (timing experiments): 3 = no sub-row loads, 4 = no loads and no stores,
                // 5 = as 4 with every sub-row's twiddles taken from sub-row 0 (L1-resident)
                const uint32_t st = ONLY == 5 ? 0u : (uint32_t)s;
                uint32_t x[16];
                {   // stage 1: layers A..A+3, thread (b, c), elements a (stride 256)
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) {
                        x[i] = S[v8_phys(i, b, c)];
                        if constexpr (EPI == 1 && A == 0) x[i] = rs_in(x[i], a.rs_thr, rsc, q);
                    }
                    fwd_radix<4>(x, tw, A, st, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(i, b, c)] = x[i];
                }
                __syncthreads();                         // stage 1 done everywhere; sub-row s-1 fully consumed
                if ((ONLY < 3 || ONLY >= 7) && s + 1 < s1) v8_load_fwd_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, src + (s + 1) * V8_SUBW);
                uint2 w3[JIT3 ? 1 : 15];
                if constexpr (!JIT3) load_tw16(w3, tw, A + 8, st * 256 + t);   // stage-3 twiddles, in flight
                {   // stage 2: layers A+4..A+7, thread (a, c), elements b (stride 16)
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    fwd_radix<4>(x, tw, A + 4, st * 16 + aa, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                }
                __syncwarp();                            // rows a are exchanged inside the half-warp
                {   // stage 3: layers A+8..A+11, thread (a, b), 16 contiguous elements
                    const int aa = hi4, b = lo4;
                    const uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    if constexpr (JIT3) fwd_radix<4>(x, tw, A + 8, st * 256 + t, q, q2);
                    else fwd16_tw(x, w3, q, q2);
                    uint4* o = reinterpret_cast<uint4*>(out + s * V8_SUBW + t * 16);
                    if constexpr (ONLY == 6 || ONLY == 7) {   // coalesced stores in the wrong order (timing only)
                        uint4* o2 = reinterpret_cast<uint4*>(out + s * V8_SUBW);
#pragma unroll
                        for (int v = 0; v < 4; ++v)
                            __stcs(o2 + v * V8_T + t, make_uint4(canon4(x[4 * v], q, q2), canon4(x[4 * v + 1], q, q2),
                                                     canon4(x[4 * v + 2], q, q2), canon4(x[4 * v + 3], q, q2)));
                    } else if constexpr (ONLY == 4 || ONLY == 5) {
                        uint32_t z = 0;
#pragma unroll
                        for (int i = 0; i < 16; ++i) z ^= x[i];
                        if (z == 0xFFFFFFFFu && x[0] == 0xFFFFFFFFu) o[0] = make_uint4(z, z, z, z);
                    } else if constexpr (ONLY != 8) {
                        // Coalesced store through the warp's own 2 KB of S: stage 3 of warp w covers
                        // words 512w .. 512w+511 of the sub-row, so after writing them back (the same
                        // conflict-free 16-byte slots it read) each lane re-reads granules 128v + 4*lane
                        // and every STG.128 of the warp writes 512 contiguous bytes (the direct
                        // per-thread 64-byte stores cost 4x the L1 wavefronts: v86 vs v83, DESIGN 5.1).
                        uint32_t* wb = S + aa * 256 + ((b ^ (aa & 1)) << 4);
#pragma unroll
                        for (int v = 0; v < 4; ++v)
                            *reinterpret_cast<uint4*>(wb + ((v ^ sw) << 2)) =
                                make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
                        __syncwarp();
                        const int wbase = (t >> 5) * 512 + 4 * (t & 31);
#pragma unroll
                        for (int v = 0; v < 4; ++v) {
                            const int e = wbase + 128 * v;
                            const uint4 u = *reinterpret_cast<const uint4*>(S + v8_phys(e >> 8, (e >> 4) & 15, e & 15));
                            uint4* og = reinterpret_cast<uint4*>(out + s * V8_SUBW + e);
                            if constexpr (EPI) {
                                const uint4 av = __ldcs(reinterpret_cast<const uint4*>(ain + s * V8_SUBW + e));
                                __stcs(og, make_uint4(rs_out(av.x, umin32(u.x, u.x - q2), rsc, q),
                                                      rs_out(av.y, umin32(u.y, u.y - q2), rsc, q),
                                                      rs_out(av.z, umin32(u.z, u.z - q2), rsc, q),
                                                      rs_out(av.w, umin32(u.w, u.w - q2), rsc, q)));
                            } else {
                                __stcs(og, make_uint4(canon4(u.x, q, q2), canon4(u.y, q, q2),
                                                      canon4(u.z, q, q2), canon4(u.w, q, q2)));
                            }
                        }
                    } else if constexpr (EPI) {
                        const uint4* ai = reinterpret_cast<const uint4*>(ain + s * V8_SUBW + t * 16);
#pragma unroll
                        for (int v = 0; v < 4; ++v) {
                            const uint4 u = __ldcs(ai + v);
                            __stcs(o + v, make_uint4(rs_out(u.x, umin32(x[4 * v], x[4 * v] - q2), rsc, q),
                                                     rs_out(u.y, umin32(x[4 * v + 1], x[4 * v + 1] - q2), rsc, q),
                                                     rs_out(u.z, umin32(x[4 * v + 2], x[4 * v + 2] - q2), rsc, q),
                                                     rs_out(u.w, umin32(x[4 * v + 3], x[4 * v + 3] - q2), rsc, q)));
                        }
                    } else {
#pragma unroll
                    for (int v = 0; v < 4; ++v)
                        __stcs(o + v, make_uint4(canon4(x[4 * v], q, q2), canon4(x[4 * v + 1], q, q2),
                                                 canon4(x[4 * v + 2], q, q2), canon4(x[4 * v + 3], q, q2)));
                    }
                }
            }
            }
        } else {
            // ---- phase 2': layers A+11..A on sub-rows s (input in bit-reversed order) ----
            if constexpr (ONLY != 1) {
            const uint32_t* in2 = a.in2 + ((size_t)row << LOGN);
            v8_load_inv_slice(smem, in + s0 * V8_SUBW);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                uint2 w3[JIT3 ? 1 : 15];
                if constexpr (!JIT3) load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);   // in flight across the wait
                cp_async_wait<0>();
                __syncwarp();                            // this warp's rows of sub-row s landed
                if (a.cpy) {                             // ModUp: pass the NTT-domain input through
                    const int wbase = (t >> 5) * 512 + 4 * (t & 31);
                    uint32_t* cp = a.cpy + ((size_t)row_map(row, a.L, a.cpy_ls) << LOGN) + s * V8_SUBW;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {        // the warp's own 2 KB slice, 512 B per store
                        const int e = wbase + 128 * v;
                        __stcs(reinterpret_cast<uint4*>(cp + e),
                               *reinterpret_cast<const uint4*>(S + v8_phys(e >> 8, (e >> 4) & 15, e & 15)));
                    }
                }
                if constexpr (PW) {                      // row f1: pointwise product, coalesced
                    // the warp's own 2 KB slice: in2 read 512 B per instruction, the Montgomery
                    // product a*b*2^-32 in (0, 2q) written back to the same shared-memory slots
                    // before stage 3' reads them; the last layer's lcl constants restore 2^32
                    const int wbase = (t >> 5) * 512 + 4 * (t & 31);
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const int e = wbase + 128 * v;
                        uint4* sp = reinterpret_cast<uint4*>(S + v8_phys(e >> 8, (e >> 4) & 15, e & 15));
                        const uint4 u = *sp;
                        const uint4 m = __ldcs(reinterpret_cast<const uint4*>(in2 + s * V8_SUBW + e));
                        *sp = make_uint4(mont_mul(u.x, m.x, lc), mont_mul(u.y, m.y, lc), mont_mul(u.z, m.z, lc),
                                         mont_mul(u.w, m.w, lc));
                    }
                    __syncwarp();
                }
                uint32_t x[16];
                {   // stage 3': layers A+11..A+8, thread (a, b), 16 contiguous elements
                    const int aa = hi4, b = lo4;
                    uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    if constexpr (JIT3) inv_radix<4, false>(x, tw, A + 8, (uint32_t)s * 256 + t, lc);
                    else inv16_tw(x, w3, q, q2);
#pragma unroll
                    for (int v = 0; v < 4; ++v)
                        *reinterpret_cast<uint4*>(base + ((v ^ sw) << 2)) =
                            make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
                }
                __syncwarp();                            // rows a are exchanged inside the half-warp
                {   // stage 2': layers A+7..A+4, thread (a, c), elements b
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    inv_radix<4, false>(x, tw, A + 4, (uint32_t)s * 16 + aa, lc);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                }
                __syncthreads();                         // stage 2' done everywhere; sub-row s-1 fully consumed
                if (s + 1 < s1) v8_load_inv_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, in + (s + 1) * V8_SUBW);
                {   // stage 1': layers A+3..A, thread (b, c), elements a -> global (coalesced)
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    inv_radix<4, A == 0>(x, tw, A, (uint32_t)s, lcl);
                    uint32_t* o = out + s * V8_SUBW + b * 16 + c;
#pragma unroll
                    for (int i = 0; i < 16; ++i) {
                        if constexpr (A == 0) __stcs(o + i * 256, canon2(x[i], q));
                        else o[i * 256] = x[i];             // lazy intermediate, in [0,2q)
                    }
                }
            }
            }
            // ---- phase 1': layers A-1..0 on columns, N^-1 folded into layer 0 ----
            if constexpr (A > 0 && ONLY != 2) {
                if constexpr (CL > 1) cluster_sync();    // the whole intermediate is written
                else __syncthreads();
                if constexpr (PF) {                       // two register sets, as in phase 1
                    uint32_t xa[R], xb[R];
                    auto ldp = [&](uint32_t (&v)[R], int pass) {
                        const int c = pass * V8_T + t;
#pragma unroll
                        for (int k = 0; k < R; ++k) v[k] = __ldcs(out + k * V8_SUBW + c);   // last use
                    };
                    auto cmp = [&](uint32_t (&v)[R], int pass) {
                        const int c = pass * V8_T + t;
                        inv_radix<A, true>(v, tw, 0, 0, lcl);
#pragma unroll
                        for (int k = 0; k < R; ++k) __stcs(out + k * V8_SUBW + c, canon2(v[k], q));
                    };
                    ldp(xa, p0);
#pragma unroll 1
                    for (int pass = p0; pass < p0 + NP; pass += 2) {
                        ldp(xb, pass + 1);
                        cmp(xa, pass);
                        if (pass + 2 < p0 + NP) ldp(xa, pass + 2);
                        cmp(xb, pass + 1);
                    }
                } else
#pragma unroll 1
                for (int pass = p0; pass < p0 + NP; ++pass) {
                    const int c = pass * V8_T + t;
                    uint32_t x[R];
#pragma unroll
                    for (int k = 0; k < R; ++k) x[k] = __ldcs(out + k * V8_SUBW + c);
                    inv_radix<A, true>(x, tw, 0, 0, lcl);
#pragma unroll
                    for (int k = 0; k < R; ++k) __stcs(out + k * V8_SUBW + c, canon2(x[k], q));
                }
            }
        }
        __syncthreads();                                 // smem buffers free for the next row
    }
}


// ---------------------------------------------------------------------------------------------
// v9: v8 with the column phase staged through shared memory by cp.async (N = 2^13 .. 2^16).
// ncu of v8 (profiles/r01/g1) puts ~20% of the stall samples on the first use of the column
// loads (long scoreboard): a thread issues its 2^A column loads and waits for them.  Here each
// warp prefetches its OWN slice of the next column pass (2^A rows x 32 words, 16-byte
// cp.async) while it computes the current one, so no CTA barrier is added; a third buffer
// takes the first unit of the NEXT row (forward: its first column pass, issued at the start of
// this row's sub-row phase; inverse: its first sub-row, issued at the start of the column
// phase), so the HBM latency of every input unit is hidden behind the current row's work.
constexpr int V9_SMEM = 3 * V8_SUBW * 4;     // B0, B1 (ping-pong), B2 (next-row unit) = 48 KB

// column pass slice of warp w: rows k = 0..R-1 of columns c0 + 32w .. c0 + 32w + 31 of `src`
// -> buf[w*32R + 32k + lane] (warp-private: the warp alone writes and reads it)
template <int R>
__device__ __forceinline__ void v9_load_cols(uint32_t* buf, const uint32_t* src, int c0) {
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    uint32_t* b = buf + w * 32 * R;
    const uint32_t* g = src + c0 + 32 * w;
#pragma unroll
    for (int G = l; G < R * 8; G += 32)                 // granule G: row G/8, words 4(G%8)..+3
        cp_async16(b + (G >> 3) * 32 + 4 * (G & 7), g + (G >> 3) * V8_SUBW + 4 * (G & 7));
    cp_async_commit();
}

template <int LOGN, bool FWD, bool PW, int CL = 1>
__global__ void __launch_bounds__(V8_T, 4) ntt_v9(NttArgs a, uint32_t rows) {
    constexpr int A = LOGN - 12;
    constexpr int R = 1 << A;
    static_assert(A >= 1 && A <= 4, "v9: N = 2^13 .. 2^16 (a column pass must fit one 16 KB buffer)");
    static_assert(R % CL == 0 && (V8_SUBW / V8_T) % CL == 0, "cluster splits passes and sub-rows evenly");
    constexpr int NP = V8_SUBW / V8_T / CL;
    constexpr int NS = R / CL;
    const int rank = CL > 1 ? (int)(blockIdx.x % CL) : 0;
    const int p0 = rank * NP, s0 = rank * NS, s1 = s0 + NS;
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* const B0 = smem;
    uint32_t* const B1 = smem + V8_SUBW;
    uint32_t* const B2 = smem + 2 * V8_SUBW;
    const int t = threadIdx.x, w = t >> 5, lane = t & 31;
    const int hi4 = t >> 4, lo4 = t & 15;
    const uint32_t rstep = gridDim.x / CL;
    uint32_t row = blockIdx.x / CL;

    // prologue: the first unit of the first row into B2 (forward) / B0 (inverse)
    if (row < rows) {
        if constexpr (FWD) v9_load_cols<R>(B2, a.in + ((size_t)row << LOGN), p0 * V8_T);
        else v8_load_inv_slice(B0, a.in + ((size_t)row << LOGN) + s0 * V8_SUBW);
    }
#pragma unroll 1
    for (; row < rows; row += rstep) {
        const uint32_t nrow = row + rstep;
        const uint32_t limb = row % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q, q2 = lc.q2;
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        const uint32_t* in = a.in + ((size_t)row << LOGN);
        uint32_t* out = a.out + ((size_t)row << LOGN);

        if constexpr (FWD) {
            // ---- phase 1: layers 0..A-1 on columns; pass i in B2 (i = 0) or B[(i-1)&1]
#pragma unroll 1
            for (int i = 0; i < NP; ++i) {
                const uint32_t* buf = i == 0 ? B2 : ((i - 1) & 1 ? B1 : B0);
                if (i + 1 < NP) {
                    __syncwarp();                                   // pass i-1's slice fully read
                    v9_load_cols<R>(i & 1 ? B1 : B0, in, (p0 + i + 1) * V8_T);
                    cp_async_wait<1>();
                } else {
                    cp_async_wait<0>();
                }
                __syncwarp();
                uint32_t x[R];
#pragma unroll
                for (int k = 0; k < R; ++k) x[k] = buf[w * 32 * R + 32 * k + lane];
                fwd_radix<A>(x, tw, 0, 0, q, q2);
                const int c = (p0 + i) * V8_T + t;
#pragma unroll
                for (int k = 0; k < R; ++k) out[k * V8_SUBW + c] = x[k];
            }
            if constexpr (CL > 1) cluster_sync(); else __syncthreads();
            // ---- phase 2: layers A..A+11 on sub-rows; the next row's first pass goes to B2
            v8_load_fwd_slice(B0, out + s0 * V8_SUBW);
            if (nrow < rows) v9_load_cols<R>(B2, a.in + ((size_t)nrow << LOGN), p0 * V8_T);
            else cp_async_commit();                                 // keep the group count uniform
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = (s - s0) & 1 ? B1 : B0;
                if (s == s0) cp_async_wait<1>(); else cp_async_wait<0>();
                __syncwarp();
                uint32_t x[16];
                {
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    fwd_radix<4>(x, tw, A, (uint32_t)s, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(i, b, c)] = x[i];
                }
                __syncthreads();
                if (s + 1 < s1) v8_load_fwd_slice((s + 1 - s0) & 1 ? B1 : B0, out + (s + 1) * V8_SUBW);
                uint2 w3[15];
                load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                {
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    fwd_radix<4>(x, tw, A + 4, (uint32_t)s * 16 + aa, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                }
                __syncwarp();
                {
                    const int aa = hi4, b = lo4;
                    const uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    fwd16_tw(x, w3, q, q2);
                    v8_store_sub(S, aa, b, x, out + s * V8_SUBW, [&](uint32_t y) { return canon4(y, q, q2); });
                }
            }
        } else {
            // ---- phase 2': layers A+11..A on sub-rows (the first one is already in flight in B0)
            const uint32_t* in2 = a.in2 + ((size_t)row << LOGN);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = (s - s0) & 1 ? B1 : B0;
                uint2 w3[15];
                load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                cp_async_wait<0>();
                __syncwarp();
                uint32_t x[16];
                {
                    const int aa = hi4, b = lo4;
                    uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    if constexpr (PW) {
                        const uint4* ip2 = reinterpret_cast<const uint4*>(in2 + s * V8_SUBW + t * 16);
#pragma unroll
                        for (int v = 0; v < 4; ++v) {
                            const uint4 u = __ldcs(ip2 + v);
                            x[4 * v] = mul_mod(x[4 * v], u.x, lc); x[4 * v + 1] = mul_mod(x[4 * v + 1], u.y, lc);
                            x[4 * v + 2] = mul_mod(x[4 * v + 2], u.z, lc); x[4 * v + 3] = mul_mod(x[4 * v + 3], u.w, lc);
                        }
                    }
                    inv16_tw(x, w3, q, q2);
#pragma unroll
                    for (int v = 0; v < 4; ++v)
                        *reinterpret_cast<uint4*>(base + ((v ^ sw) << 2)) =
                            make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
                }
                __syncwarp();
                {
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    inv_radix<4, false>(x, tw, A + 4, (uint32_t)s * 16 + aa, lc);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                }
                __syncthreads();
                if (s + 1 < s1) v8_load_inv_slice((s + 1 - s0) & 1 ? B1 : B0, in + (s + 1) * V8_SUBW);
                {
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    inv_radix<4, false>(x, tw, A, (uint32_t)s, lc);
                    uint32_t* o = out + s * V8_SUBW + b * 16 + c;
#pragma unroll
                    for (int i = 0; i < 16; ++i) o[i * 256] = x[i];             // lazy intermediate, [0,2q)
                }
            }
            if constexpr (CL > 1) cluster_sync(); else __syncthreads();
            // ---- phase 1': layers A-1..0 on columns (N^-1 folded); pass i in B2 / B1 alternately,
            // the next row's first sub-row goes to B0
            v9_load_cols<R>(B2, out, p0 * V8_T);
            if (nrow < rows) v8_load_inv_slice(B0, a.in + ((size_t)nrow << LOGN) + s0 * V8_SUBW);
            else cp_async_commit();
#pragma unroll 1
            for (int i = 0; i < NP; ++i) {
                const uint32_t* buf = i & 1 ? B1 : B2;
                if (i + 1 < NP) {
                    __syncwarp();
                    v9_load_cols<R>(i & 1 ? B2 : B1, out, (p0 + i + 1) * V8_T);
                    if (i == 0) cp_async_wait<2>();                 // the next row's sub-row may stay in flight
                    else cp_async_wait<1>();
                } else {
                    cp_async_wait<0>();
                }
                __syncwarp();
                uint32_t x[R];
#pragma unroll
                for (int k = 0; k < R; ++k) x[k] = buf[w * 32 * R + 32 * k + lane];
                inv_radix<A, true>(x, tw, 0, 0, lc);
                const int c = (p0 + i) * V8_T + t;
#pragma unroll
                for (int k = 0; k < R; ++k) __stcs(out + k * V8_SUBW + c, canon2(x[k], q));
            }
        }
        __syncthreads();                                 // B0/B1 free for the next row
    }
    cp_async_wait<0>();
}


// ---------------------------------------------------------------------------------------------
// v10 (N = 2^16): v8 with its column phase on the tensor cores -- the concurrent tensor +
// CUDA-core design of SURVEY.md 8 row a9 (PAPER.md:316-330 WD-FUSE, re-derived for sm_100a).
// The column phase (layers 0..3, forward; layers 3..0 with N^-1, inverse) is ONE 16x16 matrix
// M0 (MI0) applied to all 4096 columns of the row, i.e. a plain GEMM X[4096 x 16] . M0^T: it runs
// as tcgen05.mma.kind::i8 tiles of 128 columns (byte-plane identity of ntt_tensor.cuh: the u8 view
// of the 16 input words is K = 64, the 4 pre-shifted byte planes of M0 are N = 64).  The
// per-element-twiddle layers 4..15 stay on the CUDA cores (v8 phase 2).  Warps of the 4
// co-resident CTAs of an SM are in different phases at any time, so the tensor pipe and the
// CUDA-core butterflies overlap on the same SM.  Per 128-column tile: the 8 warps load the tile
// (warp w: 32 columns x 8 coefficients, coalesced) straight into TMEM (tcgen05.st, lane =
// column, column = coefficient: the A operand), one thread issues 2 MMAs (K = 2 x 32 bytes),
// every warp reads its 8 outputs x 4 planes back (tcgen05.ld) and recombines them:
//   y = (D0 + 2^8 D1) + Shoup(D2 + 2^8 D3, 2^16)   (D_b < 2^22, so D0 + 2^8 D1 < 2^30)
// which is < 2^30 + 2q, i.e. < 4q (the CT butterflies' input range) once q > 2^29.
// TMEM: 128 columns per CTA (4 CTAs per SM = all 512): [0,16) A, [64,128) D.
constexpr int V10_SMEM = V8_SMEM + 4096 + 64;            // sub-row buffers, B planes, mbarrier + TMEM slot

__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t* v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
                 :: "r"(taddr), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
                 : "memory");
}

// y = sum_b 2^(8b) D_b (mod q) in [0, 4q) for every q < 2^30 (the q <= 2^29 branch reduces the
// low half first); uniform branch per limb
__device__ __forceinline__ uint32_t v10_combine(const uint32_t* d, uint32_t q, uint32_t q2, uint32_t c16s,
                                                uint32_t one_s) {
    const uint32_t lo = d[0] + (d[1] << 8);
    const uint32_t hi = shoup_mul(d[2] + (d[3] << 8), 65536u, c16s, q);
    if (q > (1u << 29)) return lo + hi;
    return shoup_mul(lo, 1u, one_s, q) + hi;
}

// the column phase of one row on the tensor cores: tiles of 128 columns [c_lo, c_hi)
// FWD: src = input row, dst = intermediate (lazy [0,4q)); inverse: src = dst = row's out slot,
// canonical result.  Bt = the 4 KB byte-plane image of M0 / MI0 (already in smem, fenced).
template <bool FWD>
__device__ __forceinline__ void v10_columns(const uint32_t* src, uint32_t* dst, int c_lo, int c_hi,
                                            uint32_t tmem, uint32_t bt, uint64_t* bar, uint32_t& ph,
                                            uint32_t q, uint32_t q2, uint32_t c16s, uint32_t one_s) {
    const int t = threadIdx.x, w = t >> 5, lane = t & 31;
    const int lq = w & 3, kh = w >> 2;                     // TMEM lane quarter, coefficient half
    const uint32_t tl = tmem + ((uint32_t)(32 * lq) << 16);
    uint32_t x[8];
    int c = c_lo + 32 * lq + lane;
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] = FWD ? __ldcs(src + (8 * kh + i) * V8_SUBW + c) : src[(8 * kh + i) * V8_SUBW + c];
#pragma unroll 1
    for (int c0 = c_lo; c0 < c_hi; c0 += 128) {
        tmem_st8(tl + 8 * kh, x);                          // A: lane = column, TMEM column = coefficient
        tmem_wait_st();
        tc_fence_before();
        __syncthreads();                                   // A complete; the previous tile's D fully read
        if (t == 0) {
            tc_fence_after();
            tc_mma_ts(tmem + 64, tmem, umma_desc(bt), 0);
            tc_mma_ts(tmem + 64, tmem + 8, umma_desc(bt + 256), 1);
            tc_commit(bar);
        }
        c = c0 + 32 * lq + lane;
        if (c0 + 128 < c_hi) {                             // next tile's loads in flight during the MMA
            const int cn = c + 128;
#pragma unroll
            for (int i = 0; i < 8; ++i) x[i] = FWD ? __ldcs(src + (8 * kh + i) * V8_SUBW + cn) : src[(8 * kh + i) * V8_SUBW + cn];
        }
        mbar_wait(bar, ph);
        ph ^= 1;
        tc_fence_after();
        uint32_t d[32];
        tmem_ld32(tl + 64 + 32 * kh, d);                   // outputs k = 8 kh .. 8 kh + 7, 4 planes each
        tmem_wait_ld();
        tc_fence_before();
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
            const uint32_t y = v10_combine(d + 4 * kk, q, q2, c16s, one_s);
            if (FWD) dst[(8 * kh + kk) * V8_SUBW + c] = y;
            else __stcs(dst + (8 * kh + kk) * V8_SUBW + c, canon4(y, q, q2));
        }
    }
}

template <bool FWD, bool PW, int CL = 2>
__global__ void __launch_bounds__(V8_T, 4) ntt_v10(NttArgs a, const uint8_t* G, const uint2* c16, uint32_t rows) {
    constexpr int LOGN = 16, A = 4;
    constexpr int NP = V8_SUBW / V8_T / CL;
    constexpr int NS = 16 / CL;
    const int rank = CL > 1 ? (int)(blockIdx.x % CL) : 0;
    const int p0 = rank * NP, s0 = rank * NS, s1 = s0 + NS;
    extern __shared__ __align__(1024) uint32_t smem_v10[];
    uint32_t* const smem = smem_v10;
    uint8_t* Bt = reinterpret_cast<uint8_t*>(smem + 2 * V8_SUBW);
    uint64_t* bar = reinterpret_cast<uint64_t*>(Bt + 4096);
    uint32_t* tslot = reinterpret_cast<uint32_t*>(bar + 1);
    const int t = threadIdx.x;
    const int hi4 = t >> 4, lo4 = t & 15;
    if (t == 0) {
        mbar_init(bar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (t < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" :: "r"(smem_addr(tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tslot;
    const uint32_t bt = smem_addr(Bt);
    uint32_t ph = 0;

#pragma unroll 1
    for (uint32_t row = blockIdx.x / CL; row < rows; row += gridDim.x / CL) {
        const uint32_t limb = row % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q, q2 = lc.q2;
        const uint2 cc = c16[limb];
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        const uint32_t* in = a.in + ((size_t)row << LOGN);
        uint32_t* out = a.out + ((size_t)row << LOGN);
        // B planes of this limb's single-group column matrix (M0 forward, MI0 inverse)
        cp_async16(Bt + 16 * t, G + ((size_t)limb * 2 + (FWD ? 0 : 1)) * 17 * 4096 + 16 * t);
        cp_async_commit();

        if constexpr (FWD) {
            cp_async_wait<0>();
            fence_async_smem();
            // ---- phase 1 on the tensor cores (the __syncthreads inside publishes Bt)
            v10_columns<true>(in, out, p0 * V8_T, (p0 + NP) * V8_T, tmem, bt, bar, ph, q, q2, cc.x, cc.y);
            if constexpr (CL > 1) cluster_sync(); else __syncthreads();
            // ---- phase 2: layers 4..15 on sub-rows (v8)
            v8_load_fwd_slice(smem, out + s0 * V8_SUBW);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                cp_async_wait<0>();
                __syncwarp();
                uint32_t x[16];
                {
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    fwd_radix<4>(x, tw, A, (uint32_t)s, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(i, b, c)] = x[i];
                }
                __syncthreads();
                if (s + 1 < s1) v8_load_fwd_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, out + (s + 1) * V8_SUBW);
                uint2 w3[15];
                load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                {
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    fwd_radix<4>(x, tw, A + 4, (uint32_t)s * 16 + aa, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                }
                __syncwarp();
                {
                    const int aa = hi4, b = lo4;
                    const uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    fwd16_tw(x, w3, q, q2);
                    v8_store_sub(S, aa, b, x, out + s * V8_SUBW, [&](uint32_t y) { return canon4(y, q, q2); });
                }
            }
        } else {
            // ---- phase 2': layers 15..4 on sub-rows (v8)
            const uint32_t* in2 = a.in2 + ((size_t)row << LOGN);
            v8_load_inv_slice(smem, in + s0 * V8_SUBW);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                uint2 w3[15];
                load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                cp_async_wait<0>();
                __syncwarp();
                uint32_t x[16];
                {
                    const int aa = hi4, b = lo4;
                    uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    if constexpr (PW) {
                        const uint4* ip2 = reinterpret_cast<const uint4*>(in2 + s * V8_SUBW + t * 16);
#pragma unroll
                        for (int v = 0; v < 4; ++v) {
                            const uint4 u = __ldcs(ip2 + v);
                            x[4 * v] = mul_mod(x[4 * v], u.x, lc); x[4 * v + 1] = mul_mod(x[4 * v + 1], u.y, lc);
                            x[4 * v + 2] = mul_mod(x[4 * v + 2], u.z, lc); x[4 * v + 3] = mul_mod(x[4 * v + 3], u.w, lc);
                        }
                    }
                    inv16_tw(x, w3, q, q2);
#pragma unroll
                    for (int v = 0; v < 4; ++v)
                        *reinterpret_cast<uint4*>(base + ((v ^ sw) << 2)) =
                            make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
                }
                __syncwarp();
                {
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    inv_radix<4, false>(x, tw, A + 4, (uint32_t)s * 16 + aa, lc);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                }
                __syncthreads();
                if (s + 1 < s1) v8_load_inv_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, in + (s + 1) * V8_SUBW);
                {
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    inv_radix<4, false>(x, tw, A, (uint32_t)s, lc);
                    uint32_t* o = out + s * V8_SUBW + b * 16 + c;
#pragma unroll
                    for (int i = 0; i < 16; ++i) o[i * 256] = x[i];
                }
            }
            cp_async_wait<0>();
            fence_async_smem();
            if constexpr (CL > 1) cluster_sync(); else __syncthreads();
            // ---- phase 1' on the tensor cores: layers 3..0 with N^-1 (MI0), canonical output
            v10_columns<false>(out, out, p0 * V8_T, (p0 + NP) * V8_T, tmem, bt, bar, ph, q, q2, cc.x, cc.y);
        }
        __syncthreads();                                 // smem buffers / Bt free for the next row
    }
    tc_fence_before();
    __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" :: "r"(tmem));
}


// ---------------------------------------------------------------------------------------------
// WD-CUDA ("CUDA Cores ... directly compute high-precision
// (32-bit) GEMM"): the same 4 radix-16 stages of N = 2^16 as the tensor path, but
// every inner 16-point DFT is a 32-bit matrix-vector product on the CUDA cores --
//   forward stage s >= 1:  x_j <- x_j * tau_g[j];  y = F x        (stage 0: y = M0 x)
//   inverse stage s >= 1:  y = F' x;  y_k <- y_k * sigma_g[k]      (stage 0': y = MI0 x, N^-1 in MI0)
// with the matrices and twists of the tensor tables (ntt_tensor.cuh build_tensor_tables), each
// output a pair of 8-term 64-bit multiply-accumulates (x < 2^31, M < 2^30: < 2^64) reduced by a
// 64-bit Barrett step.  It is the paper's comparison variant (Fig. 6): 16 wide multiplies per
// element per stage instead of 2 Shoup butterflies, so it is expected to be slower than WD-BO.
// Data movement is v8's (N = 16 x 4096, 2-CTA cluster per row).
__device__ __forceinline__ uint32_t wdc_reduce(uint64_t v, const LimbConst& lc) {
    const uint64_t quo = __umul64hi(v, lc.mu);
    const uint32_t r = (uint32_t)(v - quo * lc.q);       // < 3q
    return umin32(r, r - lc.q);                          // < 2q (lazy)
}
// y = M x (M row-major [16][16] in shared memory, broadcast reads), x_j < 2^31 -> y_k < 4q
__device__ __forceinline__ void wdc_gemm16(uint32_t* x, const uint32_t* M, const LimbConst& lc) {
    uint32_t y[16];
#pragma unroll
    for (int k = 0; k < 16; ++k) {
        const uint4* row = reinterpret_cast<const uint4*>(M + 16 * k);
        uint64_t a0 = 0, a1 = 0;
#pragma unroll
        for (int v = 0; v < 2; ++v) {
            const uint4 m = row[v];
            a0 += (uint64_t)x[4 * v] * m.x + (uint64_t)x[4 * v + 1] * m.y + (uint64_t)x[4 * v + 2] * m.z +
                  (uint64_t)x[4 * v + 3] * m.w;
        }
#pragma unroll
        for (int v = 2; v < 4; ++v) {
            const uint4 m = row[v];
            a1 += (uint64_t)x[4 * v] * m.x + (uint64_t)x[4 * v + 1] * m.y + (uint64_t)x[4 * v + 2] * m.z +
                  (uint64_t)x[4 * v + 3] * m.w;
        }
        y[k] = wdc_reduce(a0, lc) + wdc_reduce(a1, lc);
    }
#pragma unroll
    for (int k = 0; k < 16; ++k) x[k] = y[k];
}
// x_j <- x_j * t[j] (Shoup, result < 2q); t = 16 consecutive (w, w') pairs of one group
__device__ __forceinline__ void wdc_twist(uint32_t* x, const uint2* __restrict__ t, uint32_t q) {
#pragma unroll
    for (int j = 0; j < 16; j += 2) {
        const uint4 w = __ldg(reinterpret_cast<const uint4*>(t + j));
        x[j] = shoup_mul(x[j], w.x, w.y, q);
        x[j + 1] = shoup_mul(x[j + 1], w.z, w.w, q);
    }
}
__device__ __forceinline__ uint32_t wdc_canon(uint32_t v, uint32_t q, uint32_t q2) { return canon4(v, q, q2); }

struct WdcArgs {
    NttArgs a;
    const uint32_t* mat;     // [L][4][256]: M0, F, MI0 (with N^-1), F'
    const uint2 *t1, *t2, *t3;   // twists of this direction: tau (forward) / sigma (inverse)
};

template <bool FWD>
__global__ void __launch_bounds__(V8_T, 3) ntt_wdcuda16(WdcArgs wa, uint32_t rows) {
    constexpr int LOGN = 16, CL = 2;
    constexpr int NP = V8_SUBW / V8_T / CL, NS = 16 / CL;
    const NttArgs& a = wa.a;
    const int rank = (int)(blockIdx.x % CL);
    const int p0 = rank * NP, s0 = rank * NS, s1 = s0 + NS;
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* Mst = smem + 2 * V8_SUBW;                 // [2][256]: stage-0 matrix, fixed DFT
    const int t = threadIdx.x, hi4 = t >> 4, lo4 = t & 15;
#pragma unroll 1
    for (uint32_t row = blockIdx.x / CL; row < rows; row += gridDim.x / CL) {
        const uint32_t limb = row % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q, q2 = lc.q2;
        const uint32_t* in = a.in + ((size_t)row << LOGN);
        uint32_t* out = a.out + ((size_t)row << LOGN);
        const uint32_t* mats = wa.mat + ((size_t)limb * 4 + (FWD ? 0 : 2)) * 256;
        for (int i = t; i < 512; i += V8_T) Mst[i] = mats[i];
        const uint2* T1 = wa.t1 + (size_t)limb * 256;
        const uint2* T2 = wa.t2 + (size_t)limb * 4096;
        const uint2* T3 = wa.t3 + (size_t)limb * 65536;
        __syncthreads();
        if constexpr (FWD) {
#pragma unroll 1
            for (int pass = p0; pass < p0 + NP; ++pass) {          // stage 0 on columns: y = M0 x
                const int c = pass * V8_T + t;
                uint32_t x[16];
#pragma unroll
                for (int k = 0; k < 16; ++k) x[k] = __ldcs(in + k * V8_SUBW + c);
                wdc_gemm16(x, Mst, lc);
#pragma unroll
                for (int k = 0; k < 16; ++k) out[k * V8_SUBW + c] = x[k];
            }
            cluster_sync();
            v8_load_fwd_slice(smem, out + s0 * V8_SUBW);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                cp_async_wait<0>();
                __syncwarp();
                uint32_t x[16];
                {   // stage 1, group s
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    wdc_twist(x, T1 + s * 16, q);
                    wdc_gemm16(x, Mst + 256, lc);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(i, b, c)] = x[i];
                }
                __syncthreads();
                if (s + 1 < s1) v8_load_fwd_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, out + (s + 1) * V8_SUBW);
                {   // stage 2, group s * 16 + aa
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    wdc_twist(x, T2 + (s * 16 + aa) * 16, q);
                    wdc_gemm16(x, Mst + 256, lc);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                }
                __syncwarp();
                {   // stage 3, group s * 256 + t
                    const int aa = hi4, b = lo4;
                    const uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    wdc_twist(x, T3 + ((size_t)s * 256 + t) * 16, q);
                    wdc_gemm16(x, Mst + 256, lc);
                    v8_store_sub(S, aa, b, x, out + s * V8_SUBW, [&](uint32_t y) { return wdc_canon(y, q, q2); });
                }
            }
        } else {
            v8_load_inv_slice(smem, in + s0 * V8_SUBW);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                cp_async_wait<0>();
                __syncwarp();
                uint32_t x[16];
                {   // stage 3', group s * 256 + t: y = F' x, then sigma
                    const int aa = hi4, b = lo4;
                    uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    wdc_gemm16(x, Mst + 256, lc);
                    wdc_twist(x, T3 + ((size_t)s * 256 + t) * 16, q);
#pragma unroll
                    for (int v = 0; v < 4; ++v)
                        *reinterpret_cast<uint4*>(base + ((v ^ sw) << 2)) =
                            make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
                }
                __syncwarp();
                {   // stage 2', group s * 16 + aa
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    wdc_gemm16(x, Mst + 256, lc);
                    wdc_twist(x, T2 + (s * 16 + aa) * 16, q);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                }
                __syncthreads();
                if (s + 1 < s1) v8_load_inv_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, in + (s + 1) * V8_SUBW);
                {   // stage 1', group s
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    wdc_gemm16(x, Mst + 256, lc);
                    wdc_twist(x, T1 + s * 16, q);
                    uint32_t* o = out + s * V8_SUBW + b * 16 + c;
#pragma unroll
                    for (int i = 0; i < 16; ++i) o[i * 256] = x[i];
                }
            }
            cluster_sync();
#pragma unroll 1
            for (int pass = p0; pass < p0 + NP; ++pass) {          // stage 0' on columns: y = MI0 x
                const int c = pass * V8_T + t;
                uint32_t x[16];
#pragma unroll
                for (int k = 0; k < 16; ++k) x[k] = out[k * V8_SUBW + c];
                wdc_gemm16(x, Mst, lc);
#pragma unroll
                for (int k = 0; k < 16; ++k) __stcs(out + k * V8_SUBW + c, wdc_canon(x[k], q, q2));
            }
        }
        __syncthreads();
    }
}


// ---------------------------------------------------------------------------------------------
// v11 (N = 2^16): v8's data movement with the ROW-phase radix-16 stages on the tensor cores.
// Within a 4096-word sub-row s (elements a*256 + b*16 + c) the three stages are
//   stage 1 (layers 4..7,  group s):            folded matrix M1_s (twist inside, no extra work)
//   stage 2 (layers 8..11, group s*16 + a):      M = F diag(tau2_g)  -> Shoup twist, then fixed F
//   stage 3 (layers 12..15, group s*256 + a*16 + b): M = F diag(tau3_g)
// (inverse: MI1_s, and F' followed by the sigma twist), i.e. the tensor tables' factorisation,
// over 256 instances = 2 MMA tiles of 128 per stage.  TMASK selects which of the three stages run
// on the tensor cores (bit st-1); the others keep v8's butterflies, and the column phase (layers
// 0..3) is always v8's register-only butterflies, so the tensor pipe of one CTA's row phase
// overlaps the CUDA-core butterflies of the other CTAs on the SM.  Per
// tile: every warp moves 32 instances x 8 coefficients smem -> registers (conflict-free in v8's
// layout) -> TMEM (tcgen05.st), one thread issues 2 MMAs, every warp reads back its 8 outputs x
// 4 planes (tcgen05.ld), recombines and writes them in place (or to global, forward stage 3).
constexpr int V11_SMEM = V8_SMEM + 3 * 4096 + 64;    // sub-rows, B: F/F' + 2 x M1_s/MI1_s, mbarrier

struct V11Args {
    NttArgs a;
    const uint8_t* G;        // [L][2][17][4096] byte planes: [0] M0/MI0, [1+g] M1_g/MI1_g
    const uint8_t* B;        // [L][4][4096]: M0, F, MI0, F'
    const uint2 *t2, *t3;    // twists of this direction (tau forward / sigma inverse), stages 2, 3
    const uint2* c16;
};

template <bool FWD, int ST>
__device__ __forceinline__ void v11_stage(uint32_t* S, uint32_t* gout, uint32_t tmem, uint32_t bimg,
                                          uint64_t* bar, uint32_t& ph, const uint2* __restrict__ tws,
                                          uint32_t q, uint32_t q2, uint32_t c16s, uint32_t one_s) {
    const int t = threadIdx.x, w = t >> 5, lane = t & 31;
    const int lq = w & 3, h = w >> 2;
    const uint32_t tl = tmem + ((uint32_t)(32 * lq) << 16);
#pragma unroll 1
    for (int tt = 0; tt < 2; ++tt) {
        const int i = tt * 128 + lq * 32 + lane;          // instance (u, v) = (i >> 4, i & 15)
        const int u = i >> 4, v = i & 15;
        uint32_t x[8];
        if constexpr (ST == 1) {
#pragma unroll
            for (int jj = 0; jj < 8; ++jj) x[jj] = S[v8_phys(8 * h + jj, u, v)];
        } else if constexpr (ST == 2) {
#pragma unroll
            for (int jj = 0; jj < 8; ++jj) x[jj] = S[v8_phys(u, 8 * h + jj, v)];
        } else {
            const uint32_t* base = S + u * 256 + ((v ^ (u & 1)) << 4);
            const int sw = (v >> 1) & 3;
#pragma unroll
            for (int vv = 0; vv < 2; ++vv) {
                const uint4 g = *reinterpret_cast<const uint4*>(base + (((2 * h + vv) ^ sw) << 2));
                x[4 * vv] = g.x; x[4 * vv + 1] = g.y; x[4 * vv + 2] = g.z; x[4 * vv + 3] = g.w;
            }
        }
        if constexpr (FWD && ST >= 2) {                    // x_j <- x_j * tau_g[j]
            const uint4* tp = reinterpret_cast<const uint4*>(tws + (size_t)(ST == 2 ? u : i) * 16 + 8 * h);
#pragma unroll
            for (int jj = 0; jj < 8; jj += 2) {
                const uint4 tw = __ldg(tp + jj / 2);
                x[jj] = shoup_mul(x[jj], tw.x, tw.y, q);
                x[jj + 1] = shoup_mul(x[jj + 1], tw.z, tw.w, q);
            }
        }
        tmem_st8(tl + 8 * h, x);
        tmem_wait_st();
        tc_fence_before();
        __syncthreads();                                   // A complete; previous tile's D read
        if (t == 0) {
            tc_fence_after();
            tc_mma_ts(tmem + 64, tmem, umma_desc(bimg), 0);
            tc_mma_ts(tmem + 64, tmem + 8, umma_desc(bimg + 256), 1);
            tc_commit(bar);
        }
        uint4 sg[4];
        if constexpr (!FWD && ST >= 2) {                   // sigma_g[k], k = 8h .. 8h+7, in flight
            const uint4* sp = reinterpret_cast<const uint4*>(tws + (size_t)(ST == 2 ? u : i) * 16 + 8 * h);
#pragma unroll
            for (int k2 = 0; k2 < 4; ++k2) sg[k2] = __ldg(sp + k2);
        }
        mbar_wait(bar, ph);
        ph ^= 1;
        tc_fence_after();
        uint32_t d[32];
        tmem_ld32(tl + 64 + 32 * h, d);
        tmem_wait_ld();
        tc_fence_before();
        uint32_t y[8];
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
            y[kk] = v10_combine(d + 4 * kk, q, q2, c16s, one_s);        // [0, 4q)
            if constexpr (!FWD && ST >= 2)
                y[kk] = shoup_mul(y[kk], (kk & 1) ? sg[kk / 2].z : sg[kk / 2].x, (kk & 1) ? sg[kk / 2].w : sg[kk / 2].y, q);
            if constexpr (!FWD && ST == 1) y[kk] = umin32(y[kk], y[kk] - q2);   // GS column phase wants [0, 2q)
        }
        if constexpr (ST == 1) {
#pragma unroll
            for (int kk = 0; kk < 8; ++kk) S[v8_phys(8 * h + kk, u, v)] = y[kk];
        } else if constexpr (ST == 2) {
#pragma unroll
            for (int kk = 0; kk < 8; ++kk) S[v8_phys(u, 8 * h + kk, v)] = y[kk];
        } else if (FWD) {
            uint4* o = reinterpret_cast<uint4*>(gout + i * 16 + 8 * h);
#pragma unroll
            for (int vv = 0; vv < 2; ++vv)
                __stcs(o + vv, make_uint4(canon4(y[4 * vv], q, q2), canon4(y[4 * vv + 1], q, q2),
                                          canon4(y[4 * vv + 2], q, q2), canon4(y[4 * vv + 3], q, q2)));
        } else {
            uint32_t* base = S + u * 256 + ((v ^ (u & 1)) << 4);
            const int sw = (v >> 1) & 3;
#pragma unroll
            for (int vv = 0; vv < 2; ++vv)
                *reinterpret_cast<uint4*>(base + (((2 * h + vv) ^ sw) << 2)) =
                    make_uint4(y[4 * vv], y[4 * vv + 1], y[4 * vv + 2], y[4 * vv + 3]);
        }
    }
    __syncthreads();                                       // the stage's results visible to every warp
}

template <bool FWD, int TMASK, int CL = 2>
__global__ void __launch_bounds__(V8_T, 4) ntt_v11(V11Args va, uint32_t rows) {
    constexpr int LOGN = 16, A = 4;
    constexpr int NP = V8_SUBW / V8_T / CL, NS = 16 / CL;
    constexpr bool T1 = TMASK & 1, T2 = TMASK & 2, T3 = TMASK & 4;
    const NttArgs& a = va.a;
    const int rank = CL > 1 ? (int)(blockIdx.x % CL) : 0;
    const int p0 = rank * NP, s0 = rank * NS, s1 = s0 + NS;
    extern __shared__ __align__(1024) uint32_t smem_v11[];
    uint32_t* const smem = smem_v11;
    uint8_t* Bf = reinterpret_cast<uint8_t*>(smem + 2 * V8_SUBW);       // F / F'
    uint8_t* B1 = Bf + 4096;                                            // [2] M1_s / MI1_s
    uint64_t* bar = reinterpret_cast<uint64_t*>(Bf + 3 * 4096);
    uint32_t* tslot = reinterpret_cast<uint32_t*>(bar + 1);
    const int t = threadIdx.x, hi4 = t >> 4, lo4 = t & 15;
    if (t == 0) {
        mbar_init(bar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (t < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" :: "r"(smem_addr(tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tslot;
    uint32_t ph = 0;
#pragma unroll 1
    for (uint32_t row = blockIdx.x / CL; row < rows; row += gridDim.x / CL) {
        const uint32_t limb = row % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q, q2 = lc.q2;
        const uint2 cc = va.c16[limb];
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        const uint32_t* in = a.in + ((size_t)row << LOGN);
        uint32_t* out = a.out + ((size_t)row << LOGN);
        const uint8_t* Gl = va.G + ((size_t)limb * 2 + (FWD ? 0 : 1)) * 17 * 4096;
        const uint2* tw2 = va.t2 + (size_t)limb * 4096;
        const uint2* tw3 = va.t3 + (size_t)limb * 65536;
        if constexpr (TMASK != 0) {                                       // F / F' of this limb
            cp_async16(Bf + 16 * t, va.B + ((size_t)limb * 4 + (FWD ? 1 : 3)) * 4096 + 16 * t);
            cp_async_commit();
        }
        auto load_b1 = [&](int s) {                                      // M1_s / MI1_s
            if constexpr (T1) {
                cp_async16(B1 + ((s - s0) & 1) * 4096 + 16 * t, Gl + (1 + s) * 4096 + 16 * t);
                cp_async_commit();
            }
        };
        if constexpr (FWD) {
#pragma unroll 1
            for (int pass = p0; pass < p0 + NP; ++pass) {                   // phase 1 (v8)
                const int c = pass * V8_T + t;
                uint32_t x[16];
#pragma unroll
                for (int k = 0; k < 16; ++k) x[k] = __ldcs(in + k * V8_SUBW + c);
                fwd_radix<A>(x, tw, 0, 0, q, q2);
#pragma unroll
                for (int k = 0; k < 16; ++k) out[k * V8_SUBW + c] = x[k];
            }
            if constexpr (CL > 1) cluster_sync(); else __syncthreads();
            v8_load_fwd_slice(smem, out + s0 * V8_SUBW);
            load_b1(s0);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                cp_async_wait<0>();
                if constexpr (TMASK != 0) fence_async_smem();
                if constexpr (T1) __syncthreads(); else __syncwarp();
                uint32_t x[16];
                if constexpr (T1) {
                    v11_stage<true, 1>(S, nullptr, tmem, smem_addr(B1 + ((s - s0) & 1) * 4096), bar, ph, nullptr,
                                       q, q2, cc.x, cc.y);
                } else {
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    fwd_radix<4>(x, tw, A, (uint32_t)s, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(i, b, c)] = x[i];
                    __syncthreads();
                }
                if (s + 1 < s1) {
                    v8_load_fwd_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, out + (s + 1) * V8_SUBW);
                    load_b1(s + 1);
                }
                if constexpr (T2) {
                    v11_stage<true, 2>(S, nullptr, tmem, smem_addr(Bf), bar, ph, tw2 + (size_t)s * 16 * 16,
                                       q, q2, cc.x, cc.y);
                } else {
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    fwd_radix<4>(x, tw, A + 4, (uint32_t)s * 16 + aa, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                    if constexpr (T3) __syncthreads(); else __syncwarp();
                }
                if constexpr (T3) {
                    v11_stage<true, 3>(S, out + s * V8_SUBW, tmem, smem_addr(Bf), bar, ph, tw3 + (size_t)s * 256 * 16,
                                       q, q2, cc.x, cc.y);
                } else {
                    uint2 w3[15];
                    load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                    const int aa = hi4, b = lo4;
                    const uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    fwd16_tw(x, w3, q, q2);
                    v8_store_sub(S, aa, b, x, out + s * V8_SUBW, [&](uint32_t y) { return canon4(y, q, q2); });
                }
            }
        } else {
            v8_load_inv_slice(smem, in + s0 * V8_SUBW);
            load_b1(s0);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                cp_async_wait<0>();
                if constexpr (TMASK != 0) fence_async_smem();
                if constexpr (T3) __syncthreads(); else __syncwarp();
                uint32_t x[16];
                if constexpr (T3) {
                    v11_stage<false, 3>(S, nullptr, tmem, smem_addr(Bf), bar, ph, tw3 + (size_t)s * 256 * 16,
                                        q, q2, cc.x, cc.y);
                } else {
                    uint2 w3[15];
                    load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
                    const int aa = hi4, b = lo4;
                    uint32_t* base = S + aa * 256 + ((b ^ (aa & 1)) << 4);
                    const int sw = (b >> 1) & 3;
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        const uint4 u = *reinterpret_cast<const uint4*>(base + ((v ^ sw) << 2));
                        x[4 * v] = u.x; x[4 * v + 1] = u.y; x[4 * v + 2] = u.z; x[4 * v + 3] = u.w;
                    }
                    inv16_tw(x, w3, q, q2);
#pragma unroll
                    for (int v = 0; v < 4; ++v)
                        *reinterpret_cast<uint4*>(base + ((v ^ sw) << 2)) =
                            make_uint4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
                    if constexpr (T2) __syncthreads(); else __syncwarp();
                }
                if constexpr (T2) {
                    v11_stage<false, 2>(S, nullptr, tmem, smem_addr(Bf), bar, ph, tw2 + (size_t)s * 16 * 16,
                                        q, q2, cc.x, cc.y);
                } else {
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    inv_radix<4, false>(x, tw, A + 4, (uint32_t)s * 16 + aa, lc);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                    __syncthreads();
                }
                if (s + 1 < s1) {
                    v8_load_inv_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, in + (s + 1) * V8_SUBW);
                    load_b1(s + 1);
                }
                if constexpr (T1) {
                    // MI1_s of THIS sub-row: its group was committed with sub-row s (waited above)
                    v11_stage<false, 1>(S, nullptr, tmem, smem_addr(B1 + ((s - s0) & 1) * 4096), bar, ph, nullptr,
                                        q, q2, cc.x, cc.y);
                    const int b = hi4, c = lo4;
                    uint32_t* o = out + s * V8_SUBW + b * 16 + c;
#pragma unroll
                    for (int i = 0; i < 16; ++i) o[i * 256] = S[v8_phys(i, b, c)];
                } else {
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    inv_radix<4, false>(x, tw, A, (uint32_t)s, lc);
                    uint32_t* o = out + s * V8_SUBW + b * 16 + c;
#pragma unroll
                    for (int i = 0; i < 16; ++i) o[i * 256] = x[i];
                }
            }
            if constexpr (CL > 1) cluster_sync(); else __syncthreads();
#pragma unroll 1
            for (int pass = p0; pass < p0 + NP; ++pass) {                   // phase 1' (v8)
                const int c = pass * V8_T + t;
                uint32_t x[16];
#pragma unroll
                for (int k = 0; k < 16; ++k) x[k] = out[k * V8_SUBW + c];
                inv_radix<A, true>(x, tw, 0, 0, lc);
#pragma unroll
                for (int k = 0; k < 16; ++k) __stcs(out + k * V8_SUBW + c, canon2(x[k], q));
            }
        }
        __syncthreads();
    }
    cp_async_wait<0>();
    tc_fence_before();
    __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" :: "r"(tmem));
}

}  // namespace wd
