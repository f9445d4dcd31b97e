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
#include "common.cuh"
#include "ntt_cuda_core.cuh"
#include "tma.cuh"

// the v8 kernels declare their dynamic shared memory 1024-byte aligned (TMA destinations); the
// kernels of ntt_cuda_core.cuh declare the same extern array with 16 (same storage, harmless)
#pragma nv_diag_suppress 1886

namespace wd {

constexpr int V8_T = 256;                    // threads per CTA (4 CTAs per SM at 64 registers)
constexpr int V8_SUBW = 4096;                // words per phase-2 sub-row
constexpr int V8_SMEM = 2 * V8_SUBW * 4;     // two sub-row buffers = 32 KB
// The radix-16 twiddles of row stages 1 and 2 (1 + 16 groups x 15 per sub-row) are staged in shared
// memory by cp.async together with the sub-row they belong to (one sub-row ahead), instead of being
// __ldg'd right before use: with the 228 KB carveout L1 is small and those loads were L2 round trips
// on the critical path (config 3: forward 1.097 -> 1.062 ms, inverse 1.086 -> 1.037 ms)
constexpr int V8_TWW = 768;                  // words per buffer's twiddle area (<= 384 pairs)
constexpr int V8_TWOFF = 2 * V8_SUBW + 16;   // its word offset: after the buffers and the mbarriers
// the v8 kernel's dynamic shared memory: two sub-row buffers, the TMA column phase's mbarriers (64 B)
// and two twiddle areas
constexpr int V8_SMEM_K = V8_SMEM + 64 + 2 * V8_TWW * 4;

__device__ __forceinline__ void cp_async8(void* smem_dst, const void* gsrc) {
    const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem_dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" :: "r"(d), "l"(gsrc) : "memory");
}
// forward, sub-row s: every warp copies the stage-1 runs (group s, layers A..A+3: 1, 2, 4, 8 pairs at
// 0, 2, 4, 8) into its own 16 pairs at TW + 16w (read before the CTA barrier, after the warp's own
// cp.async wait), and threads 0..239 copy the stage-2 runs (groups 16s..16s+15, layers A+4..A+7:
// 16, 32, 64, 128 pairs at 128 + 0, 16, 48, 112; read after the barrier).  No commit (the caller's
// slice load commits the group).
template <int A>
__device__ __forceinline__ void v8_tw_fwd(uint2* TW, const uint2* __restrict__ tw, uint32_t s) {
    const int t = threadIdx.x, w = t >> 5, l = t & 31;
    if (l < 15) {
        const int k = 31 - __clz(l + 1), g = l - ((1 << k) - 1);
        cp_async8(TW + 16 * w + (k ? (1 << k) : 0) + g, tw + (1u << (A + k)) + (s << k) + g);
    }
    if (t < 240) {
        const int k = 31 - __clz((t >> 4) + 1), g = t - 16 * ((1 << k) - 1);
        cp_async8(TW + 128 + 16 * ((1 << k) - 1) + g, tw + (16u << (A + k)) + ((s * 16) << k) + g);
    }
}
// inverse, sub-row s: every warp copies the stage-2' runs of its two groups 16s + 2w, 16s + 2w + 1
// (2, 4, 8, 16 pairs at TW + 32w + 0, 2, 6, 14; read before the barrier), threads 0..14 the stage-1'
// runs of group s (at 256 + 0, 2, 4, 8; read after it)
template <int A>
__device__ __forceinline__ void v8_tw_inv(uint2* TW, const uint2* __restrict__ tw, uint32_t s) {
    const int t = threadIdx.x, w = t >> 5, l = t & 31;
    if (l < 30) {
        const int k = 31 - __clz((l >> 1) + 1), g = l - 2 * ((1 << k) - 1);
        cp_async8(TW + 32 * w + 2 * ((1 << k) - 1) + g, tw + (16u << (A + k)) + ((s * 16 + 2 * w) << k) + g);
    }
    if (t < 15) {
        const int k = 31 - __clz(t + 1), g = t - ((1 << k) - 1);
        cp_async8(TW + 256 + (k ? (1 << k) : 0) + g, tw + (1u << (A + k)) + (s << k) + g);
    }
}
__device__ __forceinline__ uint2 lo2(uint4 v) { return make_uint2(v.x, v.y); }
__device__ __forceinline__ uint2 hi2(uint4 v) { return make_uint2(v.z, v.w); }
// radix-16 blocks whose layer-t twiddle of group g is p_t[g] (shared memory; p1..p3 16-byte aligned),
// the same butterfly network as fwd16_tw / inv16_tw
__device__ __forceinline__ void fwd16_sp(uint32_t* x, const uint2* p0, const uint2* p1, const uint2* p2,
                                         const uint2* p3, uint32_t q, uint32_t q2) {
    {
        const uint2 w = *p0;
#pragma unroll
        for (int r = 0; r < 8; ++r) ct_bfly(x[r], x[r + 8], w, q, q2);
    }
    {
        const uint4 v = *reinterpret_cast<const uint4*>(p1);
#pragma unroll
        for (int r = 0; r < 4; ++r) { ct_bfly(x[r], x[r + 4], lo2(v), q, q2); ct_bfly(x[8 + r], x[12 + r], hi2(v), q, q2); }
    }
#pragma unroll
    for (int k = 0; k < 2; ++k) {
        const uint4 v = reinterpret_cast<const uint4*>(p2)[k];
#pragma unroll
        for (int r = 0; r < 2; ++r) {
            ct_bfly(x[8 * k + r], x[8 * k + r + 2], lo2(v), q, q2);
            ct_bfly(x[8 * k + 4 + r], x[8 * k + 6 + r], hi2(v), q, q2);
        }
    }
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const uint4 v = reinterpret_cast<const uint4*>(p3)[k];
        ct_bfly(x[4 * k], x[4 * k + 1], lo2(v), q, q2);
        ct_bfly(x[4 * k + 2], x[4 * k + 3], hi2(v), q, q2);
    }
}
template <bool LAST>
__device__ __forceinline__ void inv16_sp(uint32_t* x, const uint2* p0, const uint2* p1, const uint2* p2,
                                         const uint2* p3, const LimbConst& c) {
    const uint32_t q = c.q, q2 = c.q2;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const uint4 v = reinterpret_cast<const uint4*>(p3)[k];
        gs_bfly(x[4 * k], x[4 * k + 1], lo2(v), q, q2);
        gs_bfly(x[4 * k + 2], x[4 * k + 3], hi2(v), q, q2);
    }
#pragma unroll
    for (int k = 0; k < 2; ++k) {
        const uint4 v = reinterpret_cast<const uint4*>(p2)[k];
#pragma unroll
        for (int r = 0; r < 2; ++r) {
            gs_bfly(x[8 * k + r], x[8 * k + r + 2], lo2(v), q, q2);
            gs_bfly(x[8 * k + 4 + r], x[8 * k + 6 + r], hi2(v), q, q2);
        }
    }
    {
        const uint4 v = *reinterpret_cast<const uint4*>(p1);
#pragma unroll
        for (int r = 0; r < 4; ++r) { gs_bfly(x[r], x[r + 4], lo2(v), q, q2); gs_bfly(x[8 + r], x[12 + r], hi2(v), q, q2); }
    }
    if constexpr (LAST) {
#pragma unroll
        for (int r = 0; r < 8; ++r) gs_bfly_last(x[r], x[r + 8], c);
    } else {
        const uint2 w = *p0;
#pragma unroll
        for (int r = 0; r < 8; ++r) gs_bfly(x[r], x[r + 8], w, q, q2);
    }
}

__device__ __forceinline__ int v8_phys(int a, int b, int c) {
    return a * 256 + ((b ^ (a & 1)) << 4) + (c ^ (((b >> 1) & 3) << 2));
}

// Per-warp slices: in phase 2 each warp cp.asyncs exactly the words its own FIRST stage reads,
// so the first stage needs only the warp's own wait + __syncwarp, and the stage pair that stays
// inside a half-warp (forward 2->3, inverse 3'->2') needs only __syncwarp: one CTA barrier per
// sub-row instead of three.
// forward (stage 1, thread (b,c) loops a): warp w reads words a*256 + 32w .. +31, a = 0..15
__device__ __forceinline__ void v8_load_fwd_slice(uint32_t* S, const uint32_t* src) {
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const int a = 4 * k + (l >> 3), g = l & 7;           // 128-byte segment a, granule g
        cp_async16(S + v8_phys(a, 2 * w + (g >> 2), (g & 3) << 2), src + a * 256 + 32 * w + 4 * g);
    }
    cp_async_commit();
}
// inverse (stage 3', thread (a,b) reads 16 contiguous c): warp w reads words 512w .. 512w + 511
__device__ __forceinline__ void v8_load_inv_slice(uint32_t* S, const uint32_t* src) {
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const int e = 512 * w + 4 * (32 * k + l);
        cp_async16(S + v8_phys(e >> 8, (e >> 4) & 15, e & 15), src + e);
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
// TM (EPI = 0, no pointwise product, 2 <= 2^A <= 16): the column phase is fed by TMA instead of
// register loads.  Each column pass (256 columns x 2^A lines = 2^A KB, one 2-D box of tm_in) lands in
// one of the two sub-row buffers and the next pass is in flight while a pass computes; threads read
// their column with conflict-free LDS.  Forward: tm_in maps the input, and the first pass of the CTA's
// next row is issued during the last sub-row of the current one, so the HBM latency of the column
// loads is no longer exposed.  Inverse: tm_in maps the output slot (the L2-resident intermediate,
// made visible to the async proxy by fence.proxy.async.global before the cluster barrier), and the
// last pass starts the cp.async of the next row's first sub-row.
template <int LOGN, bool FWD, bool PW, int CL = 1, int EPI = 0, int TM = 0>
__global__ void __launch_bounds__(V8_T, 4) ntt_v8(NttArgs a, uint32_t rows, const __grid_constant__ CUtensorMap tm_in) {
    constexpr int A = LOGN - 12;             // phase-1 layers (radix 2^A columns)
    constexpr int R = 1 << A;                // column length = number of sub-rows
    static_assert(A >= 0 && A <= 5, "N = 2^12 .. 2^17");
    static_assert(R % CL == 0 && (V8_SUBW / V8_T) % CL == 0, "cluster splits passes and sub-rows evenly");
    constexpr int NP = V8_SUBW / V8_T / CL;  // phase-1 column passes per CTA
    constexpr int NS = R / CL;               // phase-2 sub-rows per CTA
    const int rank = CL > 1 ? (int)(blockIdx.x % CL) : 0;
    const int p0 = rank * NP, s0 = rank * NS, s1 = s0 + NS;
    extern __shared__ __align__(1024) uint32_t smem[];
    const int t = threadIdx.x;
    const int hi4 = t >> 4, lo4 = t & 15;

    const uint32_t nb = a.nb_total ? a.nb_total : rows / a.L;   // polynomials of the schedule
    const uint32_t send = a.slot0 + rows;        // the launch covers schedule slots slot0 .. send - 1
    static_assert(TM != 1 || (EPI == 0 && !PW && A >= 1 && R <= 16), "TMA column phase: EPI 0, no PW, 2 <= R <= 16");
    static_assert(TM != 2 || (!FWD && EPI == 0 && A >= 1), "early sub-row prefetch: inverse with a column phase");
    constexpr int PF = ((NS - 1) & 1) ^ 1;       // TM: the buffer free during a row's last sub-row
    // TM: one mbarrier per buffer, after the two buffers (dynamic shared memory V8_SMEM_K; a static
    // __shared__ would shift the dynamic buffers off the alignment TMA needs)
    uint64_t* tbar = reinterpret_cast<uint64_t*>(smem + 2 * V8_SUBW);
    auto TWB = [&](int b) { return reinterpret_cast<uint2*>(smem + V8_TWOFF + b * V8_TWW); };
    uint32_t tph = 0;                            // TM: parity of each buffer's next completion
    auto map_row = [&](uint32_t sr) {            // limb-major schedule (below)
        const uint32_t lb = a.limb_major ? sr / nb : sr % a.L;
        return a.limb_major ? (sr - lb * nb) * a.L + lb : sr;
    };
    if constexpr (TM == 1) {
        if (t == 0) {
            mb_init(&tbar[0], 1); mb_init(&tbar[1], 1);
            mb_init_fence();
            const uint32_t sr = a.slot0 + blockIdx.x / CL;
            if (FWD && sr < send) {              // the CTA's first column pass
                mb_expect(&tbar[PF], R * V8_T * 4);
                tma2_load_hint(smem + PF * V8_SUBW, &tm_in, p0 * V8_T, (int)(row_map(map_row(sr), a.L, a.in_ls) * R), &tbar[PF],
                               l2_evict_first_policy());
            }
        }
        __syncthreads();
    }
    bool sub0_ready = false;                     // TM inverse: this row's first sub-row already requested
#pragma unroll 1
    for (uint32_t srow = a.slot0 + blockIdx.x / CL; srow < send; srow += gridDim.x / CL) {
        // limb-major schedule (a.limb_major): the rows in flight at any time share a few limbs,
        // so their twiddle tables (N x 8 bytes per limb and direction) stay a small part of L2
        // next to the L2-resident intermediates; the data layout is unchanged
        const uint32_t limb = a.limb_major ? srow / nb : srow % a.L;
        const uint32_t row = map_row(srow);
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
            if constexpr (A > 0) {
#pragma unroll 1
                for (int pass = p0; pass < p0 + NP; ++pass) {
                    const int c = pass * V8_T + t;
                    uint32_t x[R];
                    if constexpr (TM == 1) {
                        const int b = (pass - p0 + PF) & 1;
                        if (t == 0 && pass + 1 < p0 + NP) {   // the next pass into the other buffer
                            fence_proxy_async();
                            mb_expect(&tbar[b ^ 1], R * V8_T * 4);
                            tma2_load_hint(smem + (b ^ 1) * V8_SUBW, &tm_in, (pass + 1) * V8_T,
                                           (int)(row_map(row, a.L, a.in_ls) * R), &tbar[b ^ 1], l2_evict_first_policy());
                        }
                        mb_wait(&tbar[b], (tph >> b) & 1);
                        tph ^= 1u << b;
                        const uint32_t* B = smem + b * V8_SUBW;
#pragma unroll
                        for (int k = 0; k < R; ++k) x[k] = B[k * V8_T + t];
                        __syncthreads();                      // buffer b read by every thread
                    } else {
#pragma unroll
                        for (int k = 0; k < R; ++k) {
                            if constexpr (EPI == 1) x[k] = rs_in(__ldg(in + k * V8_SUBW + c), a.rs_thr, rsc, q);
                            else x[k] = __ldcs(in + k * V8_SUBW + c);
                        }
                    }
                    fwd_radix<A>(x, tw, 0, 0, q, q2);
#pragma unroll
                    for (int k = 0; k < R; ++k) out[k * V8_SUBW + c] = x[k];
                }
                if constexpr (CL > 1) cluster_sync();    // the whole intermediate is written
                else __syncthreads();
            }
            // ---- phase 2: layers A..A+11 on sub-rows s ----
            const uint32_t* src = A > 0 ? out : in;
            v8_tw_fwd<A>(TWB(0), tw, s0);
            v8_load_fwd_slice(smem, src + s0 * V8_SUBW);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                cp_async_wait<0>();
                __syncwarp();                            // this warp's stage-1 slice of sub-row s landed
                const uint32_t st = (uint32_t)s;
                uint32_t x[16];
                {   // stage 1: layers A..A+3, thread (b, c), elements a (stride 256)
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) {
                        x[i] = S[v8_phys(i, b, c)];
                        if constexpr (EPI == 1 && A == 0) x[i] = rs_in(x[i], a.rs_thr, rsc, q);
                    }
                    const uint2* W = TWB((s - s0) & 1) + 16 * (t >> 5);
                    fwd16_sp(x, W, W + 2, W + 4, W + 8, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(i, b, c)] = x[i];
                }
                __syncthreads();                         // stage 1 done everywhere; sub-row s-1 fully consumed
                if (s + 1 < s1) {
                    v8_tw_fwd<A>(TWB((s + 1 - s0) & 1), tw, s + 1);
                    v8_load_fwd_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, src + (s + 1) * V8_SUBW);
                } else if constexpr (TM == 1) {               // the next row's first column pass
                    const uint32_t sr = srow + gridDim.x / CL;
                    if (t == 0 && sr < send) {
                        fence_proxy_async();
                        mb_expect(&tbar[PF], R * V8_T * 4);
                        tma2_load_hint(smem + PF * V8_SUBW, &tm_in, p0 * V8_T, (int)(row_map(map_row(sr), a.L, a.in_ls) * R),
                                       &tbar[PF], l2_evict_first_policy());
                    }
                }
                uint2 w3[15];
                load_tw16(w3, tw, A + 8, st * 256 + t);  // stage-3 twiddles, in flight
                {   // stage 2: layers A+4..A+7, thread (a, c), elements b (stride 16)
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    const uint2* T2 = TWB((s - s0) & 1) + 128;
                    fwd16_sp(x, T2 + aa, T2 + 16 + 2 * aa, T2 + 48 + 4 * aa, T2 + 112 + 8 * aa, q, q2);
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
                    fwd16_tw(x, w3, q, q2);
                    // Coalesced store through the warp's own 2 KB of S: stage 3 of warp w covers
                    // words 512w .. 512w+511 of the sub-row, so after writing them back (the same
                    // conflict-free 16-byte slots it read) each lane re-reads granules 128v + 4*lane
                    // and every STG.128 of the warp writes 512 contiguous bytes (the direct
                    // per-thread 64-byte stores cost 4x the L1 wavefronts: DESIGN.md 5.1).
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
                }
            }
        } else {
            // ---- phase 2': layers A+11..A on sub-rows s (input in bit-reversed order) ----
            const uint32_t* in2 = a.in2 + ((size_t)row << LOGN);
            if (!sub0_ready) {
                v8_tw_inv<A>(TWB(0), tw, s0);
                v8_load_inv_slice(smem, in + s0 * V8_SUBW);
            }
            sub0_ready = false;
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                uint2 w3[15];
                load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);   // in flight across the wait
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
                    inv16_tw(x, w3, q, q2);
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
                    const uint2* W = TWB((s - s0) & 1) + 32 * (t >> 5) + (aa & 1);
                    inv16_sp<false>(x, W, W + 2 + (aa & 1), W + 6 + 3 * (aa & 1), W + 14 + 7 * (aa & 1), lc);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
                }
                __syncthreads();                         // stage 2' done everywhere; sub-row s-1 fully consumed
                if (s + 1 < s1) {
                    v8_tw_inv<A>(TWB((s + 1 - s0) & 1), tw, s + 1);
                    v8_load_inv_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, in + (s + 1) * V8_SUBW);
                }
                {   // stage 1': layers A+3..A, thread (b, c), elements a -> global (coalesced)
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    const uint2* T1 = TWB((s - s0) & 1) + 256;
                    inv16_sp<A == 0>(x, T1, T1 + 2, T1 + 4, T1 + 8, lcl);
                    uint32_t* o = out + s * V8_SUBW + b * 16 + c;
#pragma unroll
                    for (int i = 0; i < 16; ++i) {
                        if constexpr (A == 0) __stcs(o + i * 256, canon2(x[i], q));
                        else o[i * 256] = x[i];             // lazy intermediate, in [0,2q)
                    }
                }
            }
            // ---- phase 1': layers A-1..0 on columns, N^-1 folded into layer 0 ----
            if constexpr (A > 0) {
                if constexpr (TM == 1) fence_proxy_async_global();   // the intermediate is read back by TMA
                if constexpr (CL > 1) cluster_sync();    // the whole intermediate is written
                else __syncthreads();
                const int orow = (int)(row_map(row, a.L, a.out_ls) * R);
                if constexpr (TM == 2) {                 // the register-fed column phase leaves both buffers
                    const uint32_t sr = srow + gridDim.x / CL;     // idle: next row's first sub-row now
                    if (sr < send) {
                        const uint32_t nl = a.limb_major ? sr / nb : sr % a.L;
                        v8_tw_inv<A>(TWB(0), a.tw + ((size_t)nl << LOGN), s0);
                        v8_load_inv_slice(smem, a.in + ((size_t)row_map(map_row(sr), a.L, a.in_ls) << LOGN) + s0 * V8_SUBW);
                        sub0_ready = true;
                    }
                }
                if constexpr (TM == 1) {
                    if (t == 0) {
                        mb_expect(&tbar[0], R * V8_T * 4);
                        tma2_load_hint(smem, &tm_in, p0 * V8_T, orow, &tbar[0], l2_evict_first_policy());
                    }
                }
#pragma unroll 1
                for (int pass = p0; pass < p0 + NP; ++pass) {
                    const int c = pass * V8_T + t;
                    uint32_t x[R];
                    if constexpr (TM == 1) {
                        const int b = (pass - p0) & 1;
                        if (t == 0 && pass + 1 < p0 + NP) {   // the next pass into the other buffer
                            fence_proxy_async();
                            mb_expect(&tbar[b ^ 1], R * V8_T * 4);
                            tma2_load_hint(smem + (b ^ 1) * V8_SUBW, &tm_in, (pass + 1) * V8_T, orow, &tbar[b ^ 1], l2_evict_first_policy());
                        }
                        mb_wait(&tbar[b], (tph >> b) & 1);
                        tph ^= 1u << b;
                        const uint32_t* B = smem + b * V8_SUBW;
#pragma unroll
                        for (int k = 0; k < R; ++k) x[k] = B[k * V8_T + t];
                        __syncthreads();                      // buffer b read by every thread
                        static_assert((NP & 1) == 0, "the last pass reads buffer 1: buffer 0 is free");
                        if (pass + 1 == p0 + NP) {            // the next row's first sub-row into buffer 0
                            const uint32_t sr = srow + gridDim.x / CL;
                            if (sr < send) {
                                const uint32_t nl = a.limb_major ? sr / nb : sr % a.L;
                                v8_tw_inv<A>(TWB(0), a.tw + ((size_t)nl << LOGN), s0);
                                v8_load_inv_slice(smem, a.in + ((size_t)row_map(map_row(sr), a.L, a.in_ls) << LOGN) +
                                                            s0 * V8_SUBW);
                                sub0_ready = true;
                            }
                        }
                    } else {
#pragma unroll
                        for (int k = 0; k < R; ++k) x[k] = __ldcs(out + k * V8_SUBW + c);
                    }
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


}  // namespace wd
