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

namespace wd {

constexpr int V8_T = 256;                    // threads per CTA (4 CTAs per SM at 64 registers)
constexpr int V8_SUBW = 4096;                // words per phase-2 sub-row
constexpr int V8_SMEM = 2 * V8_SUBW * 4;     // two sub-row buffers = 32 KB

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

// cp.async one 4096-word sub-row (contiguous in global) into the swizzled layout
__device__ __forceinline__ void v8_load_sub(uint32_t* S, const uint32_t* src) {
#pragma unroll
    for (int k = 0; k < V8_SUBW / 4 / V8_T; ++k) {
        const int G = threadIdx.x + k * V8_T;               // 16-byte granule: words 4G..4G+3
        cp_async16(S + v8_phys(G >> 6, (G >> 2) & 15, (G & 3) << 2), src + 4 * G);
    }
    cp_async_commit();
}

// MINB: resident CTAs per SM the register budget is cut for (4 -> 64 registers; 5, 6 -> 48, 40
// with per-layer just-in-time stage-3 twiddles instead of 15 preloaded pairs).
// ONLY: 1 = phase 1 only, 2 = phase 2 only (timing experiments; results are wrong).
// CL > 1: a cluster of CL CTAs shares each row -- CTA rank r takes column passes and sub-rows
// [r, r+1) * (16|R)/CL, with ONE cluster barrier (release/acquire) between the phases.  Rows
// in flight, hence the L2 footprint of the intermediate, shrink by CL.
template <int LOGN, bool FWD, bool PW, int ONLY = 0, int MINB = 4, int CL = 1>
__global__ void __launch_bounds__(V8_T, MINB) ntt_v8(NttArgs a, uint32_t rows) {
    constexpr bool JIT3 = MINB > 4;
    constexpr int A = LOGN - 12;             // phase-1 layers (radix 2^A columns)
    constexpr int R = 1 << A;                // column length = number of sub-rows
    static_assert(A >= 0 && A <= 5, "N = 2^12 .. 2^17");
    static_assert(R % CL == 0 && (V8_SUBW / V8_T) % CL == 0, "cluster splits passes and sub-rows evenly");
    constexpr int NP = V8_SUBW / V8_T / CL;  // phase-1 column passes per CTA
    constexpr int NS = R / CL;               // phase-2 sub-rows per CTA
    const int rank = CL > 1 ? (int)(blockIdx.x % CL) : 0;
    const int p0 = rank * NP, s0 = rank * NS, s1 = s0 + NS;
    extern __shared__ __align__(16) uint32_t smem[];
    const int t = threadIdx.x;
    const int hi4 = t >> 4, lo4 = t & 15;

#pragma unroll 1
    for (uint32_t row = blockIdx.x / CL; row < rows; row += gridDim.x / CL) {
        const uint32_t limb = row % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q, q2 = lc.q2;
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        const uint32_t* in = a.in + ((size_t)row << LOGN);
        uint32_t* out = a.out + ((size_t)row << LOGN);

        if constexpr (FWD) {
            // ---- phase 1: layers 0..A-1 on columns c (elements c + 4096 k) ----
            if constexpr (A > 0 && ONLY != 2) {
#pragma unroll 1
                for (int pass = p0; pass < p0 + NP; ++pass) {
                    const int c = pass * V8_T + t;
                    uint32_t x[R];
#pragma unroll
                    for (int k = 0; k < R; ++k) x[k] = __ldcs(in + k * V8_SUBW + c);
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
            v8_load_fwd_slice(smem, src + s0 * V8_SUBW);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                uint32_t* S = smem + ((s - s0) & 1) * V8_SUBW;
                cp_async_wait<0>();
                __syncwarp();                            // this warp's stage-1 slice of sub-row s landed
                uint32_t x[16];
                {   // stage 1: layers A..A+3, thread (b, c), elements a (stride 256)
                    const int b = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                    fwd_radix<4>(x, tw, A, (uint32_t)s, q, q2);
#pragma unroll
                    for (int i = 0; i < 16; ++i) S[v8_phys(i, b, c)] = x[i];
                }
                __syncthreads();                         // stage 1 done everywhere; sub-row s-1 fully consumed
                if (s + 1 < s1) v8_load_fwd_slice(smem + ((s + 1 - s0) & 1) * V8_SUBW, src + (s + 1) * V8_SUBW);
                uint2 w3[JIT3 ? 1 : 15];
                if constexpr (!JIT3) load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);   // stage-3 twiddles, in flight
                {   // stage 2: layers A+4..A+7, thread (a, c), elements b (stride 16)
                    const int aa = hi4, c = lo4;
#pragma unroll
                    for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                    fwd_radix<4>(x, tw, A + 4, (uint32_t)s * 16 + aa, q, q2);
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
                    if constexpr (JIT3) fwd_radix<4>(x, tw, A + 8, (uint32_t)s * 256 + t, q, q2);
                    else fwd16_tw(x, w3, q, q2);
                    uint4* o = reinterpret_cast<uint4*>(out + s * V8_SUBW + t * 16);
#pragma unroll
                    for (int v = 0; v < 4; ++v)
                        __stcs(o + v, make_uint4(canon4(x[4 * v], q, q2), canon4(x[4 * v + 1], q, q2),
                                                 canon4(x[4 * v + 2], q, q2), canon4(x[4 * v + 3], q, q2)));
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
                    if constexpr (PW) {
                        const uint4* ip2 = reinterpret_cast<const uint4*>(in2 + s * V8_SUBW + t * 16);
#pragma unroll
                        for (int v = 0; v < 4; ++v) {
                            const uint4 u = __ldcs(ip2 + v);
                            x[4 * v] = mul_mod(x[4 * v], u.x, lc); x[4 * v + 1] = mul_mod(x[4 * v + 1], u.y, lc);
                            x[4 * v + 2] = mul_mod(x[4 * v + 2], u.z, lc); x[4 * v + 3] = mul_mod(x[4 * v + 3], u.w, lc);
                        }
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
                    inv_radix<4, A == 0>(x, tw, A, (uint32_t)s, lc);
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
#pragma unroll 1
                for (int pass = p0; pass < p0 + NP; ++pass) {
                    const int c = pass * V8_T + t;
                    uint32_t x[R];
#pragma unroll
                    for (int k = 0; k < R; ++k) x[k] = out[k * V8_SUBW + c];
                    inv_radix<A, true>(x, tw, 0, 0, lc);
#pragma unroll
                    for (int k = 0; k < R; ++k) __stcs(out + k * V8_SUBW + c, canon2(x[k], q));
                }
            }
        }
        __syncthreads();                                 // smem buffers free for the next row
    }
}

}  // namespace wd
