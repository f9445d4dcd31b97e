// ntt_v12.cuh -- v8 with the phases of consecutive rows interleaved inside each CTA (forward,
// N = 2^13 .. 2^16).
//
// Measured on v8: the column phase of a row is memory-bound (0.41 ms alone at
// config 3) and its row phase is fma/issue-bound (0.77 ms alone), but the full kernel takes
// about the sum of the two (1.05 ms): the 4 CTAs of an SM run their phases in near lock-step,
// so the memory phase of one does not hide under the butterflies of another.  v12 interleaves
// them inside every CTA instead: while it runs the row phase of row k (sub-row j), the 16 KB
// column pass j of row k+1 streams into a third shared-memory buffer (warp-private 16-byte
// cp.async slices, v9_load_cols), and right after sub-row j's stage 3 the CTA runs column pass
// j of row k+1 from that buffer.  Every compute-bound sub-row therefore has one memory-bound
// column pass in flight under it.  Arithmetic, layouts, twiddles and the stage code are v8's;
// the result is bit-identical.
//
// cp.async group order per sub-row j: [sub-row j (issued during j-1)] [column pass j]
// [sub-row j+1 (after stage 1's barrier), or an empty group] -> wait_group<1> before stage 1
// (sub-row j landed), wait_group<1> before the column pass (pass j landed).
#pragma once
#include "ntt_v8.cuh"

namespace wd {

constexpr int V12_SMEM = 3 * V8_SUBW * 4;    // two sub-row buffers + one column-pass buffer

template <int LOGN>
__global__ void __launch_bounds__(V8_T, 4) ntt_v12f(NttArgs a, uint32_t rows) {
    constexpr int A = LOGN - 12;
    constexpr int R = 1 << A;
    constexpr int CL = 2;
    static_assert(A >= 1 && A <= 4, "v12: N = 2^13 .. 2^16");
    constexpr int NP = V8_SUBW / V8_T / CL;  // column passes per CTA (8)
    constexpr int NS = R / CL;               // sub-rows per CTA
    static_assert(NS <= NP, "one column pass per sub-row slot, the rest after the last sub-row");
    const int rank = (int)(blockIdx.x % CL);
    const int p0 = rank * NP, s0 = rank * NS, s1 = s0 + NS;
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* const CB = smem + 2 * V8_SUBW;
    const int t = threadIdx.x, w = t >> 5, lane = t & 31;
    const int hi4 = t >> 4, lo4 = t & 15;
    const uint32_t rstep = gridDim.x / CL;
    uint32_t row = blockIdx.x / CL;
    if (row >= rows) return;                                 // uniform over the cluster

    // column pass `pass` of row r from the warp-private slice in CB -> r's out slot
    auto col_from_cb = [&](uint32_t r, int pass) {
        const uint32_t limb = r % a.L;
        const LimbConst lc = a.lc[limb];
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        uint32_t* out = a.out + ((size_t)r << LOGN);
        const int c = pass * V8_T + t;
        uint32_t x[R];
#pragma unroll
        for (int k = 0; k < R; ++k) x[k] = CB[w * 32 * R + 32 * k + lane];
        fwd_radix<A>(x, tw, 0, 0, lc.q, lc.q2);
#pragma unroll
        for (int k = 0; k < R; ++k) out[k * V8_SUBW + c] = x[k];
    };
    // prologue: the column phase of the first row, straight from global (as v8)
    {
        const uint32_t limb = row % a.L;
        const LimbConst lc = a.lc[limb];
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        const uint32_t* in = a.in + ((size_t)row << LOGN);
        uint32_t* out = a.out + ((size_t)row << LOGN);
#pragma unroll 1
        for (int pass = p0; pass < p0 + NP; ++pass) {
            const int c = pass * V8_T + t;
            uint32_t x[R];
#pragma unroll
            for (int k = 0; k < R; ++k) x[k] = __ldcs(in + k * V8_SUBW + c);
            fwd_radix<A>(x, tw, 0, 0, lc.q, lc.q2);
#pragma unroll
            for (int k = 0; k < R; ++k) out[k * V8_SUBW + c] = x[k];
        }
        cluster_sync();
    }

#pragma unroll 1
    for (; row < rows; row += rstep) {
        const uint32_t nrow = row + rstep;
        const bool has_next = nrow < rows;
        const uint32_t limb = row % a.L;
        const LimbConst lc = a.lc[limb];
        const uint32_t q = lc.q, q2 = lc.q2;
        const uint2* __restrict__ tw = a.tw + ((size_t)limb << LOGN);
        uint32_t* out = a.out + ((size_t)row << LOGN);
        const uint32_t* nin = a.in + ((size_t)nrow << LOGN);

        v8_load_fwd_slice(smem, out + s0 * V8_SUBW);          // group: sub-row s0
#pragma unroll 1
        for (int j = 0; j < NS; ++j) {
            const int s = s0 + j;
            uint32_t* S = smem + (j & 1) * V8_SUBW;
            if (has_next) v9_load_cols<R>(CB, nin, (p0 + j) * V8_T);   // group: column pass j of nrow
            else cp_async_commit();
            cp_async_wait<1>();
            __syncwarp();                                     // this warp's stage-1 slice of sub-row s landed
            uint32_t x[16];
            {   // stage 1: layers A..A+3, thread (b, c), elements a (stride 256)
                const int b = hi4, c = lo4;
#pragma unroll
                for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(i, b, c)];
                fwd_radix<4>(x, tw, A, (uint32_t)s, q, q2);
#pragma unroll
                for (int i = 0; i < 16; ++i) S[v8_phys(i, b, c)] = x[i];
            }
            __syncthreads();                                  // stage 1 done everywhere; sub-row s-1 consumed
            if (s + 1 < s1) v8_load_fwd_slice(smem + ((j + 1) & 1) * V8_SUBW, out + (s + 1) * V8_SUBW);
            else cp_async_commit();                           // keep the group count uniform
            uint2 w3[15];
            load_tw16(w3, tw, A + 8, (uint32_t)s * 256 + t);
            {   // stage 2: layers A+4..A+7, thread (a, c), elements b (stride 16)
                const int aa = hi4, c = lo4;
#pragma unroll
                for (int i = 0; i < 16; ++i) x[i] = S[v8_phys(aa, i, c)];
                fwd_radix<4>(x, tw, A + 4, (uint32_t)s * 16 + aa, q, q2);
#pragma unroll
                for (int i = 0; i < 16; ++i) S[v8_phys(aa, i, c)] = x[i];
            }
            __syncwarp();
            {   // stage 3: layers A+8..A+11, thread (a, b), 16 contiguous elements -> global
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
            if (has_next) {                                   // column pass j of the next row
                cp_async_wait<1>();
                __syncwarp();
                col_from_cb(nrow, p0 + j);
                __syncwarp();                                 // CB slice read before it is refilled
            }
        }
        if (has_next) {                                       // passes without a sub-row slot (NS < NP)
#pragma unroll 1
            for (int j = NS; j < NP; ++j) {
                v9_load_cols<R>(CB, nin, (p0 + j) * V8_T);
                cp_async_wait<0>();
                __syncwarp();
                col_from_cb(nrow, p0 + j);
                __syncwarp();
            }
        }
        cp_async_wait<0>();
        cluster_sync();                                       // next row's intermediate complete
    }
}

}  // namespace wd
