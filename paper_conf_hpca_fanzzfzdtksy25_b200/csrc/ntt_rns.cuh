// ntt_rns.cuh -- RNS operations built around the NTT as PE kernels.
//
// RESCALE ("RSCALE(ct0) = (a0', b0') in R^2_{Q_{l-1}}"; reading C-18):
// a' = round(a / q_last) coefficient-wise, inputs and outputs in the NTT domain.  The RNS
// algorithm (oracle/rns.py is its independent CPU statement):
//   1. c  = INTT_{q_last}(a_last)                         -- one row per polynomial
//   2. v  = c - q_last [c >= q_last - floor(q_last/2)]     -- centred residue of A mod q_last
//   3. a'_i = (a_i - NTT_{q_i}(v mod q_i)) * q_last^{-1}   -- every i < last
// Launches (all polynomials of the batch in each, the PE-kernel rule of PAPER.md:334-352):
//   K1 rs_gather   copies the last-limb rows into the caller's work buffer (batch x N words),
//   K2 inverse NTT of those rows (the plan's CUDA-core kernels, a 1-limb view of the plan),
//   K3 ntt_v8<..., EPI = 1>: the forward NTT of all batch x (L-1) output rows whose phase-1
//      load applies step 2 (+ reduction mod q_i) to the shared row of its polynomial and whose
//      final store applies step 3 against the input limb -- no intermediate v_i rows in HBM.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include "ntt_cuda_core.cuh"

namespace wd {

// work[p][n] = in[p][L-1][n]: 16-byte vectors, grid-stride
__global__ void __launch_bounds__(256) rs_gather(const uint4* __restrict__ in, uint4* __restrict__ work,
                                                 uint32_t n4, uint32_t L, uint32_t batch) {
    const size_t total = (size_t)batch * n4;
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total; i += (size_t)gridDim.x * blockDim.x) {
        const size_t p = i / n4, j = i - p * n4;
        work[i] = __ldcs(in + (p * L + (L - 1)) * n4 + j);
    }
}

}  // namespace wd
