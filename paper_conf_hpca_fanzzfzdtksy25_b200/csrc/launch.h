// launch.h -- internal host interface between the C ABI (wd_ntt.cu) and the kernel translation units.
// Every function here only configures and enqueues kernels on the given stream: no allocation, no
// synchronisation, no environment reads (those happen once, at plan creation).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <vector>
#include "common.cuh"
#include "tensor_tables.h"

namespace wd {

// ---- k_cc.cu: v1 (one CTA per row, N = 2^12..2^17), ntt_small (N < 2^12), v5 (row over a cluster,
//      N = 2^14..2^17)
int prep_cc(uint32_t logN);
void launch_v1(uint32_t logN, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s);
void launch_v5(uint32_t logN, bool fwd, const NttArgs& a, uint32_t rows, int sm_count, cudaStream_t s);

// ---- k_v8.cu: v8 (N = 2^12..2^17) and WD-CUDA (N = 2^16)
struct V8Occ { int ncl[4] = {0, 0, 0, 0}; };   // resident clusters per GPU for CL = 1, 2, 4, 8
int prep_v8(uint32_t logN, int sm_count, V8Occ* occ);
// cl in {1, 2, 4, 8}; epi: 0 plain, 1 RESCALE store map, 2 ModDown store map (forward only)
// tma (N = 2^13..2^16, epi = 0; ignored otherwise), bits: 1 = forward column phase fed by TMA,
// 2 = inverse column phase fed by TMA, 4 = inverse: next row's first sub-row requested during the
// column phase (register-fed)
void launch_v8(uint32_t logN, bool fwd, const NttArgs& a, uint32_t rows, int cl, int epi, const V8Occ& occ, int tma,
               cudaStream_t s);
int prep_wdcuda();
void launch_wdcuda(bool fwd, const NttArgs& a, const TensorTables& tc, uint32_t rows, int sm_count, cudaStream_t s);

// ---- k_tmr.cu: "tm", the TMEM-resident CUDA-core kernels (N = 2^13..2^16, plain transforms;
//      ntt_tmr.cuh, ntt_tms.cuh, ntt_tmt.cuh)
int prep_tmr();
// returns launches (1), -1 if the size or the arguments need v8 (pointwise product, store maps, strided
// rows), -2 if the tensor map cannot be encoded
int launch_tmr(uint32_t logN, bool fwd, const NttArgs& a, uint32_t rows, int sm_count, cudaStream_t s);
// N = 2^17 forward on its two 2^16 halves: `a` is the virtual half plan (2 L limbs, the re-indexed twiddles
// and LimbConst of wd_ntt.cu), rows2 = 2 x the 2^17 rows; a.in / a.out the 2^17 data
int launch_tmr17(const NttArgs& a, uint32_t rows2, int sm_count, cudaStream_t s);

// ---- k_tensor.cu: the round-1 tensor path (TENSOR, FUSED modes; N = 2^16)
int prep_tensor();
int launch_tensor(bool fwd, const NttArgs& a, const TensorTables& tc, uint32_t rows, int sm_count, cudaStream_t s);
int launch_fused(bool fwd, const NttArgs& a, const TensorTables& tc, uint32_t rows, int sm_count, float share,
                 cudaStream_t s);

// ---- k_tc4.cu: tensor-map encoding (cuTensorMapEncodeTiled through the runtime's driver entry
//      point), u32 elements, no interleave, 256-B L2 promotion; false if unavailable or rejected
bool tma_encode_u32(CUtensorMap* m, const void* base, uint32_t rank, const cuuint64_t* dims,
                    const cuuint64_t* strides, const cuuint32_t* box, CUtensorMapSwizzle sw);

// ---- k_tc4.cu: the warp-specialised 4-step tcgen05 kernel (N = 2^16, ntt_tc4.cuh)
struct Tc4Tables {
    uint8_t* d_mat = nullptr;      // [L][2 sets][17][4096] byte-plane stage matrices (forward)
    uint2* d_tw = nullptr;         // [L][2][16][16][128] per-element twist in worker-lane order (forward)
    uint4* d_lq = nullptr;         // [L] {q, Shoup(2^16), Shoup(1), 0}
    bool ok = false;
};
int build_tc4_tables(Tc4Tables& t, const std::vector<uint32_t>& primes, const std::vector<uint32_t>& psis);
void free_tc4_tables(Tc4Tables& t);
int prep_tc4();
// returns launches (> 0), -1 unsupported arguments, -2 tensor-map encoding failure
void tc4_set_trace(void* dev_buf);   // diagnostics: CTA-0 event timestamps (20480 x u64) or nullptr
int launch_tc4(bool fwd, const NttArgs& a, const Tc4Tables& t, uint32_t rows, int sm_count, cudaStream_t s);

// ---- k_rns.cu: RESCALE gather, fast basis conversion, 64-bit share reduction
struct BconvTab {
    const uint4* src;       // [S] {q_i, (Q/q_i)^-1 mod q_i, Shoup, 0}
    const uint2* w;         // [S][D] {(Q/q_i) mod p_j, its Shoup companion mod p_j}
    const uint4* dst;       // [D] {p_j, mu_lo, mu_hi, 0}: mu = floor((2^64 - 1) / p_j)
    uint32_t S, D;
};
constexpr int BC_MAX = 64;                // max source / target limbs of a conversion
int prep_rns();
void launch_rs_gather(const uint32_t* in, uint32_t* work, uint32_t N, uint32_t L, uint32_t batch, int sm_count,
                      cudaStream_t s);
void launch_bconv(const uint32_t* x, uint32_t x_ls, uint32_t* y, uint32_t y_ls, uint32_t y_off, const BconvTab& t,
                  uint32_t N, uint32_t batch, int sm_count, cudaStream_t s);
void launch_bconv_partial(const uint32_t* x, uint32_t x_ls, uint64_t* y64, const BconvTab& t, uint32_t N,
                          uint32_t batch, int sm_count, cudaStream_t s);
void launch_reduce64(const uint64_t* sum, uint32_t* out, const uint4* dst, uint32_t D, uint32_t N, uint32_t rows,
                     int sm_count, cudaStream_t s);

}  // namespace wd
