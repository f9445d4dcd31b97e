// k_tmr.cu -- launcher of the TMEM-resident CUDA-core NTT "tm" (N = 2^13..2^16; kernels in ntt_tmr.cuh,
// ntt_tms.cuh and ntt_tmt.cuh).
// This unit compiles the Harvey butterflies with their X + t / X + Y adds pinned to the ALU pipe
// (modarith.cuh WD_BFLY_ALU: min(x + t, 4q), one VIADDMNMX instead of an IMAD.IADD on the fma pipe).
// In the TMEM-resident kernel the fma pipe is the busiest one (ncu math_pipe_throttle); measured on
// config 3: forward 1.022 -> 1.007 ms, inverse 0.963 -> 0.957 ms.  The v8 unit keeps the default
// (there the same change made the forward slower: 1.061 -> 1.080 ms).  Device functions are compiled
// per translation unit (no relocatable device code), so the two choices never meet.
#define WD_BFLY_ALU 1
#include <algorithm>
#include <cstring>
#include "launch.h"
#include "ntt_tmt.cuh"

namespace wd {

namespace {
template <typename K>
int set_attr(K k, int smem) {
    if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess ||
        cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, 100) != cudaSuccess)
        return 4;
    return 0;
}
}  // namespace

int prep_tmr() {
    return set_attr(tmr::ntt_tmr16<true>, tmr::SMEM) | set_attr(tmr::ntt_tmr16<false>, tmr::SMEM) |
           set_attr(tms::ntt_tms<2, true>, tms::SMEM) | set_attr(tms::ntt_tms<2, false>, tms::SMEM) |
           set_attr(tms::ntt_tms<3, true>, tms::SMEM) | set_attr(tms::ntt_tms<3, false>, tms::SMEM) |
           set_attr(tmt::ntt_tmt13<true>, tmt::SMEM) | set_attr(tmt::ntt_tmt13<false>, tmt::SMEM) |
           set_attr(tmr::ntt_tmr16<true, true>, tmr::SMEM);
}

// plain transforms only (contiguous [batch][L][N] rows, no pointwise product / store maps / copies);
// returns launches (1), -1 if the arguments need v8, -2 if the tensor map cannot be encoded
int launch_tmr(uint32_t logN, bool fwd, const NttArgs& a, uint32_t rows, int sm_count, cudaStream_t s) {
    // rows_all: the whole batch's rows (the launch may cover its first `rows` schedule slots only)
    const uint64_t rows_all = a.nb_total ? (uint64_t)a.nb_total * a.L : rows;
    if (logN < 13 || logN > 16 || a.in2 || a.aux || a.cpy || a.in_ls || a.out_ls || rows_all % a.L || a.slot0 ||
        rows > rows_all)
        return -1;                               // (the tm kernels start at schedule slot 0)
    const uint32_t R = 1u << (logN - 12);
    alignas(64) CUtensorMap tm;
    std::memset(&tm, 0, sizeof(tm));
    if (fwd && logN == 13) {   // {256 columns, 16 passes, one line per (row, k)}; box: 8 passes x 2 lines
        const cuuint64_t dims[3] = {tmr::TT, 16, (cuuint64_t)rows_all * R};
        const cuuint64_t strides[2] = {tmr::TT * 4, tmr::SUBW * 4};
        const cuuint32_t box[3] = {tmr::TT, 8, R};
        if (!tma_encode_u32(&tm, a.in, 3, dims, strides, box, CU_TENSOR_MAP_SWIZZLE_NONE)) return -2;
    } else if (fwd) {   // the column passes: inner dimension the 4096 columns, one line per (row, k); box 256 x R
        const cuuint64_t dims[2] = {tmr::SUBW, (cuuint64_t)rows_all * R}, strides[1] = {tmr::SUBW * 4};
        const cuuint32_t box[2] = {tmr::TT, R};
        if (!tma_encode_u32(&tm, a.in, 2, dims, strides, box, CU_TENSOR_MAP_SWIZZLE_NONE)) return -2;
    }
    const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)sm_count);
    if (logN == 16) {
        if (fwd) tmr::ntt_tmr16<true><<<grid, tmr::NT, tmr::SMEM, s>>>(a, rows, tm);
        else tmr::ntt_tmr16<false><<<grid, tmr::NT, tmr::SMEM, s>>>(a, rows, tm);
    } else if (logN == 15) {
        if (fwd) tms::ntt_tms<3, true><<<grid, tmr::NT, tms::SMEM, s>>>(a, rows, tm);
        else tms::ntt_tms<3, false><<<grid, tmr::NT, tms::SMEM, s>>>(a, rows, tm);
    } else if (logN == 14) {
        if (fwd) tms::ntt_tms<2, true><<<grid, tmr::NT, tms::SMEM, s>>>(a, rows, tm);
        else tms::ntt_tms<2, false><<<grid, tmr::NT, tms::SMEM, s>>>(a, rows, tm);
    } else {   // N = 2^13: one team per row, four rows per CTA
        const uint32_t g13 = std::min<uint32_t>((rows + 3) / 4, (uint32_t)sm_count);
        if (fwd) tmt::ntt_tmt13<true><<<g13, tmr::NT, tmt::SMEM, s>>>(a, rows, tm);
        else tmt::ntt_tmt13<false><<<g13, tmr::NT, tmt::SMEM, s>>>(a, rows, tm);
    }
    return 1;
}

int launch_tmr17(const NttArgs& a, uint32_t rows2, int sm_count, cudaStream_t s) {
    alignas(64) CUtensorMap tm;
    std::memset(&tm, 0, sizeof(tm));
    // the 2^17 input as lines of 4096 words (32 per row, 16 per half-row); a column pass loads two 256 x 16
    // boxes (both halves of its columns)
    const cuuint64_t dims[2] = {tmr::SUBW, (cuuint64_t)rows2 * 16}, strides[1] = {tmr::SUBW * 4};
    const cuuint32_t box[2] = {tmr::TT, 16};
    if (!tma_encode_u32(&tm, a.in, 2, dims, strides, box, CU_TENSOR_MAP_SWIZZLE_NONE)) return -2;
    const uint32_t grid = std::min<uint32_t>(rows2, (uint32_t)sm_count);
    tmr::ntt_tmr16<true, true><<<grid, tmr::NT, tmr::SMEM, s>>>(a, rows2, tm);
    return 1;
}

}  // namespace wd
