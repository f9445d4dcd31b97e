// k_cc.cu -- launchers of the small-row-count CUDA-core kernels:
//   v1 (ntt_cuda_core.cuh): one 256/512-thread CTA per row, N = 2^12..2^17 -- AUTO below the SM count
//      of rows for N <= 2^14;
//   ntt_small: N < 2^12 (debug sizes);
//   v5 (ntt_cluster.cuh): one row over a 2^(logN-14)-CTA cluster, the row resident in distributed
//      shared memory -- AUTO below a quarter of the SM count of rows for N = 2^15, 2^16.
#include <algorithm>
#include "launch.h"
#include "ntt_cuda_core.cuh"
#include "ntt_cluster.cuh"

namespace wd {
namespace {

template <typename K>
int set_smem(K kern, int bytes) {
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess) return 4;
    if (cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100) != cudaSuccess) return 4;
    return 0;
}

template <int LOGN>
int prep_logn() {
    using S = CcShape<LOGN>;
    int e = set_smem(ntt_fwd_cc<LOGN>, S::SMEM_BYTES) | set_smem(ntt_inv_cc<LOGN, false>, S::SMEM_BYTES) |
            set_smem(ntt_inv_cc<LOGN, true>, S::SMEM_BYTES);
    if constexpr (LOGN >= 14) {
        e |= set_smem(ntt_fwd_cl<LOGN>, CL_BYTES) | set_smem(ntt_inv_cl<LOGN, false>, CL_BYTES) |
             set_smem(ntt_inv_cl<LOGN, true>, CL_BYTES);
        if constexpr (LOGN == 17) {     // 8-CTA clusters need the non-portable-size opt-in on some drivers
            cudaFuncSetAttribute(ntt_fwd_cl<LOGN>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            cudaFuncSetAttribute(ntt_inv_cl<LOGN, false>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            cudaFuncSetAttribute(ntt_inv_cl<LOGN, true>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            cudaGetLastError();
        }
    }
    return e;
}

template <int LOGN>
void v1(bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    using S = CcShape<LOGN>;
    if (fwd) ntt_fwd_cc<LOGN><<<rows, S::T, S::SMEM_BYTES, s>>>(a);
    else if (a.in2) ntt_inv_cc<LOGN, true><<<rows, S::T, S::SMEM_BYTES, s>>>(a);
    else ntt_inv_cc<LOGN, false><<<rows, S::T, S::SMEM_BYTES, s>>>(a);
}

template <int LOGN>
void v5(bool fwd, const NttArgs& a, uint32_t rows, int sm_count, cudaStream_t s) {
    constexpr int CLN = 1 << (LOGN - 14);
    const uint32_t units = std::max<uint32_t>(1, std::min<uint32_t>(rows, (uint32_t)(2 * sm_count / CLN)));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(units * CLN); cfg.blockDim = dim3(CL_T); cfg.dynamicSmemBytes = CL_BYTES; cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CLN; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cfg.attrs = at; cfg.numAttrs = 1;
    if (fwd) cudaLaunchKernelEx(&cfg, ntt_fwd_cl<LOGN>, a, rows);
    else if (a.in2) cudaLaunchKernelEx(&cfg, ntt_inv_cl<LOGN, true>, a, rows);
    else cudaLaunchKernelEx(&cfg, ntt_inv_cl<LOGN, false>, a, rows);
}

}  // namespace

int prep_cc(uint32_t logN) {
    switch (logN) {
        case 12: return prep_logn<12>();
        case 13: return prep_logn<13>();
        case 14: return prep_logn<14>();
        case 15: return prep_logn<15>();
        case 16: return prep_logn<16>();
        case 17: return prep_logn<17>();
        default:
            return set_smem(ntt_small<true, false>, 4 << logN) | set_smem(ntt_small<false, false>, 4 << logN) |
                   set_smem(ntt_small<false, true>, 4 << logN);
    }
}

void launch_v1(uint32_t logN, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    switch (logN) {
        case 12: v1<12>(fwd, a, rows, s); break;
        case 13: v1<13>(fwd, a, rows, s); break;
        case 14: v1<14>(fwd, a, rows, s); break;
        case 15: v1<15>(fwd, a, rows, s); break;
        case 16: v1<16>(fwd, a, rows, s); break;
        case 17: v1<17>(fwd, a, rows, s); break;
        default: {
            const int thr = std::min<int>(256, std::max<int>(32, (1 << logN) / 2));
            if (fwd) ntt_small<true, false><<<rows, thr, 4 << logN, s>>>(a, (int)logN);
            else if (a.in2) ntt_small<false, true><<<rows, thr, 4 << logN, s>>>(a, (int)logN);
            else ntt_small<false, false><<<rows, thr, 4 << logN, s>>>(a, (int)logN);
        }
    }
}

void launch_v5(uint32_t logN, bool fwd, const NttArgs& a, uint32_t rows, int sm_count, cudaStream_t s) {
    switch (logN) {
        case 14: v5<14>(fwd, a, rows, sm_count, s); break;
        case 15: v5<15>(fwd, a, rows, sm_count, s); break;
        case 16: v5<16>(fwd, a, rows, sm_count, s); break;
        case 17: v5<17>(fwd, a, rows, sm_count, s); break;
        default: break;
    }
}

}  // namespace wd
