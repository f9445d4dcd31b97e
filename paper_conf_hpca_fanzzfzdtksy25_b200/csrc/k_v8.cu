// k_v8.cu -- launchers of the CUDA-core v8 kernel and of
// WD-CUDA (row f2).  Kernels in ntt_v8.cuh.
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include "launch.h"
#include "ntt_v8.cuh"

namespace wd {
namespace {

constexpr int v8_cl_index(int cl) { return cl == 1 ? 0 : cl == 2 ? 1 : cl == 4 ? 2 : 3; }

template <typename K>
int set_smem(K kern, int bytes) {
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess) return 4;
    if (cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100) != cudaSuccess) return 4;
    return 0;
}

template <int LOGN, int CL>
constexpr bool cl_ok() { return (1 << (LOGN - 12)) % CL == 0; }
template <int LOGN>
constexpr bool tm_ok() { return LOGN >= 13 && LOGN <= 16; }   // the TMA column phase: 2 <= 2^A <= 16

template <int LOGN, int CL>
int prep_cl(int sm_count, V8Occ* occ) {
    if constexpr (!cl_ok<LOGN, CL>()) {
        return 0;
    } else {
        int e = set_smem(ntt_v8<LOGN, true, false, CL>, V8_SMEM_K) | set_smem(ntt_v8<LOGN, false, false, CL>, V8_SMEM_K) |
                set_smem(ntt_v8<LOGN, false, true, CL>, V8_SMEM_K);
        if constexpr (tm_ok<LOGN>())
            e |= set_smem(ntt_v8<LOGN, true, false, CL, 0, 1>, V8_SMEM_K) |
                 set_smem(ntt_v8<LOGN, false, false, CL, 0, 1>, V8_SMEM_K) |
                 set_smem(ntt_v8<LOGN, false, false, CL, 0, 2>, V8_SMEM_K);
        if (CL == (LOGN > 12 ? 2 : 1))
            e |= set_smem(ntt_v8<LOGN, true, false, CL, 1>, V8_SMEM_K) | set_smem(ntt_v8<LOGN, true, false, CL, 2>, V8_SMEM_K);
        if (e) return e;
        // WD_NTT_V8_CTAS (A/B runs; read once per process, at the first plan): CTAs per SM the
        // persistent grid is sized for
        static const int ctas_env = getenv("WD_NTT_V8_CTAS") ? std::max(1, std::min(4, atoi(getenv("WD_NTT_V8_CTAS")))) : 4;
        int ncl = sm_count * ctas_env / CL;
        if (CL > 1) {                    // resident clusters, queried once per plan (not per launch)
            cudaLaunchConfig_t cfg = {};
            cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V8_SMEM_K;
            cfg.gridDim = dim3(sm_count * 4 / CL * CL);
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = CL; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
            cfg.attrs = at; cfg.numAttrs = 1;
            int n = 0;
            if (cudaOccupancyMaxActiveClusters(&n, ntt_v8<LOGN, true, false, CL>, &cfg) != cudaSuccess || n < 1) {
                cudaGetLastError();
                n = sm_count * 4 / CL;
            }
            ncl = std::min(n, sm_count * ctas_env / CL);
        }
        occ->ncl[v8_cl_index(CL)] = ncl;
        return 0;
    }
}

template <int LOGN>
int prep_logn(int sm_count, V8Occ* occ) {
    return prep_cl<LOGN, 1>(sm_count, occ) | prep_cl<LOGN, 2>(sm_count, occ) | prep_cl<LOGN, 4>(sm_count, occ) |
           prep_cl<LOGN, 8>(sm_count, occ);
}

// the column-phase input as a 2-D tensor: inner dimension the 4096 columns, outer one line per
// (physical row, k); box = one column pass (256 columns x 2^A lines)
// (forward: the input rows; inverse: the output rows, which hold the intermediate)
bool encode_v8_cols(CUtensorMap* m, uint32_t logN, const uint32_t* base, uint32_t ls, uint32_t L, uint32_t rows) {
    const uint32_t R = 1u << (logN - 12);
    const uint64_t phys = ls ? (uint64_t)(rows / L - 1) * ls + L : rows;
    const cuuint64_t dims[2] = {V8_SUBW, phys * R}, strides[1] = {V8_SUBW * 4};
    const cuuint32_t box[2] = {V8_T, R};
    return tma_encode_u32(m, base, 2, dims, strides, box, CU_TENSOR_MAP_SWIZZLE_NONE);
}

template <int LOGN, int CL, int EPI>
void launch_k(bool fwd, const NttArgs& a, uint32_t rows, int ncl, int tma, cudaStream_t s) {
    if constexpr (!cl_ok<LOGN, CL>()) {
        return;
    } else {
        auto k = fwd ? ntt_v8<LOGN, true, false, CL, EPI> : (a.in2 ? ntt_v8<LOGN, false, true, CL> : ntt_v8<LOGN, false, false, CL>);
        alignas(64) CUtensorMap tm;
        std::memset(&tm, 0, sizeof(tm));
        const int smem = V8_SMEM_K;
        if constexpr (tm_ok<LOGN>() && EPI == 0) {
            if ((tma & 1) && fwd && encode_v8_cols(&tm, LOGN, a.in, a.in_ls, a.L, a.nb_total ? a.nb_total * a.L : rows)) {
                k = ntt_v8<LOGN, true, false, CL, 0, 1>;
            } else if ((tma & 2) && !fwd && !a.in2 && encode_v8_cols(&tm, LOGN, a.out, a.out_ls, a.L, a.nb_total ? a.nb_total * a.L : rows)) {
                k = ntt_v8<LOGN, false, false, CL, 0, 1>;
            } else if ((tma & 4) && !fwd && !a.in2) {
                k = ntt_v8<LOGN, false, false, CL, 0, 2>;
            }
        }
        const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)ncl) * CL;
        if constexpr (CL == 1) {
            k<<<grid, V8_T, smem, s>>>(a, rows, tm);
        } else {
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(grid); cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = smem; cfg.stream = s;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = CL; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
            cfg.attrs = at; cfg.numAttrs = 1;
            cudaLaunchKernelEx(&cfg, k, a, rows, tm);
        }
    }
}

template <int LOGN>
void launch_logn(bool fwd, const NttArgs& a, uint32_t rows, int cl, int epi, const V8Occ& occ, int tma,
                 cudaStream_t s) {
    const int n = occ.ncl[v8_cl_index(cl)];
    if (epi) {                           // the RNS store maps exist at the default cluster size only
        constexpr int CD = LOGN > 12 ? 2 : 1;
        const int nd = occ.ncl[v8_cl_index(CD)];
        if (epi == 1) launch_k<LOGN, CD, 1>(true, a, rows, nd, 0, s);
        else launch_k<LOGN, CD, 2>(true, a, rows, nd, 0, s);
        return;
    }
    switch (cl) {
        case 8: launch_k<LOGN, 8, 0>(fwd, a, rows, n, tma, s); break;
        case 4: launch_k<LOGN, 4, 0>(fwd, a, rows, n, tma, s); break;
        case 2: launch_k<LOGN, 2, 0>(fwd, a, rows, n, tma, s); break;
        default: launch_k<LOGN, 1, 0>(fwd, a, rows, n, tma, s); break;
    }
}

}  // namespace

int prep_v8(uint32_t logN, int sm_count, V8Occ* occ) {
    switch (logN) {
        case 12: return prep_logn<12>(sm_count, occ);
        case 13: return prep_logn<13>(sm_count, occ);
        case 14: return prep_logn<14>(sm_count, occ);
        case 15: return prep_logn<15>(sm_count, occ);
        case 16: return prep_logn<16>(sm_count, occ);
        case 17: return prep_logn<17>(sm_count, occ);
        default: return 0;
    }
}

void launch_v8(uint32_t logN, bool fwd, const NttArgs& a, uint32_t rows, int cl, int epi, const V8Occ& occ, int tma,
               cudaStream_t s) {
    const int maxcl = 1 << std::min<int>(3, (int)logN - 12);
    cl = std::max(1, std::min(cl, maxcl));
    switch (logN) {
        case 12: launch_logn<12>(fwd, a, rows, cl, epi, occ, tma, s); break;
        case 13: launch_logn<13>(fwd, a, rows, cl, epi, occ, tma, s); break;
        case 14: launch_logn<14>(fwd, a, rows, cl, epi, occ, tma, s); break;
        case 15: launch_logn<15>(fwd, a, rows, cl, epi, occ, tma, s); break;
        case 16: launch_logn<16>(fwd, a, rows, cl, epi, occ, tma, s); break;
        default: launch_logn<17>(fwd, a, rows, cl, epi, occ, tma, s); break;
    }
}

int prep_wdcuda() {
    return set_smem(ntt_wdcuda16<true>, V8_SMEM + 2048) | set_smem(ntt_wdcuda16<false>, V8_SMEM + 2048);
}

// WD-CUDA (row f2): the four radix-16 inner DFTs as 32-bit GEMMs on the CUDA cores, N = 2^16
void launch_wdcuda(bool fwd, const NttArgs& a, const TensorTables& tc, uint32_t rows, int sm_count, cudaStream_t s) {
    WdcArgs wa;
    wa.a = a; wa.mat = tc.d_mat;
    wa.t1 = fwd ? tc.d_tw1 : tc.d_sg1; wa.t2 = fwd ? tc.d_tw2 : tc.d_sg2; wa.t3 = fwd ? tc.d_tw3 : tc.d_sg3;
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V8_SMEM + 2048; cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cfg.attrs = at; cfg.numAttrs = 1;
    cfg.gridDim = dim3(std::min<uint32_t>(rows, (uint32_t)(sm_count * 3 / 2)) * 2);
    if (fwd) cudaLaunchKernelEx(&cfg, ntt_wdcuda16<true>, wa, rows);
    else cudaLaunchKernelEx(&cfg, ntt_wdcuda16<false>, wa, rows);
}

}  // namespace wd
