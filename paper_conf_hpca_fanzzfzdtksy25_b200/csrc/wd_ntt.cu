// wd_ntt.cu -- libwdntt.so: plan precompute, C ABI and dispatch (b).
//
// The ABI is declared and documented in include/wd_ntt.h.  Everything on the
// call path is asynchronous on the caller's stream; the only host<->device
// copies are the one-time table upload in wd_ntt_plan_create
// and the explicit host-buffer entry points.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <vector>

#include "wd_ntt.h"
#include "modarith.cuh"
#include "ntt_cuda_core.cuh"
#include "ntt_persist.cuh"
#include "ntt_v8.cuh"
#include "ntt_v12.cuh"
#include "ntt_smem.cuh"
#include "ntt_cluster.cuh"
#include "ntt_tensor.cuh"
#include "ntt_fused.cuh"
#include "ntt_rns.cuh"
#include "plan_math.h"

using namespace wd;

namespace {
thread_local int g_last_error = WD_OK;
thread_local uint32_t g_last_launches = 0;
int set_err(int e) { g_last_error = e; return e; }
}  // namespace

struct wd_ntt_plan {
    uint32_t N = 0, logN = 0, L = 0;
    int device = -1;
    int sm_count = 148;
    int v6_ctas = 4;               // resident 256-thread CTAs per SM for v6 (WD_NTT_CTAS: 2..4, A/B runs)
    int v8_minb = 0;               // v8 CTAs per SM (WD_NTT_MINB: 4..6; 0 = measured default)
    int v8_cl = 0;                 // v8 CTAs per row cluster (WD_NTT_CL: 1, 2, 4; 0 = measured default)
    uint32_t stagger_ns = 0;       // WD_NTT_STAGGER (v8 experiment)
    uint32_t limb_major = 1;       // v8 row schedule, limb by limb (WD_NTT_LM=0: natural order)
    int kernel_ver = 0;            // 0 = AUTO, the measured default per N and row count (launch_cc);
                                   // WD_NTT_KERNEL=v1|v2|v3|v5|v6 forces a generation (A/B runs)
    std::vector<uint32_t> primes, psi;
    uint2* d_fwd = nullptr;        // [L][N]  (psi^brv(i), Shoup)
    uint2* d_inv = nullptr;        // [L][N]  (psi^-brv(i), Shoup)
    LimbConst* d_lc = nullptr;     // [L]
    uint4* d_rs = nullptr;         // [L] RESCALE constants vs the last prime (ntt_rns.cuh); L >= 2
    uint32_t rs_thr = 0;           // q_last - floor(q_last / 2)
    bool rs_ok = false;            // L >= 2 and q_last differs from every other prime
    TensorTables tc;               // tensor-path planes (ntt_tensor.cuh)
    int mode = WD_MODE_AUTO;
    float tensor_share = 0.5f;
    cudaStream_t hs[3] = {nullptr, nullptr, nullptr};   // host-path pipeline streams
    cudaEvent_t he[4] = {nullptr, nullptr, nullptr, nullptr};
    float ftc_share = 0.7f;        // WD_MODE_FTC: polynomials on WD-Tensor (best of 0.5/0.6/0.7 at config 3)
    cudaStream_t fs = nullptr;     // WD_MODE_FTC fork stream and its fork / join events
    cudaEvent_t fe[2] = {nullptr, nullptr};
    mutable std::mutex ftc_mu;     // orders fork/join event use across host threads
    std::mutex host_mu;
};

namespace {

bool is_pow2(uint32_t n) { return n && !(n & (n - 1)); }
uint32_t ilog2u(uint32_t n) { uint32_t l = 0; while ((1u << l) < n) ++l; return l; }

int check_prime(uint32_t q, uint32_t N) {
    if (q >= (1u << 30) || q < 3) return WD_EPRIME;
    if ((q - 1) % (2ull * N) != 0) return WD_EPRIME;
    if (!pm_is_prime(q)) return WD_EPRIME;
    return WD_OK;
}

template <typename K>
int set_smem(K kern, int bytes) {
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess)
        return WD_ECUDA;
    // ask for the maximum shared-memory carveout so occupancy is limited by our own budget
    if (cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100) != cudaSuccess)
        return WD_ECUDA;
    return WD_OK;
}

template <int LOGN>
int prep_cc() {
    using S = CcShape<LOGN>;
    if (set_smem(ntt_fwd_cc<LOGN>, S::SMEM_BYTES) || set_smem(ntt_inv_cc<LOGN, false>, S::SMEM_BYTES) ||
        set_smem(ntt_inv_cc<LOGN, true>, S::SMEM_BYTES))
        return WD_ECUDA;
    if constexpr (LOGN >= 12) {
        if (set_smem(ntt_v8<LOGN, true, false, 0, 4>, V8_SMEM) || set_smem(ntt_v8<LOGN, false, false, 0, 4>, V8_SMEM) ||
            set_smem(ntt_v8<LOGN, false, true, 0, 4>, V8_SMEM) || set_smem(ntt_v8<LOGN, true, false, 0, 5>, V8_SMEM) ||
            set_smem(ntt_v8<LOGN, false, false, 0, 5>, V8_SMEM) || set_smem(ntt_v8<LOGN, false, true, 0, 5>, V8_SMEM) ||
            set_smem(ntt_v8<LOGN, true, false, 0, 6>, V8_SMEM) || set_smem(ntt_v8<LOGN, false, false, 0, 6>, V8_SMEM) ||
            set_smem(ntt_v8<LOGN, false, true, 0, 6>, V8_SMEM))
            return WD_ECUDA;
    }
    if constexpr (LOGN >= 12) {
        if (set_smem(ntt_v8<LOGN, true, false, 0, 4, (LOGN > 12 ? 2 : 1), 1>, V8_SMEM) ||
            set_smem(ntt_v8<LOGN, true, false, 0, 4, (LOGN > 12 ? 2 : 1), 2>, V8_SMEM))
            return WD_ECUDA;
    }
    if constexpr (LOGN == 16) {
        if (set_smem(ntt_wdcuda16<true>, V8_SMEM + 2048) || set_smem(ntt_wdcuda16<false>, V8_SMEM + 2048)) return WD_ECUDA;
        if (set_smem(ntt_v11<true, 1>, V11_SMEM) || set_smem(ntt_v11<false, 1>, V11_SMEM) ||
            set_smem(ntt_v11<true, 3>, V11_SMEM) || set_smem(ntt_v11<false, 3>, V11_SMEM) ||
            set_smem(ntt_v11<true, 6>, V11_SMEM) || set_smem(ntt_v11<false, 6>, V11_SMEM) ||
            set_smem(ntt_v11<true, 7>, V11_SMEM) || set_smem(ntt_v11<false, 7>, V11_SMEM))
            return WD_ECUDA;
        if (set_smem(ntt_v10<true, false, 1>, V10_SMEM) || set_smem(ntt_v10<false, false, 1>, V10_SMEM) ||
            set_smem(ntt_v10<false, true, 1>, V10_SMEM) || set_smem(ntt_v10<true, false, 2>, V10_SMEM) ||
            set_smem(ntt_v10<false, false, 2>, V10_SMEM) || set_smem(ntt_v10<false, true, 2>, V10_SMEM))
            return WD_ECUDA;
    }
    if constexpr (LOGN >= 13 && LOGN <= 16) {
        if (set_smem(ntt_v9<LOGN, true, false, 1>, V9_SMEM) || set_smem(ntt_v9<LOGN, false, false, 1>, V9_SMEM) ||
            set_smem(ntt_v9<LOGN, false, true, 1>, V9_SMEM) || set_smem(ntt_v9<LOGN, true, false, 2>, V9_SMEM) ||
            set_smem(ntt_v9<LOGN, false, false, 2>, V9_SMEM) || set_smem(ntt_v9<LOGN, false, true, 2>, V9_SMEM))
            return WD_ECUDA;
    }
    if constexpr (LOGN >= 14) {
        if (set_smem(ntt_fwd_cl<LOGN>, CL_BYTES) || set_smem(ntt_inv_cl<LOGN, false>, CL_BYTES) ||
            set_smem(ntt_inv_cl<LOGN, true>, CL_BYTES))
            return WD_ECUDA;
        if constexpr (LOGN == 17) {     // 8-CTA clusters need the non-portable-size opt-in on some drivers
            cudaFuncSetAttribute(ntt_fwd_cl<LOGN>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            cudaFuncSetAttribute(ntt_inv_cl<LOGN, false>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            cudaFuncSetAttribute(ntt_inv_cl<LOGN, true>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            cudaGetLastError();
        }
    }
    if constexpr (LOGN == 15 || LOGN == 16) {
        if (set_smem(ntt_fwd_smem<LOGN>, SM_BYTES) || set_smem(ntt_inv_smem<LOGN, false>, SM_BYTES) ||
            set_smem(ntt_inv_smem<LOGN, true>, SM_BYTES))
            return WD_ECUDA;
    }
    if constexpr (LOGN >= 15) {
        using G = PGeo<LOGN>;
        if (set_smem(ntt_persist_cc<LOGN, true, false>, G::SMEM_BYTES) ||
            set_smem(ntt_persist_cc<LOGN, false, false>, G::SMEM_BYTES) ||
            set_smem(ntt_persist_cc<LOGN, false, true>, G::SMEM_BYTES))
            return WD_ECUDA;
    }
    if constexpr (LOGN == 16 || LOGN == 17) {
        using G7 = PGeo<LOGN, 128>;
        if (set_smem(ntt_persist_cc<LOGN, true, false, 128>, G7::SMEM_BYTES) ||
            set_smem(ntt_persist_cc<LOGN, false, false, 128>, G7::SMEM_BYTES) ||
            set_smem(ntt_persist_cc<LOGN, false, true, 128>, G7::SMEM_BYTES))
            return WD_ECUDA;
        using G = PGeo<LOGN, 256>;
        if (set_smem(ntt_persist_cc<LOGN, true, false, 256>, G::SMEM_BYTES) ||
            set_smem(ntt_persist_cc<LOGN, false, false, 256>, G::SMEM_BYTES) ||
            set_smem(ntt_persist_cc<LOGN, false, true, 256>, G::SMEM_BYTES))
            return WD_ECUDA;
    }
    return WD_OK;
}

int prepare_kernels(uint32_t logN) {
    switch (logN) {
        case 12: return prep_cc<12>();
        case 13: return prep_cc<13>();
        case 14: return prep_cc<14>();
        case 15: return prep_cc<15>();
        case 16: return prep_cc<16>();
        case 17: return prep_cc<17>();
        default:
            if (set_smem(ntt_small<true, false>, 4 << logN) || set_smem(ntt_small<false, false>, 4 << logN) ||
                set_smem(ntt_small<false, true>, 4 << logN))
                return WD_ECUDA;
            return WD_OK;
    }
}

constexpr int V8_DEFAULT_MINB = 4;   // measured, see DESIGN.md 5.1
constexpr int V8_DEFAULT_CL = 2;

// v8 with a CL-CTA cluster per row: grid = resident clusters x CL
template <int LOGN, int MINB, int CL, int EPI = 0>
void launch_v8_cluster(bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    if constexpr ((1 << (LOGN - 12)) % CL != 0) {
        return;
    } else {
        cudaLaunchConfig_t cfg = {};
        cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V8_SMEM; cfg.stream = s;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = CL; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
        cfg.attrs = at; cfg.numAttrs = 1;
        auto kf = ntt_v8<LOGN, true, false, 0, MINB, CL, EPI>;
        auto ki = ntt_v8<LOGN, false, false, 0, MINB, CL>;
        auto kp = ntt_v8<LOGN, false, true, 0, MINB, CL>;
        auto k = fwd ? kf : (a.in2 ? kp : ki);
        int ncl = 0;
        cfg.gridDim = dim3(148 * MINB / CL * CL);
        if (cudaOccupancyMaxActiveClusters(&ncl, k, &cfg) != cudaSuccess || ncl < 1) { cudaGetLastError(); ncl = 1; }
        cfg.gridDim = dim3(std::min<uint32_t>(rows, (uint32_t)ncl) * CL);
        cudaLaunchKernelEx(&cfg, k, a, rows);
    }
}

// v9 (ntt_v8.cuh): v8 with cp.async-staged column passes; grid = resident clusters x CL
template <int LOGN, int CL>
void launch_v9(bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    if constexpr (LOGN < 13 || LOGN > 16 || (1 << (LOGN - 12)) % CL != 0) {
        return;
    } else {
        cudaLaunchConfig_t cfg = {};
        cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V9_SMEM; cfg.stream = s;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = CL; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
        cfg.attrs = at; cfg.numAttrs = 1;
        auto k = fwd ? ntt_v9<LOGN, true, false, CL> : (a.in2 ? ntt_v9<LOGN, false, true, CL> : ntt_v9<LOGN, false, false, CL>);
        int ncl = 0;
        cfg.gridDim = dim3(148 * 4 / CL * CL);
        if (cudaOccupancyMaxActiveClusters(&ncl, k, &cfg) != cudaSuccess || ncl < 1) { cudaGetLastError(); ncl = 1; }
        cfg.gridDim = dim3(std::min<uint32_t>(rows, (uint32_t)ncl) * CL);
        cudaLaunchKernelEx(&cfg, k, a, rows);
    }
}

// v10 (ntt_v8.cuh, N = 2^16): v8 with the column phase on the tensor cores; 2-CTA cluster per row
template <int CL>
void launch_v10(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s);
void launch_v11(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s);

// v8 forward with an epilogue variant (EPI, ntt_rns.cuh), one CTA per row (N = 2^12)
template <int LOGN, int EPI>
void launch_v8_minb_epi(const NttArgs& a, uint32_t rows, int sm_count, cudaStream_t s) {
    const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)(sm_count * 4));
    ntt_v8<LOGN, true, false, 0, 4, 1, EPI><<<grid, V8_T, V8_SMEM, s>>>(a, rows);
}

// v8 (ntt_v8.cuh): persistent grid of min(rows, SMs x MINB) 256-thread CTAs
template <int LOGN, int MINB>
void launch_v8_minb(bool fwd, const NttArgs& a, uint32_t rows, int sm_count, cudaStream_t s) {
    const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)(sm_count * MINB));
    if (fwd) ntt_v8<LOGN, true, false, 0, MINB><<<grid, V8_T, V8_SMEM, s>>>(a, rows);
    else if (a.in2) ntt_v8<LOGN, false, true, 0, MINB><<<grid, V8_T, V8_SMEM, s>>>(a, rows);
    else ntt_v8<LOGN, false, false, 0, MINB><<<grid, V8_T, V8_SMEM, s>>>(a, rows);
}
template <int LOGN>
void launch_v8(int minb, bool fwd, const NttArgs& a, uint32_t rows, int sm_count, cudaStream_t s) {
    if (minb == 6) launch_v8_minb<LOGN, 6>(fwd, a, rows, sm_count, s);
    else if (minb == 5) launch_v8_minb<LOGN, 5>(fwd, a, rows, sm_count, s);
    else launch_v8_minb<LOGN, 4>(fwd, a, rows, sm_count, s);
}

template <int LOGN>
void launch_cc(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    using S = CcShape<LOGN>;
    if constexpr (LOGN >= 14) {
        // measured: a row split over a 4-CTA cluster (v5) wins only for a handful of rows; from
        // a quarter of the SM count up v8's 2-CTA clusters win (config 2, one ciphertext = 72
        // rows at N = 2^16: v8 2006 vs v5 1681 KOPS, profiles/r01/ab/)
        const bool small = p->kernel_ver == 0 && rows < (uint32_t)p->sm_count / 4 && (LOGN == 15 || LOGN == 16);
        if (p->kernel_ver == 5 || small) {
            constexpr int CLN = 1 << (LOGN - 14);
            const uint32_t units = std::max<uint32_t>(1, std::min<uint32_t>(rows, (uint32_t)(2 * p->sm_count / CLN)));
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(units * CLN); cfg.blockDim = dim3(CL_T); cfg.dynamicSmemBytes = CL_BYTES; cfg.stream = s;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = CLN; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
            cfg.attrs = at; cfg.numAttrs = 1;
            if (fwd) cudaLaunchKernelEx(&cfg, ntt_fwd_cl<LOGN>, a, rows);
            else if (a.in2) cudaLaunchKernelEx(&cfg, ntt_inv_cl<LOGN, true>, a, rows);
            else cudaLaunchKernelEx(&cfg, ntt_inv_cl<LOGN, false>, a, rows);
            return;
        }
    }
    if constexpr (LOGN >= 12) {
        if constexpr (LOGN == 15 || LOGN == 16) {
            if (fwd && p->kernel_ver == 12) {            // v12: phases of consecutive rows interleaved
                cudaLaunchConfig_t cfg = {};
                cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V12_SMEM; cfg.stream = s;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeClusterDimension;
                at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
                cfg.attrs = at; cfg.numAttrs = 1;
                int ncl = 0;
                cfg.gridDim = dim3(148 * 4);
                if (cudaOccupancyMaxActiveClusters(&ncl, ntt_v12f<LOGN>, &cfg) != cudaSuccess || ncl < 1) { cudaGetLastError(); ncl = 1; }
                cfg.gridDim = dim3(std::min<uint32_t>(rows, (uint32_t)ncl) * 2);
                cudaLaunchKernelEx(&cfg, ntt_v12f<LOGN>, a, rows);
                return;
            }
        }
        if (fwd && p->kernel_ver == 86) { ntt_v8<LOGN, true, false, 6><<<p->sm_count * 4, V8_T, V8_SMEM, s>>>(a, rows); return; }
        if (fwd && p->kernel_ver == 88) {   // v8 (2-CTA cluster) with the old per-thread 64-byte stores
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(p->sm_count * 4); cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V8_SMEM; cfg.stream = s;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
            cfg.attrs = at; cfg.numAttrs = 1;
            if constexpr (LOGN >= 13) cudaLaunchKernelEx(&cfg, ntt_v8<LOGN, true, false, 8, 4, 2>, a, rows);
            return;
        }
        if (p->kernel_ver == 89) {   // v8 (2-CTA cluster) with the column-pass prefetch (PF)
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(p->sm_count * 4); cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V8_SMEM; cfg.stream = s;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
            cfg.attrs = at; cfg.numAttrs = 1;
            if constexpr (LOGN >= 13) cudaLaunchKernelEx(&cfg, fwd ? ntt_v8<LOGN, true, false, 9, 4, 2> : ntt_v8<LOGN, false, false, 9, 4, 2>, a, rows);
            return;
        }
        if (fwd && p->kernel_ver == 87) { ntt_v8<LOGN, true, false, 7><<<p->sm_count * 4, V8_T, V8_SMEM, s>>>(a, rows); return; }
        if (fwd && p->kernel_ver >= 83 && p->kernel_ver <= 85) {   // timing experiments (ntt_v8 ONLY 3..5)
            if (p->kernel_ver == 83) ntt_v8<LOGN, true, false, 3><<<p->sm_count * 4, V8_T, V8_SMEM, s>>>(a, rows);
            else if (p->kernel_ver == 84) ntt_v8<LOGN, true, false, 4><<<p->sm_count * 4, V8_T, V8_SMEM, s>>>(a, rows);
            else ntt_v8<LOGN, true, false, 5><<<p->sm_count * 4, V8_T, V8_SMEM, s>>>(a, rows);
            return;
        }
        if (p->kernel_ver == 81 || p->kernel_ver == 82) {   // timing experiment: one phase of v8 only
            if (fwd && p->kernel_ver == 81) ntt_v8<LOGN, true, false, 1><<<p->sm_count * 4, V8_T, V8_SMEM, s>>>(a, rows);
            else if (fwd) ntt_v8<LOGN, true, false, 2><<<p->sm_count * 4, V8_T, V8_SMEM, s>>>(a, rows);
            else if (p->kernel_ver == 81) ntt_v8<LOGN, false, false, 1><<<p->sm_count * 4, V8_T, V8_SMEM, s>>>(a, rows);
            else ntt_v8<LOGN, false, false, 2><<<p->sm_count * 4, V8_T, V8_SMEM, s>>>(a, rows);
            return;
        }
        // AUTO at or above the SM count: v8 (see DESIGN.md 5.1 for the measured (CTAs/SM,
        // cluster) choice; WD_NTT_MINB / WD_NTT_CL override it for A/B runs)
        if constexpr (LOGN == 16) {
            if (p->kernel_ver == 11 && p->tc.ok && a.in2 == nullptr) {
                launch_v11(p, fwd, a, rows, s);
                return;
            }
            if (p->kernel_ver == 10 && p->tc.ok) {
                if ((p->v8_cl ? p->v8_cl : V8_DEFAULT_CL) >= 2) launch_v10<2>(p, fwd, a, rows, s);
                else launch_v10<1>(p, fwd, a, rows, s);
                return;
            }
        }
        if (p->kernel_ver == 9 && LOGN >= 13 && LOGN <= 16) {
            const int cl = (p->v8_cl ? p->v8_cl : V8_DEFAULT_CL) >= 2 && LOGN >= 13 ? 2 : 1;
            if (cl == 2) launch_v9<LOGN, 2>(fwd, a, rows, s);
            else launch_v9<LOGN, 1>(fwd, a, rows, s);
            return;
        }
        const bool autov8 = p->kernel_ver == 0 && (rows >= (uint32_t)p->sm_count ||
                                                   ((LOGN == 15 || LOGN == 16) && rows >= (uint32_t)p->sm_count / 4) ||
                                                   LOGN == 17);
        if (p->kernel_ver == 8 || p->kernel_ver == 12 || autov8) {
            int minb = p->v8_minb ? p->v8_minb : V8_DEFAULT_MINB;
            int cl = p->v8_cl ? p->v8_cl : V8_DEFAULT_CL;
            if (LOGN == 17 && fwd && !p->v8_minb) minb = 4;     // radix-32 column phase spills at 48 regs
            // few rows (<= half the SM count, e.g. one ciphertext at L = 36): 8-CTA clusters put
            // ~4 CTAs per SM to work on them (config 2: 2105 -> 2485 KOPS, profiles/r01/f4)
            if (!p->v8_cl && LOGN >= 15 && rows * 8 <= (uint32_t)p->sm_count * 4) cl = 8;
            // N = 2^13, 2^14 with many rows: the whole row per CTA (its 2^A x 4096 intermediate is
            // 32-64 KB, so 4 rows per SM stay L2-resident without the cluster split; s13 +8.6%,
            // s14 +3.7% over 2-CTA clusters; at 1024 rows the clusters still win)
            else if (!p->v8_cl && LOGN <= 14 && rows >= 8u * (uint32_t)p->sm_count) cl = 1;
            // between half and one SM count of rows: 4-CTA clusters (config 5 sweep)
            else if (!p->v8_cl && LOGN >= 15 && rows <= (uint32_t)p->sm_count) cl = 4;
            if ((1 << (LOGN - 12)) < cl || (cl == 8 && LOGN < 15)) cl = 1;
            if (cl == 1) launch_v8<LOGN>(minb, fwd, a, rows, p->sm_count, s);
            else if (cl == 2) {
                if (minb == 4) launch_v8_cluster<LOGN, 4, 2>(fwd, a, rows, s);
                else if (LOGN == 16 && minb == 3) { if constexpr (LOGN == 16) launch_v8_cluster<LOGN, 3, 2>(fwd, a, rows, s); }
                else launch_v8_cluster<LOGN, 5, 2>(fwd, a, rows, s);
            } else if (cl == 8) {
                if constexpr (LOGN >= 15) launch_v8_cluster<LOGN, 4, 8>(fwd, a, rows, s);
            } else {
                if (minb == 4) launch_v8_cluster<LOGN, 4, 4>(fwd, a, rows, s);
                else launch_v8_cluster<LOGN, 5, 4>(fwd, a, rows, s);
            }
            return;
        }
    }
    if constexpr (LOGN == 15 || LOGN == 16) {
        if (p->kernel_ver == 3) {
            constexpr int PAIR = LOGN == 16 ? 2 : 1;
            const uint32_t units = std::min<uint32_t>(rows, (uint32_t)(p->sm_count / PAIR));
            const uint32_t grid = units * PAIR;
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(grid); cfg.blockDim = dim3(SM_T); cfg.dynamicSmemBytes = SM_BYTES; cfg.stream = s;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = PAIR; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
            cfg.attrs = at; cfg.numAttrs = 1;
            if (fwd) cudaLaunchKernelEx(&cfg, ntt_fwd_smem<LOGN>, a, rows);
            else if (a.in2) cudaLaunchKernelEx(&cfg, ntt_inv_smem<LOGN, true>, a, rows);
            else cudaLaunchKernelEx(&cfg, ntt_inv_smem<LOGN, false>, a, rows);
            return;
        }
    }
    if constexpr (LOGN == 16 || LOGN == 17) {
        if (p->kernel_ver == 7) {   // v6 with 128-thread CTAs (barriers over 4 warps), up to 8 per SM
            using G = PGeo<LOGN, 128>;
            int occ = 1;
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ntt_persist_cc<LOGN, true, false, 128>, 128, G::SMEM_BYTES);
            const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)(p->sm_count * std::max(1, occ)));
            if (fwd) ntt_persist_cc<LOGN, true, false, 128><<<grid, 128, G::SMEM_BYTES, s>>>(a, rows);
            else if (a.in2) ntt_persist_cc<LOGN, false, true, 128><<<grid, 128, G::SMEM_BYTES, s>>>(a, rows);
            else ntt_persist_cc<LOGN, false, false, 128><<<grid, 128, G::SMEM_BYTES, s>>>(a, rows);
            return;
        }
        if (p->kernel_ver == 6 || p->kernel_ver == 0) {   // v2 with 256-thread CTAs, 4 (2^16) / 3 (2^17) per SM
            using G = PGeo<LOGN, 256>;
            int occ = 1;
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ntt_persist_cc<LOGN, true, false, 256>, 256, G::SMEM_BYTES);
            const int ctas = std::max(1, std::min(p->v6_ctas, occ));   // never a second, non-resident wave
            const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)(p->sm_count * ctas));
            if (fwd) ntt_persist_cc<LOGN, true, false, 256><<<grid, 256, G::SMEM_BYTES, s>>>(a, rows);
            else if (a.in2) ntt_persist_cc<LOGN, false, true, 256><<<grid, 256, G::SMEM_BYTES, s>>>(a, rows);
            else ntt_persist_cc<LOGN, false, false, 256><<<grid, 256, G::SMEM_BYTES, s>>>(a, rows);
            return;
        }
    }
    if constexpr (LOGN >= 15) {
        if (p->kernel_ver == 2) {
            using G = PGeo<LOGN>;
            int occ = 1;
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ntt_persist_cc<LOGN, true, false>, G::T, G::SMEM_BYTES);
            const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)(p->sm_count * std::max(occ, 1)));
            if (fwd) ntt_persist_cc<LOGN, true, false><<<grid, G::T, G::SMEM_BYTES, s>>>(a, rows);
            else if (a.in2) ntt_persist_cc<LOGN, false, true><<<grid, G::T, G::SMEM_BYTES, s>>>(a, rows);
            else ntt_persist_cc<LOGN, false, false><<<grid, G::T, G::SMEM_BYTES, s>>>(a, rows);
            return;
        }
    }
    if (fwd) ntt_fwd_cc<LOGN><<<rows, S::T, S::SMEM_BYTES, s>>>(a);
    else if (a.in2) ntt_inv_cc<LOGN, true><<<rows, S::T, S::SMEM_BYTES, s>>>(a);
    else ntt_inv_cc<LOGN, false><<<rows, S::T, S::SMEM_BYTES, s>>>(a);
}

template <int CL>
void launch_v10(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V10_SMEM; cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CL; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cfg.attrs = at; cfg.numAttrs = 1;
    auto k = fwd ? ntt_v10<true, false, CL> : (a.in2 ? ntt_v10<false, true, CL> : ntt_v10<false, false, CL>);
    // 4 CTAs per SM, each holding 128 of the SM's 512 TMEM columns.  (The occupancy API
    // reports 1 block/SM for this kernel; measured, 4 co-resident CTAs run: 1.48 -> 1.29 ms.)
    int ncl = p->sm_count * 4 / CL;
    if (const char* ev = getenv("WD_NTT_V10_CLUSTERS")) ncl = std::max(1, atoi(ev));
    if (getenv("WD_NTT_DEBUG")) {
        int occ = -1;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, V8_T, V10_SMEM);
        fprintf(stderr, "v10: clusters %d, blocks/SM %d\n", ncl, occ);
    }
    cfg.gridDim = dim3(std::min<uint32_t>(rows, (uint32_t)ncl) * CL);
    cudaLaunchKernelEx(&cfg, k, a, (const uint8_t*)p->tc.d_G, (const uint2*)p->tc.d_c16, rows);
}

// v11: which row-phase stages run on the tensor cores (bit st-1); WD_NTT_TMASK overrides
template <int TM>
void launch_v11_tm(const wd_ntt_plan* p, bool fwd, const V11Args& va, uint32_t rows, cudaStream_t s) {
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V11_SMEM; cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cfg.attrs = at; cfg.numAttrs = 1;
    cfg.gridDim = dim3(std::min<uint32_t>(rows, (uint32_t)(p->sm_count * 2)) * 2);   // 4 CTAs / SM (TMEM: 4 x 128)
    if (fwd) cudaLaunchKernelEx(&cfg, ntt_v11<true, TM>, va, rows);
    else cudaLaunchKernelEx(&cfg, ntt_v11<false, TM>, va, rows);
}
void launch_v11(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    V11Args va;
    va.a = a; va.G = p->tc.d_G; va.B = p->tc.d_B; va.c16 = p->tc.d_c16;
    va.t2 = fwd ? p->tc.d_tw2 : p->tc.d_sg2; va.t3 = fwd ? p->tc.d_tw3 : p->tc.d_sg3;
    int tm = 7;
    if (const char* ev = getenv("WD_NTT_TMASK")) tm = atoi(ev);
    switch (tm) {
        case 1: launch_v11_tm<1>(p, fwd, va, rows, s); break;
        case 3: launch_v11_tm<3>(p, fwd, va, rows, s); break;
        case 6: launch_v11_tm<6>(p, fwd, va, rows, s); break;
        default: launch_v11_tm<7>(p, fwd, va, rows, s); break;
    }
}

int launch_cuda_core(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    switch (p->logN) {
        case 12: launch_cc<12>(p, fwd, a, rows, s); break;
        case 13: launch_cc<13>(p, fwd, a, rows, s); break;
        case 14: launch_cc<14>(p, fwd, a, rows, s); break;
        case 15: launch_cc<15>(p, fwd, a, rows, s); break;
        case 16: launch_cc<16>(p, fwd, a, rows, s); break;
        case 17: launch_cc<17>(p, fwd, a, rows, s); break;
        default: {
            const int thr = std::min<int>(256, std::max<int>(32, (int)p->N / 2));
            if (fwd) ntt_small<true, false><<<rows, thr, 4 << p->logN, s>>>(a, (int)p->logN);
            else if (a.in2) ntt_small<false, true><<<rows, thr, 4 << p->logN, s>>>(a, (int)p->logN);
            else ntt_small<false, false><<<rows, thr, 4 << p->logN, s>>>(a, (int)p->logN);
        }
    }
    return 1;
}

// WD-CUDA (row f2): the four radix-16 inner DFTs as 32-bit GEMMs on the CUDA cores, N = 2^16
int launch_wdcuda(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    WdcArgs wa;
    wa.a = a; wa.mat = p->tc.d_mat;
    wa.t1 = fwd ? p->tc.d_tw1 : p->tc.d_sg1; wa.t2 = fwd ? p->tc.d_tw2 : p->tc.d_sg2; wa.t3 = fwd ? p->tc.d_tw3 : p->tc.d_sg3;
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(V8_T); cfg.dynamicSmemBytes = V8_SMEM + 2048; cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cfg.attrs = at; cfg.numAttrs = 1;
    cfg.gridDim = dim3(std::min<uint32_t>(rows, (uint32_t)(p->sm_count * 3 / 2)) * 2);
    if (fwd) cudaLaunchKernelEx(&cfg, ntt_wdcuda16<true>, wa, rows);
    else cudaLaunchKernelEx(&cfg, ntt_wdcuda16<false>, wa, rows);
    return 1;
}

int effective_mode(const wd_ntt_plan* p) {
    if (p->mode != WD_MODE_AUTO) return p->mode;
    return WD_MODE_CUDA;
}

int run(const wd_ntt_plan* p, bool fwd, const uint32_t* in, const uint32_t* in2, uint32_t* out,
        uint32_t batch, cudaStream_t s) {
    g_last_launches = 0;
    if (!p || !in || !out || (in2 == nullptr && false)) return set_err(WD_EINVAL);
    if (((uintptr_t)in | (uintptr_t)out | (uintptr_t)in2) & 15) return set_err(WD_EINVAL);
    if (batch == 0) return set_err(WD_OK);
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != p->device) return set_err(WD_EINVAL);
    const uint64_t rows64 = (uint64_t)batch * p->L;
    if (rows64 > 0x7fffffffull) return set_err(WD_EINVAL);
    const uint32_t rows = (uint32_t)rows64;
    NttArgs a;
    a.in = in; a.in2 = in2; a.out = out; a.tw = fwd ? p->d_fwd : p->d_inv; a.lc = p->d_lc; a.L = p->L;
    a.stagger_ns = p->stagger_ns;
    a.limb_major = p->limb_major;
    const int mode = effective_mode(p);
    int launches = 0;
    if (mode == WD_MODE_CUDA_GEMM && in2 == nullptr && p->logN == 16 && p->tc.ok) {
        launches = launch_wdcuda(p, fwd, a, rows, s);
    } else if (mode == WD_MODE_FTC && in2 == nullptr && p->logN == 16 && p->tc.ok) {
        // WD-FTC: split at a polynomial boundary (rows stay limb-aligned), WD-Tensor on the
        // first bt polynomials in a forked stream, WD-CUDA on the rest in `s`, then join.
        const uint32_t bt = std::min<uint32_t>(batch, (uint32_t)std::lround(p->ftc_share * batch));
        NttArgs ac = a;
        const size_t off = (size_t)bt * p->L * p->N;
        ac.in = a.in + off; ac.out = a.out + off;
        if (bt == 0) {
            launches = launch_wdcuda(p, fwd, ac, rows, s);
        } else if (bt == batch) {
            launches = launch_tensor(p->logN, fwd, a, p->tc, rows, p->sm_count, s);
        } else {
            std::lock_guard<std::mutex> lk(p->ftc_mu);
            cudaEventRecord(p->fe[0], s);
            cudaStreamWaitEvent(p->fs, p->fe[0], 0);
            const int n1 = launch_tensor(p->logN, fwd, a, p->tc, bt * p->L, p->sm_count, p->fs);
            const int n2 = launch_wdcuda(p, fwd, ac, (batch - bt) * p->L, s);
            cudaEventRecord(p->fe[1], p->fs);
            cudaStreamWaitEvent(s, p->fe[1], 0);
            launches = n1 + n2;
        }
        if (launches < 0) return set_err(WD_EUNSUPPORTED);
    } else if (mode == WD_MODE_CUDA || mode == WD_MODE_CUDA_GEMM || in2 != nullptr || !tensor_supported(p->logN)) {
        if (mode != WD_MODE_CUDA && in2 == nullptr && mode != WD_MODE_AUTO) return set_err(WD_EUNSUPPORTED);
        launches = launch_cuda_core(p, fwd, a, rows, s);
    } else {
        if (mode == WD_MODE_TENSOR) launches = launch_tensor(p->logN, fwd, a, p->tc, rows, p->sm_count, s);
        else launches = launch_fused(p->logN, fwd, a, p->tc, rows, p->sm_count, p->tensor_share, s);
        if (launches < 0) return set_err(WD_EUNSUPPORTED);
    }
    if (cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    g_last_launches = (uint32_t)launches;
    return set_err(WD_OK);
}

int run_host(const wd_ntt_plan* pc, bool fwd, const uint32_t* h_in, uint32_t* h_out, uint32_t batch,
             uint32_t* d_work, cudaStream_t s) {
    if (!pc || !h_in || !h_out || !d_work || ((uintptr_t)d_work & 15)) return set_err(WD_EINVAL);
    if (batch == 0) return set_err(WD_OK);
    wd_ntt_plan* p = const_cast<wd_ntt_plan*>(pc);
    std::lock_guard<std::mutex> lk(p->host_mu);
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != p->device) return set_err(WD_EINVAL);
    const size_t row_words = (size_t)p->L * p->N;
    // chunks of >= 1 polynomial: H2D(k+1) || kernel(k) || D2H(k-1).  The first H2D and the
    // last D2H are not overlapped, so a call costs ~(nch+1)/nch of one copy direction: 8 chunks
    // for small jobs, up to 32 chunks of ~32 MB for large ones.
    const size_t total_bytes = (size_t)batch * row_words * 4;
    const uint32_t want = (uint32_t)std::min<size_t>(32, std::max<size_t>(8, total_bytes >> 25));
    const uint32_t nch = std::min<uint32_t>(batch, want);
    cudaEventRecord(p->he[3], s);
    uint32_t total = 0;
    uint32_t b0 = 0;
    for (uint32_t k = 0; k < nch; ++k) {
        const uint32_t b1 = (uint32_t)((uint64_t)batch * (k + 1) / nch);
        const uint32_t nb = b1 - b0;
        cudaStream_t st = p->hs[k % 3];
        if (k < 3) cudaStreamWaitEvent(st, p->he[3], 0);
        const size_t off = (size_t)b0 * row_words, bytes = (size_t)nb * row_words * 4;
        cudaMemcpyAsync(d_work + off, h_in + off, bytes, cudaMemcpyHostToDevice, st);
        int e = run(p, fwd, d_work + off, nullptr, d_work + off, nb, st);
        if (e) return e;
        total += g_last_launches;
        cudaMemcpyAsync(h_out + off, d_work + off, bytes, cudaMemcpyDeviceToHost, st);
        b0 = b1;
    }
    for (int i = 0; i < 3; ++i) {
        cudaEventRecord(p->he[i], p->hs[i]);
        cudaStreamWaitEvent(s, p->he[i], 0);
    }
    g_last_launches = total;
    if (cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    return set_err(WD_OK);
}

void free_plan(wd_ntt_plan* p) {
    if (!p) return;
    if (p->device >= 0) {
        int cur = -1;
        cudaGetDevice(&cur);
        if (cur != p->device) cudaSetDevice(p->device);
        cudaFree(p->d_fwd); cudaFree(p->d_inv); cudaFree(p->d_lc); cudaFree(p->d_rs);
        free_tensor_tables(p->tc);
        for (auto& s : p->hs) if (s) cudaStreamDestroy(s);
        for (auto& e : p->he) if (e) cudaEventDestroy(e);
        if (p->fs) cudaStreamDestroy(p->fs);
        for (auto& e : p->fe) if (e) cudaEventDestroy(e);
        if (cur >= 0 && cur != p->device) cudaSetDevice(cur);
    }
    delete p;
}

}  // namespace

// ---------------------------------------------------------------- ModUp / ModDown (row f3)
struct wd_rns_conv {
    const wd_ntt_plan* pq = nullptr;   // Q basis (a limbs)
    const wd_ntt_plan* pp = nullptr;   // P basis (k special limbs)
    uint4* d_up_src = nullptr; uint2* d_up_w = nullptr; uint4* d_up_dst = nullptr;      // BConv Q -> P
    uint4* d_dn_src = nullptr; uint2* d_dn_w = nullptr; uint4* d_dn_dst = nullptr;      // BConv P -> Q
    uint4* d_pinv = nullptr;           // [a] {0, 0, P^-1 mod q_i, Shoup} (EPI = 2 store map)
    bool sharded = false;              // Q-limb shard: Q -> P tables use the whole Q (wd_modup_partial)
};

namespace {

void free_conv(wd_rns_conv* c) {
    if (!c) return;
    cudaFree(c->d_up_src); cudaFree(c->d_up_w); cudaFree(c->d_up_dst);
    cudaFree(c->d_dn_src); cudaFree(c->d_dn_w); cudaFree(c->d_dn_dst); cudaFree(c->d_pinv);
    delete c;
}

// host tables of BConv src -> dst: {q_i, (Q/q_i)^-1, Shoup}, (Q/q_i) mod p_j, {p_j, mu}
// Q = product of `all` (the whole source basis; `src` is the subset this table converts --
// all of it, or one limb shard of it for the sharded ModUp)
void bconv_tables(const std::vector<uint32_t>& src, const std::vector<uint32_t>& dst, std::vector<uint4>& hs,
                  std::vector<uint2>& hw, std::vector<uint4>& hd, const std::vector<uint32_t>* all_src = nullptr) {
    const std::vector<uint32_t>& all = all_src ? *all_src : src;
    const size_t S = src.size(), D = dst.size();
    hs.resize(S); hw.resize(S * D); hd.resize(D);
    for (size_t i = 0; i < S; ++i) {
        uint32_t qh = 1;                                   // (Q/q_i) mod q_i
        for (uint32_t qk : all) if (qk != src[i]) qh = pm_mul(qh, qk % src[i], src[i]);
        const uint32_t inv = pm_pow(qh, src[i] - 2, src[i]);
        hs[i] = make_uint4(src[i], inv, pm_shoup(inv, src[i]), 0);
        for (size_t j = 0; j < D; ++j) {
            uint32_t v = 1;
            for (uint32_t qk : all) if (qk != src[i]) v = pm_mul(v, qk % dst[j], dst[j]);
            hw[i * D + j] = make_uint2(v, pm_shoup(v, dst[j]));
        }
    }
    for (size_t j = 0; j < D; ++j) {
        const uint64_t mu = ~0ull / dst[j];
        hd[j] = make_uint4(dst[j], (uint32_t)mu, (uint32_t)(mu >> 32), 0);
    }
}

template <typename T>
bool upload(T** d, const std::vector<T>& h) {
    if (cudaMalloc(d, sizeof(T) * h.size()) != cudaSuccess) return false;
    return cudaMemcpy(*d, h.data(), sizeof(T) * h.size(), cudaMemcpyHostToDevice) == cudaSuccess;
}

// v8 launch over `rows` rows of `a` (any direction / EPI), default shape for N
template <int EPI>
void launch_v8_rows(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    switch (p->logN) {
        case 12:
            if (fwd) launch_v8_minb_epi<12, EPI>(a, rows, p->sm_count, s);
            else launch_v8<12>(4, false, a, rows, p->sm_count, s);
            break;
        case 13: launch_v8_cluster<13, 4, 2, EPI>(fwd, a, rows, s); break;
        case 14: launch_v8_cluster<14, 4, 2, EPI>(fwd, a, rows, s); break;
        case 15: launch_v8_cluster<15, 4, 2, EPI>(fwd, a, rows, s); break;
        case 16: launch_v8_cluster<16, 4, 2, EPI>(fwd, a, rows, s); break;
        default: launch_v8_cluster<17, 4, 2, EPI>(fwd, a, rows, s); break;
    }
}

int launch_bconv(const wd_ntt_plan* p, const uint32_t* x, uint32_t x_ls, uint32_t* y, uint32_t y_ls, uint32_t y_off,
                 const BconvTab& t, uint32_t batch, cudaStream_t s) {
    if (t.D <= 4 && t.S > 4 && p->N >= (uint32_t)BCF_C) {   // few targets: register accumulation
        const size_t sm = sizeof(uint4) * (t.S + t.D) + sizeof(uint2) * t.S * t.D;
        const uint32_t blocks = (uint32_t)std::min<uint64_t>((uint64_t)batch * (p->N / BCF_C), (uint64_t)p->sm_count * 8);
        switch (t.D) {
            case 1: rns_bconv_few<1><<<blocks, BC_T, sm, s>>>(x, x_ls, y, y_ls, y_off, t, p->N, batch); break;
            case 2: rns_bconv_few<2><<<blocks, BC_T, sm, s>>>(x, x_ls, y, y_ls, y_off, t, p->N, batch); break;
            case 3: rns_bconv_few<3><<<blocks, BC_T, sm, s>>>(x, x_ls, y, y_ls, y_off, t, p->N, batch); break;
            default: rns_bconv_few<4><<<blocks, BC_T, sm, s>>>(x, x_ls, y, y_ls, y_off, t, p->N, batch); break;
        }
        return WD_OK;
    }
    if (t.S <= 4 && p->N >= (uint32_t)BCF_C) {         // few sources: terms in registers, 16-B stores
        const size_t sm = sizeof(uint4) * (t.S + t.D) + sizeof(uint2) * t.S * t.D;
        const uint32_t blocks = (uint32_t)std::min<uint64_t>((uint64_t)batch * (p->N / BCF_C), (uint64_t)p->sm_count * 8);
        switch (t.S) {
            case 1: rns_bconv_fewsrc<1><<<blocks, BC_T, sm, s>>>(x, x_ls, y, y_ls, y_off, t, p->N, batch); break;
            case 2: rns_bconv_fewsrc<2><<<blocks, BC_T, sm, s>>>(x, x_ls, y, y_ls, y_off, t, p->N, batch); break;
            case 3: rns_bconv_fewsrc<3><<<blocks, BC_T, sm, s>>>(x, x_ls, y, y_ls, y_off, t, p->N, batch); break;
            default: rns_bconv_fewsrc<4><<<blocks, BC_T, sm, s>>>(x, x_ls, y, y_ls, y_off, t, p->N, batch); break;
        }
        return WD_OK;
    }
    const size_t smem = sizeof(uint4) * (t.S + t.D) + sizeof(uint2) * t.S * t.D + sizeof(uint32_t) * t.S * BC_T;
    if (smem > 48 * 1024 && cudaFuncSetAttribute(rns_bconv, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
        return WD_ECUDA;
    const uint32_t blocks = (uint32_t)std::min<uint64_t>((uint64_t)batch * (p->N / BC_T), (uint64_t)p->sm_count * 8);
    rns_bconv<<<blocks, BC_T, smem, s>>>(x, x_ls, y, y_ls, y_off, t, p->N, batch);
    return WD_OK;
}

}  // namespace

extern "C" {

wd_ntt_plan* wd_ntt_plan_create(uint32_t N, const uint32_t* primes, uint32_t L) {
    if (!primes) { set_err(WD_EINVAL); return nullptr; }
    if (!is_pow2(N) || N < 2 || N > (1u << 17) || L == 0 || L > 4096) { set_err(WD_EUNSUPPORTED); return nullptr; }
    for (uint32_t l = 0; l < L; ++l)
        if (check_prime(primes[l], N)) { set_err(WD_EPRIME); return nullptr; }

    wd_ntt_plan* p = new (std::nothrow) wd_ntt_plan();
    if (!p) { set_err(WD_ENOMEM); return nullptr; }
    p->N = N; p->logN = ilog2u(N); p->L = L;
    p->primes.assign(primes, primes + L);

    // ---- host precompute (a1): psi, bit-reversed psi-power tables + Shoup companions
    std::vector<uint2> fwd((size_t)L * N), inv((size_t)L * N);
    std::vector<LimbConst> lc(L);
    for (uint32_t l = 0; l < L; ++l) {
        const uint32_t q = primes[l];
        const uint32_t psi = plan_psi_min(q, N);
        const uint32_t psi_inv = pm_pow(psi, q - 2, q);
        p->psi.push_back(psi);
        std::vector<uint32_t> pw(N), pwi(N);
        pw[0] = 1; pwi[0] = 1;
        for (uint32_t i = 1; i < N; ++i) { pw[i] = pm_mul(pw[i - 1], psi, q); pwi[i] = pm_mul(pwi[i - 1], psi_inv, q); }
        uint2* f = fwd.data() + (size_t)l * N;
        uint2* v = inv.data() + (size_t)l * N;
        for (uint32_t i = 0; i < N; ++i) {
            const uint32_t e = pm_brv(i, (int)p->logN);
            f[i] = make_uint2(pw[e], pm_shoup(pw[e], q));
            v[i] = make_uint2(pwi[e], pm_shoup(pwi[e], q));
        }
        LimbConst& c = lc[l];
        c.q = q; c.q2 = 2 * q;
        c.ninv = pm_pow(N % q, q - 2, q); c.ninv_sh = pm_shoup(c.ninv, q);
        c.wn = pm_mul(N > 1 ? v[1].x : 1, c.ninv, q); c.wn_sh = pm_shoup(c.wn, q);
        c.mu = ~0ull / q;
        {
            uint32_t qi = q;                              // Newton: q * qi = 1 (mod 2^32)
            for (int it = 0; it < 5; ++it) qi *= 2u - q * qi;
            c.qinv = qi;
            const uint32_t r = (uint32_t)((1ull << 32) % q);
            c.ninv_r = pm_mul(c.ninv, r, q); c.ninv_r_sh = pm_shoup(c.ninv_r, q);
            c.wn_r = pm_mul(c.wn, r, q); c.wn_r_sh = pm_shoup(c.wn_r, q);
            c.pad_[0] = c.pad_[1] = c.pad_[2] = 0;
        }
    }

    // ---- device upload (the only H2D copy of the plan's life)
    if (cudaGetDevice(&p->device) != cudaSuccess) { cudaGetLastError(); p->device = -1; delete p; set_err(WD_ECUDA); return nullptr; }
    cudaDeviceGetAttribute(&p->sm_count, cudaDevAttrMultiProcessorCount, p->device);
    p->kernel_ver = 0;   // AUTO: v8 at >= SM-count rows; below: v5 (2^15, 2^16), v6 (2^17), v1 (<= 2^14)
    if (const char* ev = getenv("WD_NTT_CTAS")) p->v6_ctas = std::max(1, std::min(4, atoi(ev)));
    if (const char* ev = getenv("WD_NTT_MINB")) p->v8_minb = std::max(3, std::min(6, atoi(ev)));
    if (const char* ev = getenv("WD_NTT_CL")) p->v8_cl = atoi(ev) >= 8 ? 8 : atoi(ev) >= 4 ? 4 : atoi(ev) >= 2 ? 2 : 1;
    if (const char* ev = getenv("WD_NTT_STAGGER")) p->stagger_ns = (uint32_t)atoi(ev);
    if (const char* ev = getenv("WD_NTT_LM")) p->limb_major = atoi(ev) != 0;
    if (const char* ev = getenv("WD_NTT_KERNEL")) p->kernel_ver = ev[0] == 'v' ? atoi(ev + 1) : p->kernel_ver;
    const size_t tb = sizeof(uint2) * (size_t)L * N;
    if (cudaMalloc(&p->d_fwd, tb) != cudaSuccess || cudaMalloc(&p->d_inv, tb) != cudaSuccess ||
        cudaMalloc(&p->d_lc, sizeof(LimbConst) * L) != cudaSuccess) {
        cudaGetLastError(); free_plan(p); set_err(WD_ENOMEM); return nullptr;
    }
    if (cudaMemcpy(p->d_fwd, fwd.data(), tb, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(p->d_inv, inv.data(), tb, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(p->d_lc, lc.data(), sizeof(LimbConst) * L, cudaMemcpyHostToDevice) != cudaSuccess) {
        cudaGetLastError(); free_plan(p); set_err(WD_ECUDA); return nullptr;
    }
    // RESCALE constants (row f4): per limb i < L-1 {-q_last mod q_i, Shoup(1), q_last^-1 mod q_i, Shoup}
    if (L >= 2) {
        const uint32_t ql = primes[L - 1];
        std::vector<uint4> rs(L, make_uint4(0, 0, 0, 0));
        p->rs_ok = true;
        for (uint32_t i = 0; i + 1 < L; ++i) {
            const uint32_t q = primes[i];
            if (q == ql) { p->rs_ok = false; break; }
            const uint32_t inv = pm_pow(ql % q, q - 2, q);
            rs[i] = make_uint4((q - ql % q) % q, pm_shoup(1, q), inv, pm_shoup(inv, q));
        }
        p->rs_thr = ql - ql / 2;
        if (p->rs_ok && (cudaMalloc(&p->d_rs, sizeof(uint4) * L) != cudaSuccess ||
                         cudaMemcpy(p->d_rs, rs.data(), sizeof(uint4) * L, cudaMemcpyHostToDevice) != cudaSuccess)) {
            cudaGetLastError(); free_plan(p); set_err(WD_ENOMEM); return nullptr;
        }
    }
    if (build_tensor_tables(p->tc, p->logN, p->primes, p->psi) != WD_OK) {
        cudaGetLastError(); free_plan(p); set_err(WD_ECUDA); return nullptr;
    }
    for (auto& s : p->hs) if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess) { free_plan(p); set_err(WD_ECUDA); return nullptr; }
    for (auto& e : p->he) if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) { free_plan(p); set_err(WD_ECUDA); return nullptr; }
    if (cudaStreamCreateWithFlags(&p->fs, cudaStreamNonBlocking) != cudaSuccess) { free_plan(p); set_err(WD_ECUDA); return nullptr; }
    for (auto& e : p->fe) if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) { free_plan(p); set_err(WD_ECUDA); return nullptr; }
    if (prepare_kernels(p->logN) != WD_OK || prepare_tensor_kernels(p->logN) != WD_OK ||
        prepare_fused_kernels(p->logN) != WD_OK) {
        cudaGetLastError(); free_plan(p); set_err(WD_ECUDA); return nullptr;
    }
    p->mode = WD_MODE_AUTO;
    p->tensor_share = default_tensor_share(p->logN);
    set_err(WD_OK);
    return p;
}

void wd_ntt_plan_destroy(wd_ntt_plan* plan) { free_plan(plan); }

int wd_ntt_forward(const wd_ntt_plan* p, const uint32_t* in, uint32_t* out, uint32_t batch, wd_stream_t s) {
    if (!in) return set_err(WD_EINVAL);
    return run(p, true, in, nullptr, out, batch, (cudaStream_t)s);
}
int wd_ntt_inverse(const wd_ntt_plan* p, const uint32_t* in, uint32_t* out, uint32_t batch, wd_stream_t s) {
    if (!in) return set_err(WD_EINVAL);
    return run(p, false, in, nullptr, out, batch, (cudaStream_t)s);
}
int wd_ntt_pointwise_inverse(const wd_ntt_plan* p, const uint32_t* a, const uint32_t* b, uint32_t* out,
                             uint32_t batch, wd_stream_t s) {
    if (!a || !b) return set_err(WD_EINVAL);
    return run(p, false, a, b, out, batch, (cudaStream_t)s);
}
int wd_rescale(const wd_ntt_plan* p, const uint32_t* in, uint32_t* out, uint32_t batch, uint32_t* work,
               wd_stream_t st) {
    g_last_launches = 0;
    if (!p || !in || !out || !work) return set_err(WD_EINVAL);
    if (((uintptr_t)in | (uintptr_t)out | (uintptr_t)work) & 15) return set_err(WD_EINVAL);
    if (p->L < 2 || p->logN < 12 || !p->rs_ok) return set_err(WD_EUNSUPPORTED);
    if (batch == 0) return set_err(WD_OK);
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != p->device) return set_err(WD_EINVAL);
    if ((uint64_t)batch * p->L > 0x7fffffffull) return set_err(WD_EINVAL);
    cudaStream_t s = (cudaStream_t)st;
    const uint32_t N = p->N, L = p->L;
    // K1: last-limb rows -> work
    {
        const uint32_t n4 = N / 4;
        const uint32_t blocks = (uint32_t)std::min<uint64_t>(((uint64_t)batch * n4 + 255) / 256, (uint64_t)p->sm_count * 8);
        rs_gather<<<blocks, 256, 0, s>>>(reinterpret_cast<const uint4*>(in), reinterpret_cast<uint4*>(work), n4, L, batch);
    }
    // K2: INTT of the last limb (a 1-limb view of the plan's tables), in place in work
    NttArgs ai;
    ai.in = work; ai.in2 = nullptr; ai.out = work; ai.tw = p->d_inv + (size_t)(L - 1) * N; ai.lc = p->d_lc + (L - 1); ai.L = 1;
    uint32_t launches = 1 + (uint32_t)launch_cuda_core(p, false, ai, batch, s);
    // K3: forward NTT of every output row with the rescale load / store maps (v8, EPI = 1)
    NttArgs af;
    af.in = work; af.in2 = nullptr; af.out = out; af.tw = p->d_fwd; af.lc = p->d_lc; af.L = L - 1;
    af.aux = in; af.rs = p->d_rs; af.rs_thr = p->rs_thr; af.Lfull = L;
    const uint32_t rows = batch * (L - 1);
    switch (p->logN) {
        case 12: launch_v8_minb_epi<12, 1>(af, rows, p->sm_count, s); break;
        case 13: launch_v8_cluster<13, 4, 2, 1>(true, af, rows, s); break;
        case 14: launch_v8_cluster<14, 4, 2, 1>(true, af, rows, s); break;
        case 15: launch_v8_cluster<15, 4, 2, 1>(true, af, rows, s); break;
        case 16: launch_v8_cluster<16, 4, 2, 1>(true, af, rows, s); break;
        default: launch_v8_cluster<17, 4, 2, 1>(true, af, rows, s); break;
    }
    launches += 1;
    if (cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    g_last_launches = launches;
    return set_err(WD_OK);
}

wd_rns_conv* wd_rns_conv_create_shard(const wd_ntt_plan* pq, const wd_ntt_plan* pp, const uint32_t* q_all,
                                      uint32_t a_all);

wd_rns_conv* wd_rns_conv_create(const wd_ntt_plan* pq, const wd_ntt_plan* pp) {
    if (!pq) { set_err(WD_EINVAL); return nullptr; }
    return wd_rns_conv_create_shard(pq, pp, pq->primes.data(), pq->L);
}

wd_rns_conv* wd_rns_conv_create_shard(const wd_ntt_plan* pq, const wd_ntt_plan* pp, const uint32_t* q_all,
                                      uint32_t a_all) {
    if (!pq || !pp) { set_err(WD_EINVAL); return nullptr; }
    if (!q_all || a_all < pq->L || a_all > 4096) { set_err(WD_EINVAL); return nullptr; }
    if (pq->N != pp->N || pq->device != pp->device || pq->logN < 12 || pq->L > BC_MAX || pp->L > BC_MAX) {
        set_err(WD_EUNSUPPORTED); return nullptr;
    }
    std::vector<uint32_t> all(q_all, q_all + a_all);
    for (uint32_t a : pq->primes)                          // the local limbs must be part of Q
        if (std::find(all.begin(), all.end(), a) == all.end()) { set_err(WD_EINVAL); return nullptr; }
    for (size_t i = 0; i < all.size(); ++i)
        for (size_t k = i + 1; k < all.size(); ++k) if (all[i] == all[k]) { set_err(WD_EINVAL); return nullptr; }
    for (uint32_t a : all)
        for (uint32_t b : pp->primes) if (a == b) { set_err(WD_EINVAL); return nullptr; }
    for (uint32_t a : pq->primes) {
        for (uint32_t b : pp->primes) if (a == b) { set_err(WD_EINVAL); return nullptr; }
    }
    for (size_t i = 0; i < pq->primes.size(); ++i)
        for (size_t k = i + 1; k < pq->primes.size(); ++k) if (pq->primes[i] == pq->primes[k]) { set_err(WD_EINVAL); return nullptr; }
    for (size_t i = 0; i < pp->primes.size(); ++i)
        for (size_t k = i + 1; k < pp->primes.size(); ++k) if (pp->primes[i] == pp->primes[k]) { set_err(WD_EINVAL); return nullptr; }
    wd_rns_conv* c = new (std::nothrow) wd_rns_conv();
    if (!c) { set_err(WD_ENOMEM); return nullptr; }
    c->pq = pq; c->pp = pp;
    std::vector<uint4> hs, hd, pinv(pq->L);
    std::vector<uint2> hw;
    bool ok = true;
    bconv_tables(pq->primes, pp->primes, hs, hw, hd, &all);
    ok = ok && upload(&c->d_up_src, hs) && upload(&c->d_up_w, hw) && upload(&c->d_up_dst, hd);
    c->sharded = a_all != pq->L;
    bconv_tables(pp->primes, pq->primes, hs, hw, hd);
    ok = ok && upload(&c->d_dn_src, hs) && upload(&c->d_dn_w, hw) && upload(&c->d_dn_dst, hd);
    for (uint32_t i = 0; i < pq->L; ++i) {
        const uint32_t q = pq->primes[i];
        uint32_t P = 1;
        for (uint32_t pj : pp->primes) P = pm_mul(P, pj % q, q);
        const uint32_t inv = pm_pow(P, q - 2, q);
        pinv[i] = make_uint4(0, 0, inv, pm_shoup(inv, q));
    }
    ok = ok && upload(&c->d_pinv, pinv);
    if (!ok) { cudaGetLastError(); free_conv(c); set_err(WD_ENOMEM); return nullptr; }
    set_err(WD_OK);
    return c;
}

void wd_rns_conv_destroy(wd_rns_conv* c) { free_conv(c); }

int wd_modup(const wd_rns_conv* c, const uint32_t* in, uint32_t* out, uint32_t batch, uint32_t* work, wd_stream_t st) {
    g_last_launches = 0;
    if (!c || !in || !out || !work) return set_err(WD_EINVAL);
    if (((uintptr_t)in | (uintptr_t)out | (uintptr_t)work) & 15) return set_err(WD_EINVAL);
    if (batch == 0) return set_err(WD_OK);
    const wd_ntt_plan *pq = c->pq, *pp = c->pp;
    if (c->sharded) return set_err(WD_EINVAL);             // a shard needs wd_modup_partial + all-reduce
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != pq->device) return set_err(WD_EINVAL);
    if ((uint64_t)batch * (pq->L + pp->L) > 0x7fffffffull) return set_err(WD_EINVAL);
    cudaStream_t s = (cudaStream_t)st;
    const uint32_t N = pq->N, a = pq->L, k = pp->L;
    // K1: INTT of the Q limbs -> work [batch][a][N]
    NttArgs ai;
    ai.in = in; ai.in2 = nullptr; ai.out = work; ai.tw = pq->d_inv; ai.lc = pq->d_lc; ai.L = a;
    uint32_t launches;
    if (pq->logN >= 12 && pq->kernel_ver == 0) {
        // v8 copies the Q limbs (NTT domain, unchanged) into out as it stages them: one read of
        // the input instead of two (the separate 2-D copy cost ~0.4 ms at config 3)
        ai.cpy = out; ai.cpy_ls = a + k;
        launch_v8_rows<0>(pq, false, ai, batch * a, s);
        launches = 1;
    } else {
        launches = (uint32_t)launch_cuda_core(pq, false, ai, batch * a, s);
        // the Q limbs pass through unchanged (NTT domain)
        if (cudaMemcpy2DAsync(out, (size_t)(a + k) * N * 4, in, (size_t)a * N * 4, (size_t)a * N * 4, batch,
                              cudaMemcpyDeviceToDevice, s) != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    }
    // K2: BConv Q -> P into the P section of out (coefficient domain)
    BconvTab t{c->d_up_src, c->d_up_w, c->d_up_dst, a, k};
    if (launch_bconv(pq, work, a, out, a + k, a, t, batch, s) != WD_OK) return set_err(WD_ECUDA);
    // K3: forward NTT of the P section in place (rows strided by a + k)
    NttArgs af;
    af.in = out + (size_t)a * N; af.in2 = nullptr; af.out = out + (size_t)a * N; af.tw = pp->d_fwd; af.lc = pp->d_lc;
    af.L = k; af.in_ls = a + k; af.out_ls = a + k;
    launch_v8_rows<0>(pp, true, af, batch * k, s);
    launches += 2;
    if (cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    g_last_launches = launches;
    return set_err(WD_OK);
}

int wd_modup_partial(const wd_rns_conv* c, const uint32_t* in, uint64_t* partial, uint32_t batch,
                     uint32_t* work, wd_stream_t st) {
    g_last_launches = 0;
    if (!c || !in || !partial || !work) return set_err(WD_EINVAL);
    if (((uintptr_t)in | (uintptr_t)partial | (uintptr_t)work) & 15) return set_err(WD_EINVAL);
    if (batch == 0) return set_err(WD_OK);
    const wd_ntt_plan *pq = c->pq, *pp = c->pp;
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != pq->device) return set_err(WD_EINVAL);
    if ((uint64_t)batch * (pq->L + pp->L) > 0x7fffffffull) return set_err(WD_EINVAL);
    cudaStream_t s = (cudaStream_t)st;
    const uint32_t a = pq->L, k = pp->L;
    NttArgs ai;
    ai.in = in; ai.in2 = nullptr; ai.out = work; ai.tw = pq->d_inv; ai.lc = pq->d_lc; ai.L = a;
    uint32_t launches = (uint32_t)launch_cuda_core(pq, false, ai, batch * a, s);
    BconvTab t{c->d_up_src, c->d_up_w, c->d_up_dst, a, k};
    const size_t smem = sizeof(uint4) * (t.S + t.D) + sizeof(uint2) * t.S * t.D + sizeof(uint32_t) * t.S * BC_T;
    if (smem > 48 * 1024 && cudaFuncSetAttribute(rns_bconv, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
        return set_err(WD_ECUDA);
    const uint32_t blocks = (uint32_t)std::min<uint64_t>((uint64_t)batch * (pq->N / BC_T), (uint64_t)pq->sm_count * 8);
    rns_bconv<<<blocks, BC_T, smem, s>>>(work, a, nullptr, k, 0, t, pq->N, batch,
                                         reinterpret_cast<unsigned long long*>(partial));
    if (cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    g_last_launches = launches + 1;
    return set_err(WD_OK);
}

int wd_modup_finish(const wd_rns_conv* c, const uint64_t* sum, uint32_t* out_p, uint32_t batch,
                    wd_stream_t st) {
    g_last_launches = 0;
    if (!c || !sum || !out_p) return set_err(WD_EINVAL);
    if (((uintptr_t)sum | (uintptr_t)out_p) & 15) return set_err(WD_EINVAL);
    if (batch == 0) return set_err(WD_OK);
    const wd_ntt_plan* pp = c->pp;
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != pp->device) return set_err(WD_EINVAL);
    cudaStream_t s = (cudaStream_t)st;
    const uint32_t rows = batch * pp->L;
    const uint32_t blocks = (uint32_t)std::min<uint64_t>(((uint64_t)rows * pp->N + 255) / 256, (uint64_t)pp->sm_count * 8);
    rns_reduce64<<<blocks, 256, 0, s>>>(reinterpret_cast<const unsigned long long*>(sum), out_p, c->d_up_dst, pp->L,
                                        pp->N, rows);
    NttArgs af;
    af.in = out_p; af.in2 = nullptr; af.out = out_p; af.tw = pp->d_fwd; af.lc = pp->d_lc; af.L = pp->L;
    const uint32_t launches = 1 + (uint32_t)launch_cuda_core(pp, true, af, rows, s);
    if (cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    g_last_launches = launches;
    return set_err(WD_OK);
}

int wd_moddown(const wd_rns_conv* c, const uint32_t* in, uint32_t* out, uint32_t batch, uint32_t* work, wd_stream_t st) {
    g_last_launches = 0;
    if (!c || !in || !out || !work) return set_err(WD_EINVAL);
    if (((uintptr_t)in | (uintptr_t)out | (uintptr_t)work) & 15) return set_err(WD_EINVAL);
    if (batch == 0) return set_err(WD_OK);
    const wd_ntt_plan *pq = c->pq, *pp = c->pp;
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != pq->device) return set_err(WD_EINVAL);
    if ((uint64_t)batch * (pq->L + pp->L) > 0x7fffffffull) return set_err(WD_EINVAL);
    cudaStream_t s = (cudaStream_t)st;
    const uint32_t N = pq->N, a = pq->L, k = pp->L;
    uint32_t* wp = work;                                   // [batch][k][N] P-limb coefficients
    uint32_t* wq = work + (size_t)batch * k * N;           // [batch][a][N] BConv P -> Q
    // K1: INTT of the P section of in (rows strided by a + k) -> wp
    NttArgs ai;
    ai.in = in + (size_t)a * N; ai.in2 = nullptr; ai.out = wp; ai.tw = pp->d_inv; ai.lc = pp->d_lc; ai.L = k;
    ai.in_ls = a + k;
    launch_v8_rows<0>(pp, false, ai, batch * k, s);
    // K2: BConv P -> Q (coefficient domain) -> wq
    BconvTab t{c->d_dn_src, c->d_dn_w, c->d_dn_dst, k, a};
    if (launch_bconv(pq, wp, k, wq, a, 0, t, batch, s) != WD_OK) return set_err(WD_ECUDA);
    // K3: forward NTT over Q with the store map out = (in_Q - NTT(wq)) * P^-1 (v8, EPI = 2)
    NttArgs af;
    af.in = wq; af.in2 = nullptr; af.out = out; af.tw = pq->d_fwd; af.lc = pq->d_lc; af.L = a;
    af.aux = in; af.rs = c->d_pinv; af.Lfull = a + k;
    launch_v8_rows<2>(pq, true, af, batch * a, s);
    if (cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    g_last_launches = 3;
    return set_err(WD_OK);
}

int wd_ntt_forward_host(const wd_ntt_plan* p, const uint32_t* h_in, uint32_t* h_out, uint32_t batch,
                        uint32_t* d_work, wd_stream_t s) {
    return run_host(p, true, h_in, h_out, batch, d_work, (cudaStream_t)s);
}
int wd_ntt_inverse_host(const wd_ntt_plan* p, const uint32_t* h_in, uint32_t* h_out, uint32_t batch,
                        uint32_t* d_work, wd_stream_t s) {
    return run_host(p, false, h_in, h_out, batch, d_work, (cudaStream_t)s);
}

uint32_t wd_ntt_plan_n(const wd_ntt_plan* p) { return p ? p->N : 0; }
uint32_t wd_ntt_plan_limbs(const wd_ntt_plan* p) { return p ? p->L : 0; }
uint32_t wd_ntt_plan_psi(const wd_ntt_plan* p, uint32_t limb) { return (p && limb < p->L) ? p->psi[limb] : 0; }

uint32_t wd_ntt_root(uint32_t q, uint32_t N) {
    if (!is_pow2(N) || N < 2 || N > (1u << 17) || check_prime(q, N)) return 0;
    return plan_psi_min(q, N);
}
int wd_ntt_check_prime(uint32_t q, uint32_t N) {
    if (!is_pow2(N) || N < 2) return WD_EUNSUPPORTED;
    return check_prime(q, N);
}

int wd_ntt_plan_set_mode(wd_ntt_plan* p, int mode, float tensor_share) {
    if (!p || mode < WD_MODE_AUTO || mode > WD_MODE_FTC) return set_err(WD_EINVAL);
    if ((mode == WD_MODE_TENSOR || mode == WD_MODE_FUSED || mode == WD_MODE_CUDA_GEMM || mode == WD_MODE_FTC) &&
        !tensor_supported(p->logN))
        return set_err(WD_EUNSUPPORTED);
    if ((mode == WD_MODE_CUDA_GEMM || mode == WD_MODE_FTC) && p->logN != 16) return set_err(WD_EUNSUPPORTED);
    if (tensor_share > 1.0f) return set_err(WD_EINVAL);
    p->mode = mode;
    if (tensor_share >= 0.0f) {
        if (mode == WD_MODE_FTC) p->ftc_share = tensor_share;
        else p->tensor_share = tensor_share;
    }
    return set_err(WD_OK);
}
int wd_ntt_plan_get_mode(const wd_ntt_plan* p) { return p ? effective_mode(p) : -1; }

int wd_ntt_plan_autotune(wd_ntt_plan* p, uint32_t batch, wd_stream_t st, float* best_ms) {
    if (!p || batch == 0) return set_err(WD_EINVAL);
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != p->device) return set_err(WD_EINVAL);
    if ((uint64_t)batch * p->L > 0x7fffffffull) return set_err(WD_EINVAL);
    cudaStream_t s = (cudaStream_t)st;
    const size_t bytes = sizeof(uint32_t) * (size_t)batch * p->L * p->N;
    uint32_t *x = nullptr, *y = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    auto cleanup = [&]() {
        if (x) cudaFree(x);
        if (y) cudaFree(y);
        if (e0) cudaEventDestroy(e0);
        if (e1) cudaEventDestroy(e1);
    };
    if (cudaMalloc(&x, bytes) != cudaSuccess || cudaMalloc(&y, bytes) != cudaSuccess ||
        cudaEventCreate(&e0) != cudaSuccess || cudaEventCreate(&e1) != cudaSuccess ||
        cudaMemsetAsync(x, 0, bytes, s) != cudaSuccess) {
        cudaGetLastError(); cleanup(); return set_err(WD_ECUDA);
    }
    struct Cand { int mode; float share; };
    std::vector<Cand> cands = {{WD_MODE_CUDA, p->tensor_share}};
    if (tensor_supported(p->logN) && p->tc.ok) {
        cands.push_back({WD_MODE_FUSED, default_tensor_share(p->logN)});
        for (float sh : {0.25f, 0.5f, 0.75f}) cands.push_back({WD_MODE_FUSED, sh});
        cands.push_back({WD_MODE_TENSOR, p->tensor_share});
        if (p->logN == 16) {
            cands.push_back({WD_MODE_CUDA_GEMM, p->tensor_share});
            cands.push_back({WD_MODE_FTC, p->tensor_share});     // split by the plan's ftc_share
        }
    }
    const int mode0 = p->mode;
    const float share0 = p->tensor_share;
    int best = -1;
    float best_t = 0.0f;
    for (size_t i = 0; i < cands.size(); ++i) {
        p->mode = cands[i].mode;
        p->tensor_share = cands[i].share;
        bool ok = run(p, true, x, nullptr, y, batch, s) == WD_OK && run(p, false, y, nullptr, x, batch, s) == WD_OK;
        float t = 0.0f;
        if (ok) {                                        // one warm-up pair, then 3 timed pairs
            cudaEventRecord(e0, s);
            for (int k = 0; k < 3 && ok; ++k)
                ok = run(p, true, x, nullptr, y, batch, s) == WD_OK && run(p, false, y, nullptr, x, batch, s) == WD_OK;
            cudaEventRecord(e1, s);
            ok = ok && cudaEventSynchronize(e1) == cudaSuccess && cudaEventElapsedTime(&t, e0, e1) == cudaSuccess;
        }
        if (!ok) {
            if (cudaGetLastError() != cudaSuccess || cands[i].mode == WD_MODE_CUDA) {
                p->mode = mode0; p->tensor_share = share0; cleanup(); return set_err(WD_ECUDA);
            }
            continue;                                    // this path is unsupported here: skip it
        }
        t /= 3.0f;
        if (best < 0 || t < best_t) { best = (int)i; best_t = t; }
    }
    cleanup();
    p->mode = cands[best].mode;
    p->tensor_share = cands[best].share;
    if (best_ms) *best_ms = best_t;
    return set_err(WD_OK);
}

uint32_t wd_ntt_last_launches(void) { return g_last_launches; }

int wd_ntt_occupancy(const wd_ntt_plan* p, int mode, int fwd) {
    if (!p) return -1;
    int occ = -1;
    cudaError_t e = cudaErrorInvalidValue;
    if (p->logN == 16 && mode == WD_MODE_TENSOR)
        e = fwd ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ntt_tc16<true>, TC_T, TC_SMEM)
                : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ntt_tc16<false>, TC_T, TC_SMEM);
    else if (p->logN == 16 && mode == WD_MODE_CUDA)      // the AUTO kernel at >= SM-count rows (v8)
        e = fwd ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ntt_v8<16, true, false, 0, 5>, V8_T, V8_SMEM)
                : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ntt_v8<16, false, false, 0, 5>, V8_T, V8_SMEM);
    else if (p->logN == 17 && mode == WD_MODE_CUDA)
        e = fwd ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ntt_v8<17, true, false, 0, 4>, V8_T, V8_SMEM)
                : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ntt_v8<17, false, false, 0, 5>, V8_T, V8_SMEM);
    if (e != cudaSuccess) { cudaGetLastError(); return -(int)e; }
    return occ;
}
int wd_ntt_last_error(void) { return g_last_error; }
const char* wd_ntt_strerror(int code) {
    switch (code) {
        case WD_OK: return "ok";
        case WD_EINVAL: return "invalid argument (NULL/misaligned pointer, bad size or wrong device)";
        case WD_EPRIME: return "modulus is not an NTT-friendly prime < 2^30 (q prime, q = 1 mod 2N)";
        case WD_EUNSUPPORTED: return "unsupported size or mode";
        case WD_ECUDA: return "CUDA runtime error";
        case WD_ENOMEM: return "out of memory";
        default: return "unknown error";
    }
}
const char* wd_ntt_version(void) { return "wdntt 0.1 (sm_100a)"; }

}  // extern "C"
