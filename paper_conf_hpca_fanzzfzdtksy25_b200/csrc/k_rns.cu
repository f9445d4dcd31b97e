// k_rns.cu -- launchers of the RNS kernels around the NTT (kernels in ntt_rns.cuh).
#include <algorithm>
#include "launch.h"
#include "ntt_rns.cuh"

namespace wd {

namespace {
// shared memory of the general BConv kernel for S sources and D targets
size_t bconv_smem(uint32_t S, uint32_t D) {
    return sizeof(uint4) * (S + D) + sizeof(uint2) * (size_t)S * D + sizeof(uint32_t) * (size_t)S * BC_T;
}
}  // namespace

// rns_bconv's dynamic shared-memory ceiling is set ONCE, at its worst case (S = D = BC_MAX), so
// concurrent calls with different conversion objects never race on the attribute
int prep_rns() {
    const int worst = (int)bconv_smem(BC_MAX, BC_MAX);
    if (cudaFuncSetAttribute(rns_bconv, cudaFuncAttributeMaxDynamicSharedMemorySize, worst) != cudaSuccess) return 4;
    return 0;
}

void launch_rs_gather(const uint32_t* in, uint32_t* work, uint32_t N, uint32_t L, uint32_t batch, int sm_count,
                      cudaStream_t s) {
    const uint32_t n4 = N / 4;
    const uint32_t blocks = (uint32_t)std::min<uint64_t>(((uint64_t)batch * n4 + 255) / 256, (uint64_t)sm_count * 8);
    rs_gather<<<blocks, 256, 0, s>>>(reinterpret_cast<const uint4*>(in), reinterpret_cast<uint4*>(work), n4, L, batch);
}

void launch_bconv(const uint32_t* x, uint32_t x_ls, uint32_t* y, uint32_t y_ls, uint32_t y_off, const BconvTab& t,
                  uint32_t N, uint32_t batch, int sm_count, cudaStream_t s) {
    const size_t sm_few = sizeof(uint4) * (t.S + t.D) + sizeof(uint2) * t.S * t.D;
    if (t.D <= 4 && t.S > 4 && N >= (uint32_t)BCF_C) {            // few targets: register accumulation
        const uint32_t blocks = (uint32_t)std::min<uint64_t>((uint64_t)batch * (N / BCF_C), (uint64_t)sm_count * 8);
        switch (t.D) {
            case 1: rns_bconv_few<1><<<blocks, BC_T, sm_few, s>>>(x, x_ls, y, y_ls, y_off, t, N, batch); break;
            case 2: rns_bconv_few<2><<<blocks, BC_T, sm_few, s>>>(x, x_ls, y, y_ls, y_off, t, N, batch); break;
            case 3: rns_bconv_few<3><<<blocks, BC_T, sm_few, s>>>(x, x_ls, y, y_ls, y_off, t, N, batch); break;
            default: rns_bconv_few<4><<<blocks, BC_T, sm_few, s>>>(x, x_ls, y, y_ls, y_off, t, N, batch); break;
        }
        return;
    }
    if (t.S <= 4 && N >= (uint32_t)BCF_C) {                       // few sources: terms in registers, 16-B stores
        const uint32_t blocks = (uint32_t)std::min<uint64_t>((uint64_t)batch * (N / BCF_C), (uint64_t)sm_count * 8);
        switch (t.S) {
            case 1: rns_bconv_fewsrc<1><<<blocks, BC_T, sm_few, s>>>(x, x_ls, y, y_ls, y_off, t, N, batch); break;
            case 2: rns_bconv_fewsrc<2><<<blocks, BC_T, sm_few, s>>>(x, x_ls, y, y_ls, y_off, t, N, batch); break;
            case 3: rns_bconv_fewsrc<3><<<blocks, BC_T, sm_few, s>>>(x, x_ls, y, y_ls, y_off, t, N, batch); break;
            default: rns_bconv_fewsrc<4><<<blocks, BC_T, sm_few, s>>>(x, x_ls, y, y_ls, y_off, t, N, batch); break;
        }
        return;
    }
    const uint32_t blocks = (uint32_t)std::min<uint64_t>((uint64_t)batch * (N / BC_T), (uint64_t)sm_count * 8);
    rns_bconv<<<blocks, BC_T, bconv_smem(t.S, t.D), s>>>(x, x_ls, y, y_ls, y_off, t, N, batch);
}

void launch_bconv_partial(const uint32_t* x, uint32_t x_ls, uint64_t* y64, const BconvTab& t, uint32_t N,
                          uint32_t batch, int sm_count, cudaStream_t s) {
    const uint32_t blocks = (uint32_t)std::min<uint64_t>((uint64_t)batch * (N / BC_T), (uint64_t)sm_count * 8);
    rns_bconv<<<blocks, BC_T, bconv_smem(t.S, t.D), s>>>(x, x_ls, nullptr, t.D, 0, t, N, batch,
                                                        reinterpret_cast<unsigned long long*>(y64));
}

void launch_reduce64(const uint64_t* sum, uint32_t* out, const uint4* dst, uint32_t D, uint32_t N, uint32_t rows,
                     int sm_count, cudaStream_t s) {
    const uint32_t blocks = (uint32_t)std::min<uint64_t>(((uint64_t)rows * N + 255) / 256, (uint64_t)sm_count * 8);
    rns_reduce64<<<blocks, 256, 0, s>>>(reinterpret_cast<const unsigned long long*>(sum), out, dst, D, N, rows);
}

}  // namespace wd
