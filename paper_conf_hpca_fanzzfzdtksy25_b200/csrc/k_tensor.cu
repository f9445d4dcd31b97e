// k_tensor.cu -- the round-1 tcgen05 path for N = 2^16 (TENSOR and FUSED modes)
// and its host tables (row a1).  Kernels in ntt_tensor.cuh / ntt_fused.cuh.
#include <algorithm>
#include <new>
#include "launch.h"
#include "ntt_tensor.cuh"
#include "ntt_fused.cuh"

namespace wd {

void free_tensor_tables(TensorTables& t) {
    cudaFree(t.d_G); cudaFree(t.d_B); cudaFree(t.d_tw1); cudaFree(t.d_tw2); cudaFree(t.d_tw3);
    cudaFree(t.d_sg1); cudaFree(t.d_sg2); cudaFree(t.d_sg3); cudaFree(t.d_c16); cudaFree(t.d_mat);
    t = TensorTables();
}

// Builds and verifies the factorised block tables for every limb (logN == 16 only).
int build_tensor_tables(TensorTables& tc, uint32_t logN, const std::vector<uint32_t>& primes,
                               const std::vector<uint32_t>& psis) {
    if (logN != 16) return 0;
    const uint32_t N = 1u << 16, L = (uint32_t)primes.size();
    std::vector<uint8_t> B((size_t)L * 4 * 4096), Gi((size_t)L * 2 * 17 * 4096);
    std::vector<uint2> t1((size_t)L * 256), t2((size_t)L * 4096), t3((size_t)L * 65536);
    std::vector<uint2> s1((size_t)L * 256), s2((size_t)L * 4096), s3((size_t)L * 65536);
    std::vector<uint2> c16(L);
    std::vector<uint32_t> mat((size_t)L * 4 * 256);
    for (uint32_t l = 0; l < L; ++l) {
        const uint32_t q = primes[l], psi = psis[l], psi_inv = pm_pow(psi, q - 2, q);
        std::vector<uint32_t> pw(N), pwi(N), fb(N), ib(N);
        pw[0] = pwi[0] = 1;
        for (uint32_t i = 1; i < N; ++i) { pw[i] = pm_mul(pw[i - 1], psi, q); pwi[i] = pm_mul(pwi[i - 1], psi_inv, q); }
        for (uint32_t i = 0; i < N; ++i) { fb[i] = pw[pm_brv(i, 16)]; ib[i] = pwi[pm_brv(i, 16)]; }
        const uint32_t ninv = pm_pow(N % q, q - 2, q);
        uint32_t M[16][16], F[16][16], Fi[16][16];
        block_fwd(M, fb, 0, 0, q);
        std::memcpy(&mat[((size_t)l * 4 + 0) * 256], M, 1024);
        byte_planes(&B[((size_t)l * 4 + 0) * 4096], M, q);
        byte_planes(&Gi[(((size_t)l * 2 + 0) * 17 + 0) * 4096], M, q);
        block_inv(M, ib, 0, 0, q, ninv);
        std::memcpy(&mat[((size_t)l * 4 + 2) * 256], M, 1024);
        byte_planes(&B[((size_t)l * 4 + 2) * 4096], M, q);
        byte_planes(&Gi[(((size_t)l * 2 + 1) * 17 + 0) * 4096], M, q);
        for (uint32_t g = 0; g < 16; ++g) {              // stage-1 blocks, one image per group
            block_fwd(M, fb, 4, g, q);
            byte_planes(&Gi[(((size_t)l * 2 + 0) * 17 + 1 + g) * 4096], M, q);
            block_inv(M, ib, 4, g, q, 0);
            byte_planes(&Gi[(((size_t)l * 2 + 1) * 17 + 1 + g) * 4096], M, q);
        }
        // fixed DFTs from one group, then every group of stages 1..3 must factor through them
        bool have_f = false;
        struct S { int ls; uint32_t groups; uint2* tw; uint2* sg; };
        S st[3] = {{4, 16, &t1[(size_t)l * 256], &s1[(size_t)l * 256]},
                   {8, 256, &t2[(size_t)l * 4096], &s2[(size_t)l * 4096]},
                   {12, 4096, &t3[(size_t)l * 65536], &s3[(size_t)l * 65536]}};
        for (auto& s : st) {
            for (uint32_t g = 0; g < s.groups; ++g) {
                uint32_t Mf[16][16], Mi[16][16];
                block_fwd(Mf, fb, s.ls, g, q);
                block_inv(Mi, ib, s.ls, g, q, 0);
                for (int j = 0; j < 16; ++j) {
                    const uint32_t tau = Mf[0][j], taui = pm_pow(tau, q - 2, q);
                    const uint32_t sig = Mi[j][0], sigi = pm_pow(sig, q - 2, q);
                    s.tw[g * 16 + j] = make_uint2(tau, pm_shoup(tau, q));
                    s.sg[g * 16 + j] = make_uint2(sig, pm_shoup(sig, q));
                    for (int k = 0; k < 16; ++k) {
                        const uint32_t f = pm_mul(Mf[k][j], taui, q);       // F[k][j]
                        const uint32_t fi = pm_mul(Mi[j][k], sigi, q);      // F'[j][k]
                        if (!have_f) { F[k][j] = f; Fi[j][k] = fi; }
                        else if (F[k][j] != f || Fi[j][k] != fi) return 4;  // factorisation failed
                    }
                }
                have_f = true;
            }
        }
        byte_planes(&B[((size_t)l * 4 + 1) * 4096], F, q);
        byte_planes(&B[((size_t)l * 4 + 3) * 4096], Fi, q);
        std::memcpy(&mat[((size_t)l * 4 + 1) * 256], F, 1024);
        std::memcpy(&mat[((size_t)l * 4 + 3) * 256], Fi, 1024);
        c16[l] = make_uint2(pm_shoup(65536u % q, q), pm_shoup(1u, q));
    }
    auto up = [](void** d, const void* h, size_t n) {
        if (cudaMalloc(d, n) != cudaSuccess) return false;
        return cudaMemcpy(*d, h, n, cudaMemcpyHostToDevice) == cudaSuccess;
    };
    if (!up((void**)&tc.d_G, Gi.data(), Gi.size()) || !up((void**)&tc.d_B, B.data(), B.size()) || !up((void**)&tc.d_tw1, t1.data(), t1.size() * 8) ||
        !up((void**)&tc.d_tw2, t2.data(), t2.size() * 8) || !up((void**)&tc.d_tw3, t3.data(), t3.size() * 8) ||
        !up((void**)&tc.d_sg1, s1.data(), s1.size() * 8) || !up((void**)&tc.d_sg2, s2.data(), s2.size() * 8) ||
        !up((void**)&tc.d_sg3, s3.data(), s3.size() * 8) || !up((void**)&tc.d_c16, c16.data(), c16.size() * 8) ||
        !up((void**)&tc.d_mat, mat.data(), mat.size() * 4))
        return 4;
    tc.ok = true;
    return 0;
}

int prep_tensor() {
    for (auto k : {ntt_tc16<true>, ntt_tc16<false>, ntt_tc16<true, 2>, ntt_tc16<false, 2>})
        if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, TC_SMEM) != cudaSuccess ||
            cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, 100) != cudaSuccess)
            return 4;
    for (auto k : {ntt_tcc16<true>, ntt_tcc16<false>})
        if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, TCC_SMEM) != cudaSuccess ||
            cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, 100) != cudaSuccess)
            return 4;
    return prepare_fused_kernels(16);
}

static TcArgs tc_args(bool fwd, const NttArgs& a, const TensorTables& tc) {
    TcArgs ta;
    ta.a = a;
    ta.B = tc.d_B;
    ta.t1 = fwd ? tc.d_tw1 : tc.d_sg1;
    ta.t2 = fwd ? tc.d_tw2 : tc.d_sg2;
    ta.t3 = fwd ? tc.d_tw3 : tc.d_sg3;
    ta.c16 = tc.d_c16;
    return ta;
}

// TENSOR mode: column phase (ntt_tcc16, TMEM-staged, both column stages folded, one CTA per SM) and
// row phase (ntt_tc16<PH = 2>), in the reverse order for the inverse
int launch_tensor(bool fwd, const NttArgs& a, const TensorTables& tc, uint32_t rows, int sm_count, cudaStream_t s) {
    if (!tc.ok) return -1;
    const TcArgs ta = tc_args(fwd, a, tc);
    const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)(sm_count * TC_CTAS_PER_SM));
    const uint32_t gc = std::min<uint32_t>(rows, (uint32_t)sm_count);
    const uint32_t per = (rows + gc - 1) / gc;
    if (fwd) {
        ntt_tcc16<true><<<gc, TC_T, TCC_SMEM, s>>>(ta, tc.d_G, rows, per);
        ntt_tc16<true, 2><<<grid, TC_T, TC_SMEM, s>>>(ta, rows);
    } else {
        ntt_tc16<false, 2><<<grid, TC_T, TC_SMEM, s>>>(ta, rows);
        ntt_tcc16<false><<<gc, TC_T, TCC_SMEM, s>>>(ta, tc.d_G, rows, per);
    }
    return 2;
}

int launch_fused(bool fwd, const NttArgs& a, const TensorTables& tc, uint32_t rows, int sm_count, float share,
                 cudaStream_t s) {
    return launch_fused(16u, fwd, a, tc, rows, sm_count, share, s);
}

}  // namespace wd
