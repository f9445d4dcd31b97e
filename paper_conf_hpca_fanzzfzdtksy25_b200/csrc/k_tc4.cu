// k_tc4.cu -- host side of the 4-step tcgen05 kernel (ntt_tc4.cuh): stage matrices as byte planes,
// the per-element twist in worker-lane order, TMA tensor maps per call, launch.
#include <cuda.h>
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <new>
#include <vector>
#include "wd_ntt.h"
#include "launch.h"
#include "ntt_tc4.cuh"
#include "plan_math.h"

namespace wd {

namespace {

using tc4::MAT;
using tc4::MATSET;

// psi^e for e taken mod 2N (pw has 2N entries)
struct Pow {
    std::vector<uint32_t> pw;
    uint32_t q;
    Pow(uint32_t psi, uint32_t q_, uint32_t two_n) : pw(two_n), q(q_) {
        pw[0] = 1;
        for (uint32_t i = 1; i < two_n; ++i) pw[i] = pm_mul(pw[i - 1], psi, q);
    }
    uint32_t operator()(uint64_t e) const { return pw[e % pw.size()]; }
};

// the forward stage matrices of one limb (tc4 header):
//   MA[c][a] = psi^(4096 a (2c+1)); MB_c[d][b] = psi^(256 b (2c+1+32d)); MC[g][f] = psi^(8192 g f);
//   MD_g[h'][e] = psi^(512 e (g + 16 brv4(h')))
void fwd_mats(const Pow& P, uint32_t MA[16][16], uint32_t MB[16][16][16], uint32_t MC[16][16], uint32_t MD[16][16][16]) {
    for (uint32_t c = 0; c < 16; ++c)
        for (uint32_t a = 0; a < 16; ++a) MA[c][a] = P(4096ull * a * (2 * c + 1));
    for (uint32_t c = 0; c < 16; ++c)
        for (uint32_t d = 0; d < 16; ++d)
            for (uint32_t b = 0; b < 16; ++b) MB[c][d][b] = P(256ull * b * (2 * c + 1 + 32 * d));
    for (uint32_t g = 0; g < 16; ++g)
        for (uint32_t f = 0; f < 16; ++f) MC[g][f] = P(8192ull * g * f);
    for (uint32_t g = 0; g < 16; ++g)
        for (uint32_t hp = 0; hp < 16; ++hp)
            for (uint32_t e = 0; e < 16; ++e) MD[g][hp][e] = P(512ull * e * (g + 16 * pm_brv(hp, 4)));
}

// host model of the forward decomposition on one row (exact arithmetic), for the plan's self-check
void fwd_model(const Pow& P, const uint32_t* x, uint32_t* out) {
    const uint32_t q = P.q;
    uint32_t MA[16][16], MB[16][16][16], MC[16][16], MD[16][16][16];
    fwd_mats(P, MA, MB, MC, MD);
    std::vector<uint32_t> Z(65536);               // Z[k1][j2]
    for (uint32_t j2 = 0; j2 < 256; ++j2) {
        uint32_t U[16][16];                       // U[c][b]
        for (uint32_t b = 0; b < 16; ++b)
            for (uint32_t c = 0; c < 16; ++c) {
                uint64_t s = 0;
                for (uint32_t a = 0; a < 16; ++a) s = (s + (uint64_t)MA[c][a] * x[256 * (16 * a + b) + j2]) % q;
                U[c][b] = (uint32_t)s;
            }
        for (uint32_t c = 0; c < 16; ++c)
            for (uint32_t d = 0; d < 16; ++d) {
                uint64_t s = 0;
                for (uint32_t b = 0; b < 16; ++b) s = (s + (uint64_t)MB[c][d][b] * U[c][b]) % q;
                const uint32_t k1 = c + 16 * d;
                Z[256 * k1 + j2] = pm_mul((uint32_t)s, P((uint64_t)(2 * k1 + 1) * j2), q);
            }
    }
    for (uint32_t k1 = 0; k1 < 256; ++k1) {
        uint32_t V[16][16];                       // V[g][e]
        for (uint32_t e = 0; e < 16; ++e)
            for (uint32_t g = 0; g < 16; ++g) {
                uint64_t s = 0;
                for (uint32_t f = 0; f < 16; ++f) s = (s + (uint64_t)MC[g][f] * Z[256 * k1 + 16 * f + e]) % q;
                V[g][e] = (uint32_t)s;
            }
        const uint32_t r = pm_brv(k1, 8);
        for (uint32_t g = 0; g < 16; ++g)
            for (uint32_t hp = 0; hp < 16; ++hp) {
                uint64_t s = 0;
                for (uint32_t e = 0; e < 16; ++e) s = (s + (uint64_t)MD[g][hp][e] * V[g][e]) % q;
                out[256 * r + 16 * pm_brv(g, 4) + hp] = (uint32_t)s;
            }
    }
}

// merged-psi Cooley-Tukey forward with the plan's bit-reversed psi powers (the CUDA-core definition)
void ct_forward(const std::vector<uint32_t>& psi_brv, uint32_t q, std::vector<uint32_t>& a) {
    const uint32_t N = (uint32_t)a.size();
    for (uint32_t m = 1, t = N; m < N; m <<= 1) {
        t >>= 1;
        for (uint32_t i = 0; i < m; ++i) {
            const uint64_t S = psi_brv[m + i];
            for (uint32_t j = 2 * i * t; j < 2 * i * t + t; ++j) {
                const uint32_t U = a[j], V = (uint32_t)(a[j + t] * S % q);
                a[j] = (U + V) % q;
                a[j + t] = (U + q - V) % q;
            }
        }
    }
}

using EncodeFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                              const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                              CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeFn encoder() {
    static EncodeFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, []() {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult qr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &qr) == cudaSuccess &&
            qr == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<EncodeFn>(p);
    });
    return fn;
}

bool encode(CUtensorMap* m, const void* base, uint32_t rank, const cuuint64_t* dims, const cuuint64_t* strides,
            const cuuint32_t* box, CUtensorMapSwizzle sw) {
    EncodeFn enc = encoder();
    if (!enc) return false;
    cuuint32_t es[5] = {1, 1, 1, 1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT32, rank, const_cast<void*>(base), dims, strides, box, es,
               CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

unsigned long long* g_trace = nullptr;     // diagnostics (wd_tc4_set_trace)

}  // namespace

bool tma_encode_u32(CUtensorMap* m, const void* base, uint32_t rank, const cuuint64_t* dims, const cuuint64_t* strides,
                    const cuuint32_t* box, CUtensorMapSwizzle sw) {
    return encode(m, base, rank, dims, strides, box, sw);
}

void tc4_set_trace(void* p) { g_trace = static_cast<unsigned long long*>(p); }

void free_tc4_tables(Tc4Tables& t) {
    cudaFree(t.d_mat); cudaFree(t.d_tw); cudaFree(t.d_lq);
    t = Tc4Tables();
}

int build_tc4_tables(Tc4Tables& t, const std::vector<uint32_t>& primes, const std::vector<uint32_t>& psis) {
    const uint32_t L = (uint32_t)primes.size(), N = 1u << 16;
    std::vector<uint8_t> mat((size_t)L * 2 * MATSET);
    std::vector<uint2> tw((size_t)L * 2 * 16 * 16 * 128);
    std::vector<uint4> lq(L);
    for (uint32_t l = 0; l < L; ++l) {
        const uint32_t q = primes[l];
        const Pow P(psis[l], q, 2 * N);
        uint32_t MA[16][16], MB[16][16][16], MC[16][16], MD[16][16][16];
        fwd_mats(P, MA, MB, MC, MD);
        uint8_t* m0 = &mat[((size_t)l * 2 + 0) * MATSET];
        uint8_t* m1 = &mat[((size_t)l * 2 + 1) * MATSET];
        byte_planes(m0, MA, q);
        byte_planes(m1, MC, q);
        for (int k = 0; k < 16; ++k) {
            byte_planes(m0 + (1 + k) * MAT, MB[k], q);
            byte_planes(m1 + (1 + k) * MAT, MD[k], q);
        }
        // twist T[k1][j2] = psi^((2 k1 + 1) j2) at [h][c][d][lane m], k1 = c + 16 d, j2 = 128 h + pi(m)
        for (uint32_t h = 0; h < 2; ++h)
            for (uint32_t c = 0; c < 16; ++c)
                for (uint32_t d = 0; d < 16; ++d)
                    for (uint32_t m = 0; m < 128; ++m) {
                        const uint32_t k1 = c + 16 * d, j2 = 128 * h + tc4::col_pi(m);
                        const uint32_t w = P((uint64_t)(2 * k1 + 1) * j2);
                        tw[((((size_t)l * 2 + h) * 16 + c) * 16 + d) * 128 + m] = make_uint2(w, pm_shoup(w, q));
                    }
        lq[l] = make_uint4(q, pm_shoup(65536u % q, q), pm_shoup(1u, q), 0);
        if (l == 0) {                             // self-check of the decomposition against the CT network
            std::vector<uint32_t> psi_brv(N), x(N), y(N);
            for (uint32_t i = 0; i < N; ++i) psi_brv[i] = P(pm_brv(i, 16));
            for (uint32_t i = 0; i < N; ++i) x[i] = (uint32_t)(((uint64_t)i * 2654435761u + 12345) % q);
            fwd_model(P, x.data(), y.data());
            ct_forward(psi_brv, q, x);
            if (x != y) return WD_ECUDA;
        }
    }
    auto up = [](void** d, const void* h, size_t n) {
        if (cudaMalloc(d, n) != cudaSuccess) return false;
        return cudaMemcpy(*d, h, n, cudaMemcpyHostToDevice) == cudaSuccess;
    };
    if (!up((void**)&t.d_mat, mat.data(), mat.size()) || !up((void**)&t.d_tw, tw.data(), tw.size() * sizeof(uint2)) ||
        !up((void**)&t.d_lq, lq.data(), lq.size() * sizeof(uint4)))
        return WD_ENOMEM;
    t.ok = true;
    return WD_OK;
}

int prep_tc4() {
    if (cudaFuncSetAttribute(tc4::ntt_tc4_fwd, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tc4::SMEM) != cudaSuccess)
        return 4;
    return 0;
}

// the forward over rows = batch * L rows of a [batch][L][2^16] tensor; in == out allowed
int launch_tc4(bool fwd, const NttArgs& a, const Tc4Tables& t, uint32_t rows, int sm_count, cudaStream_t s) {
    if (!t.ok || !fwd || a.in2 || a.in_ls || a.out_ls || a.aux || a.cpy) return -1;
    CUtensorMap mx, mc, mi, mo;
    {   // x pieces: (j2 256, b 16, a 16, row) -> box (128, 1, 16, 1)
        const cuuint64_t dims[4] = {256, 16, 16, rows};
        const cuuint64_t str[3] = {1024, 16384, 262144};
        const cuuint32_t box[4] = {128, 1, 16, 1};
        if (!encode(&mx, a.in, 4, dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE)) return -2;
    }
    {   // row-pass operand tiles: (w 128, row8 8, kc 2, h 2, rg rows*32) -> canonical K-major tile
        const cuuint64_t dims[5] = {128, 8, 2, 2, (cuuint64_t)rows * 32};
        const cuuint64_t str[4] = {1024, 16, 512, 8192};
        const cuuint32_t box[5] = {4, 8, 2, 2, 16};
        if (!encode(&mc, a.out, 5, dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE)) return -2;
    }
    {   // intermediate store: (cols 256, matrix rows rows*256) -> box (128, 16)
        const cuuint64_t dims[2] = {256, (cuuint64_t)rows * 256};
        const cuuint64_t str[1] = {1024};
        const cuuint32_t box[2] = {128, 16};
        if (!encode(&mi, a.out, 2, dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE)) return -2;
    }
    {   // final store: box (16 words, 128 rows), 64-byte swizzled staging
        const cuuint64_t dims[2] = {256, (cuuint64_t)rows * 256};
        const cuuint64_t str[1] = {1024};
        const cuuint32_t box[2] = {16, 128};
        if (!encode(&mo, a.out, 2, dims, str, box, CU_TENSOR_MAP_SWIZZLE_64B)) return -2;
    }
    tc4::Args ta;
    ta.mat = t.d_mat;
    ta.tw = t.d_tw;
    ta.lq = t.d_lq;
    ta.rows = rows; ta.L = a.L; ta.nb = rows / a.L;
    ta.trace = g_trace;
    const uint32_t grid = std::min<uint32_t>(rows, (uint32_t)sm_count);
    tc4::ntt_tc4_fwd<<<grid, tc4::NT, tc4::SMEM, s>>>(mx, mc, mi, mo, ta);
    return cudaPeekAtLastError() == cudaSuccess ? 1 : -2;   // the caller reports WD_ECUDA
}

}  // namespace wd
