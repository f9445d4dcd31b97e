// tensor_tables.h -- host precompute for the tcgen05 int8 path (H-3, H-4).
//
// A radix-16 block of the merged-psi NTT (4 butterfly layers starting at layer
// ls, group hi) is a 16x16 matrix M over Z_q.  We obtain it exactly by running
// the 4 layers (with the plan's own twiddles) on the 16 unit vectors, so it is
// by construction the same map the CUDA-core path applies.  Every such block
// factors as
//     forward  M_{ls,hi} = F  . diag(tau_{ls,hi})      (twist on the input side)
//     inverse  MI_{ls,hi} = diag(sig_{ls,hi}) . F'     (twist on the output side)
// with F (F') the same 16-point (inverse) DFT for every group -- the "inner
// NTT" of PAPER.md:93-100 / 272-282 (Eq.(2) with the twiddle Hadamard of
// steps 2/4/6 split off).  The factorisation is verified here for every block
// before the tables are accepted.
//
// Byte-plane GEMM (PAPER.md:102, 173-187 bit splitting, re-derived, SURVEY H-3):
// for a data vector x (any uint32, viewed as 4 little-endian bytes x_{j,a}),
//     D_b[k] = sum_{j,a} byte_b( M[k][j] * 2^(8a) mod q ) * x_{j,a}    (u8 x u8 -> s32)
//     sum_b 2^(8b) D_b[k] = sum_j M[k][j] x_j   (mod q)
// so the u8 view of the u32 data needs no splitting pass.  The B operand is
// the 64 x 64 byte matrix B[n = 4k+b][kk = 4j+a], stored in the K-major
// SWIZZLE_NONE canonical layout (8-row x 16-byte core matrices, LBO = 128 B
// between K-adjacent core matrices, SBO = 512 B between 8-row groups).
#pragma once
#include <cstdint>
#include <vector_types.h>
#include <cstring>
#include <vector>
#include "plan_math.h"

namespace wd {

struct TensorTables {
    uint8_t* d_G = nullptr;        // [L][2][17][4096]: per direction, [0] = single-group stage (M0 / MI0),
                                   //   [1+g] = stage-1 block of group g (M1_g / MI1_g), twists folded in
    uint8_t* d_B = nullptr;        // [L][4][4096]: fwd M0, fwd F, inv MI0 (with N^-1), inv F'
    uint2* d_tw1 = nullptr;        // [L][16][16]    fwd twist tau, stage 1   (group, j)
    uint2* d_tw2 = nullptr;        // [L][256][16]   fwd twist tau, stage 2
    uint2* d_tw3 = nullptr;        // [L][4096][16]  fwd twist tau, stage 3
    uint2* d_sg1 = nullptr;        // [L][16][16]    inv twist sigma, stage 1' (group, k)
    uint2* d_sg2 = nullptr;        // [L][256][16]
    uint2* d_sg3 = nullptr;        // [L][4096][16]
    uint2* d_c16 = nullptr;        // [L] Shoup companions of 2^16 and of 1
    uint32_t* d_mat = nullptr;     // [L][4][256] u32 block matrices M0, F, MI0 (N^-1), F' (WD-CUDA, row f2)
    bool ok = false;
};

inline uint32_t umma_off(int row, int kbyte) {        // byte offset in a K-major, 64-byte-K tile
    return (uint32_t)((row & 7) * 16 + (row >> 3) * 512 + (kbyte >> 4) * 128 + (kbyte & 15));
}

// 4 forward (CT) layers ls..ls+3 of group hi applied to each unit vector: M[k][j]
inline void block_fwd(uint32_t M[16][16], const std::vector<uint32_t>& psi_brv, int ls, uint32_t hi, uint32_t q) {
    for (int j = 0; j < 16; ++j) {
        uint64_t x[16] = {0};
        x[j] = 1;
        for (int t = 0; t < 4; ++t) {
            const int h = 8 >> t;
            for (int g = 0; g < (1 << t); ++g) {
                const uint64_t w = psi_brv[(1u << (ls + t)) + (hi << t) + g];
                for (int r = 0; r < h; ++r) {
                    const int a = 2 * g * h + r, b = a + h;
                    const uint64_t v = (x[b] * w) % q;
                    const uint64_t u = x[a];
                    x[a] = (u + v) % q;
                    x[b] = (u + q - v) % q;
                }
            }
        }
        for (int k = 0; k < 16; ++k) M[k][j] = (uint32_t)x[k];
    }
}
// 4 inverse (GS) layers ls+3..ls of group hi (N^-1 folded when ls == 0 and ninv != 0)
inline void block_inv(uint32_t M[16][16], const std::vector<uint32_t>& psi_inv_brv, int ls, uint32_t hi, uint32_t q,
                      uint32_t ninv) {
    for (int j = 0; j < 16; ++j) {
        uint64_t x[16] = {0};
        x[j] = 1;
        for (int t = 3; t >= 0; --t) {
            const int h = 8 >> t;
            for (int g = 0; g < (1 << t); ++g) {
                const uint64_t w = psi_inv_brv[(1u << (ls + t)) + (hi << t) + g];
                for (int r = 0; r < h; ++r) {
                    const int a = 2 * g * h + r, b = a + h;
                    const uint64_t u = x[a], v = x[b];
                    x[a] = (u + v) % q;
                    x[b] = (((u + q - v) % q) * w) % q;
                }
            }
        }
        if (ls == 0 && ninv)
            for (int k = 0; k < 16; ++k) x[k] = (x[k] * ninv) % q;
        for (int k = 0; k < 16; ++k) M[k][j] = (uint32_t)x[k];
    }
}

// 64x64 byte-plane image of M in the UMMA layout (see header)
inline void byte_planes(uint8_t* img, const uint32_t M[16][16], uint32_t q) {
    std::memset(img, 0, 4096);
    for (int k = 0; k < 16; ++k)
        for (int j = 0; j < 16; ++j)
            for (int a = 0; a < 4; ++a) {
                const uint32_t v = (uint32_t)(((uint64_t)M[k][j] << (8 * a)) % q);
                for (int b = 0; b < 4; ++b) img[umma_off(4 * k + b, 4 * j + a)] = (uint8_t)(v >> (8 * b));
            }
}

}  // namespace wd
