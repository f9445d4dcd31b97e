// int_probe.cu -- B200 integer-pipe throughput probes for the Shoup butterfly.
// Each kernel runs 16 independent chains per thread, 8 warps x 4 CTAs per SM; the host side
// reports operations per clock per SM.  Build + run: python scripts/int_probe.py
#include <cuda_runtime.h>
#include <cstdint>

#define CHAINS 16

// mode 0: IMAD.HI (__umulhi)           mode 1: IMAD.WIDE.U32, both halves used
// mode 2: IMAD (lo)                     mode 3: full Shoup multiply (HI + 2 lo)
// mode 4: LOP3 + IADD3 (ALU)           mode 5: CT butterfly (Shoup + VIADDMNMX + 2 IADD3)
// mode 6: IADD3                         mode 7: CT butterfly with 64-bit hi
template <int MODE>
__global__ void k_int(int iters, uint32_t q, uint32_t w, uint32_t ws, uint32_t* sink) {
    uint32_t x[CHAINS];
#pragma unroll
    for (int i = 0; i < CHAINS; ++i) x[i] = threadIdx.x * 16 + i + blockIdx.x;
    const uint32_t q2 = 2 * q;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < CHAINS; ++i) {
            uint32_t v = x[i];
            if (MODE == 0) v = __umulhi(v, ws) ^ v;
            if (MODE == 1) { uint64_t p; asm("mul.wide.u32 %0, %1, %2;" : "=l"(p) : "r"(v), "r"(ws)); v = (uint32_t)(p >> 32) ^ (uint32_t)p; }
            if (MODE == 2) v = v * ws + w;
            if (MODE == 3) v = v * w - __umulhi(v, ws) * q;
            if (MODE == 4) v = (v ^ w) + ws;   // LOP3 + IADD3 (ALU-only reference)
            if (MODE == 6) v = v + ws + w;
            x[i] = v;
        }
        if (MODE == 5 || MODE == 7) {
#pragma unroll
            for (int i = 0; i < CHAINS; i += 2) {
                uint32_t X = x[i], Y = x[i + 1];
                const uint32_t xx = min(X, X - q2);
                const uint32_t hq = MODE == 5 ? __umulhi(Y, ws) : (uint32_t)(((uint64_t)Y * ws) >> 32);
                const uint32_t t = Y * w - hq * q;
                x[i] = xx + t;
                x[i + 1] = xx - t + q2;
            }
        }
    }
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < CHAINS; ++i) s ^= x[i];
    sink[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

extern "C" float int_probe(int mode, int iters, int ctas_per_sm) {
    int dev = 0, sms = 0, clk = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint32_t* sink;
    const int T = 256, G = sms * ctas_per_sm;
    cudaMalloc(&sink, (size_t)G * T * 4);
    auto launch = [&](int it) {
        const uint32_t q = 1073479681u, w = 123456789u, ws = (uint32_t)(((uint64_t)w << 32) / q);
        switch (mode) {
            case 0: k_int<0><<<G, T>>>(it, q, w, ws, sink); break;
            case 1: k_int<1><<<G, T>>>(it, q, w, ws, sink); break;
            case 2: k_int<2><<<G, T>>>(it, q, w, ws, sink); break;
            case 3: k_int<3><<<G, T>>>(it, q, w, ws, sink); break;
            case 4: k_int<4><<<G, T>>>(it, q, w, ws, sink); break;
            case 5: k_int<5><<<G, T>>>(it, q, w, ws, sink); break;
            case 6: k_int<6><<<G, T>>>(it, q, w, ws, sink); break;
            default: k_int<7><<<G, T>>>(it, q, w, ws, sink); break;
        }
    };
    launch(16);
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    launch(iters);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);   // kHz (max boost)
    cudaFree(sink);
    // operations (chain steps; butterflies count CHAINS/2 per iteration) per clock per SM
    const double ops = (double)G * T * iters * ((mode == 5 || mode == 7) ? CHAINS / 2 : CHAINS);
    return (float)(ops / (ms * 1e-3) / sms / (clk * 1e3));
}
