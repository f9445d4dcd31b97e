// fp64_probe.cu -- can the FP64 pipe take the Shoup quotient off the fma pipe?
//
// The tm kernel is bound by the fma pipe: per butterfly one IMAD.HI (quarter rate) and
// two IMADs (half rate).  B200 (sm_100a, unlike sm_103a) keeps a half-rate FP64 pipe, so the quotient
// estimate e ~ a w / q can come from one DFMA instead:
//     d = 2^52 + a                    (the double with high word 0x43300000 and low word a: exact)
//     r = fma(d, wq, C)               wq = floor(w 2^52 / q) / 2^52,  C = 2^52 - 2^52 wq (an integer)
//                                     = 2^52 + a wq rounded once to the integer grid
//     e = low word of r               in {floor(a w / q), floor(a w / q) + 1}  (|a wq - a w / q| < 2^-20)
//     t = a w - e q  (mod 2^32)       in [-q, q)
// This probe measures modmul throughput (independent chains, 1024 threads per SM, all SMs) for the Shoup
// form and the DFMA form, and checks the DFMA form's range claim on random inputs.
// build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o fp64_probe scripts/fp64_probe.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

constexpr int CH = 8;   // independent chains per thread

__global__ void __launch_bounds__(1024, 1) shoup_loop(uint32_t* out, uint32_t w, uint32_t ws, uint32_t q, int iters) {
    uint32_t a[CH];
#pragma unroll
    for (int j = 0; j < CH; ++j) a[j] = threadIdx.x * 7919u + j * 104729u + blockIdx.x;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < CH; ++j) {
            const uint32_t hq = __umulhi(a[j], ws);
            a[j] = a[j] * w - hq * q;              // [0, 2q)
        }
    }
    uint32_t s = 0;
#pragma unroll
    for (int j = 0; j < CH; ++j) s ^= a[j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void __launch_bounds__(1024, 1) dfma_loop(uint32_t* out, uint32_t w, double wq, double C, uint32_t q, int iters) {
    uint32_t a[CH];
#pragma unroll
    for (int j = 0; j < CH; ++j) a[j] = threadIdx.x * 7919u + j * 104729u + blockIdx.x;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < CH; ++j) {
            const double d = __hiloint2double(0x43300000, (int)a[j]);
            const uint32_t e = (uint32_t)__double2loint(fma(d, wq, C));
            a[j] = a[j] * w - e * q + q;           // [0, 2q)
        }
    }
    uint32_t s = 0;
#pragma unroll
    for (int j = 0; j < CH; ++j) s ^= a[j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// range check: t = a w - e q in [-q, q) and t = a w mod q (mod q), for random a < 2^32, w < q
__global__ void dfma_check(uint32_t* bad, uint32_t q, uint64_t seed, int n) {
    uint64_t x = seed + (uint64_t)(blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B97F4A7C15ull;
    for (int i = 0; i < n; ++i) {
        x += 0x9E3779B97F4A7C15ull;
        uint64_t z = x;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z ^= z >> 31;
        const uint32_t a = (uint32_t)z, w = (uint32_t)((z >> 32) % q);
        const uint64_t W52 = (uint64_t)(((unsigned __int128)w << 52) / q);
        const double wq = (double)W52 / 4503599627370496.0, C = (double)((1ull << 52) - W52);
        const double d = __hiloint2double(0x43300000, (int)a);
        const uint32_t e = (uint32_t)__double2loint(fma(d, wq, C));
        const int64_t t = (int64_t)a * w - (int64_t)e * q;
        if (t < -(int64_t)q || t >= (int64_t)q || (uint64_t)((t % q + q) % q) != ((uint64_t)a * w) % q) atomicAdd(bad, 1u);
    }
}

int main() {
    int dev = 0, sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    const uint32_t q = 1073479681u;   // a 30-bit NTT prime (q = 1 mod 2^17)
    const uint32_t w = 123456789u % q;
    const uint32_t ws = (uint32_t)(((uint64_t)w << 32) / q);
    const uint64_t W52 = (uint64_t)(((unsigned __int128)w << 52) / q);
    const double wq = (double)W52 / 4503599627370496.0, C = (double)((1ull << 52) - W52);
    uint32_t *out, *bad;
    cudaMalloc(&out, sizeof(uint32_t) * sms * 1024);
    cudaMalloc(&bad, 4);
    cudaMemset(bad, 0, 4);
    dfma_check<<<sms, 256>>>(bad, q, 12345, 4096);
    dfma_check<<<sms, 256>>>(bad, 998244353u, 777, 4096);
    dfma_check<<<sms, 256>>>(bad, 65537u, 31, 4096);
    uint32_t hb = 0;
    cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost);
    printf("dfma_check: %u bad of %d samples\n", hb, 3 * sms * 256 * 4096);
    const int iters = 4096;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int rep = 0; rep < 2; ++rep) {
        for (int k = 0; k < 2; ++k) {
            if (k == 0) shoup_loop<<<sms, 1024>>>(out, w, ws, q, 64);
            else dfma_loop<<<sms, 1024>>>(out, w, wq, C, q, 64);
            cudaEventRecord(e0);
            if (k == 0) shoup_loop<<<sms, 1024>>>(out, w, ws, q, iters);
            else dfma_loop<<<sms, 1024>>>(out, w, wq, C, q, iters);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms = 0;
            cudaEventElapsedTime(&ms, e0, e1);
            const double mm = (double)sms * 1024 * CH * iters;
            printf("%s: %.3f ms, %.2f Gmodmul/s, %.2f modmul/clk/SM (at %d MHz nominal)\n", k ? "dfma " : "shoup",
                   ms, mm / ms / 1e6, mm / (ms * 1e-3) / sms / (clk * 1e3), clk / 1000);
        }
    }
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
