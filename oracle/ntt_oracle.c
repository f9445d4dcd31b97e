/*
 * ntt_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU reference for the batched negacyclic
 * RNS NTT/INTT (the WarpDrive hot path).  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this file's
 * shared object.  It shares no code, header, table or constant generator with
 * the CUDA library under paper_conf_hpca_fanzzfzdtksy25_b200/csrc/.
 *
 * What it computes:
 *   forward:  out[i] = sum_j x[j] * psi^((2*brv(i)+1)*j)  mod q
 *             -- PAPER.md:85-89 Eq.(1) made negacyclic (reading C-1),
 *                output in bit-reversed order (reading C-3);
 *   inverse:  the exact inverse, N^-1 applied (reading C-6);
 *   psi:      the minimal primitive 2N-th root of unity mod q (reading C-4),
 *             found by a plain linear scan: smallest g >= 2 with g^N = -1.
 * Every value is canonical in [0, q).  All arithmetic is (uint64)a*b % q.
 *
 * Algorithm: the textbook iterative merged-psi Cooley-Tukey forward transform
 * and Gentleman-Sande inverse (Longa-Naehrig), every twiddle recomputed with
 * a plain powmod -- no tables, no lazy reduction, no blocking.
 *
 * Pins (tests/test_oracle.py): an O(N^2) Python big-int evaluation of the
 * definition, the round trip, the negacyclic convolution theorem against a
 * schoolbook product mod X^N+1, the special cases (delta -> ones, X -> the
 * distinct roots of X^N+1), the sum rule sum_i out[i] = N*x[0], a hand-worked
 * N=4, q=17 example (tests/golden/), and exhaustive minimality of psi.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

static uint64_t mulmod(uint64_t a, uint64_t b, uint64_t q) { return (a * b) % q; }

uint32_t orc_powmod(uint32_t a, uint64_t e, uint32_t q) {
    uint64_t r = 1 % q, b = a % q;
    while (e) {
        if (e & 1) r = mulmod(r, b, q);
        b = mulmod(b, b, q);
        e >>= 1;
    }
    return (uint32_t)r;
}

/* Deterministic Miller-Rabin; bases {2, 7, 61} are exact for n < 2^32. */
int orc_is_prime(uint32_t n) {
    static const uint32_t bases[3] = {2, 7, 61};
    if (n < 2) return 0;
    for (int i = 0; i < 3; ++i) if (n == bases[i]) return 1;
    if (n % 2 == 0) return 0;
    uint32_t d = n - 1; int s = 0;
    while ((d & 1) == 0) { d >>= 1; ++s; }
    for (int i = 0; i < 3; ++i) {
        uint64_t x = orc_powmod(bases[i] % n, d, n);
        if (x == 1 || x == n - 1) continue;
        int comp = 1;
        for (int r = 1; r < s; ++r) {
            x = mulmod(x, x, n);
            if (x == n - 1) { comp = 0; break; }
        }
        if (comp) return 0;
    }
    return 1;
}

/* Smallest g >= 2 with g^N = -1 (mod q): the minimal primitive 2N-th root. 0 if none. */
uint32_t orc_psi_min(uint32_t q, uint32_t N) {
    for (uint64_t g = 2; g < q; ++g)
        if (orc_powmod((uint32_t)g, N, q) == q - 1) return (uint32_t)g;
    return 0;
}

uint32_t orc_brv(uint32_t i, int logn) {
    uint32_t r = 0;
    for (int b = 0; b < logn; ++b) { r = (r << 1) | (i & 1); i >>= 1; }
    return r;
}

static int ilog2(uint32_t n) { int l = 0; while ((1u << l) < n) ++l; return l; }

/* In place: natural-order coefficients -> evaluations in bit-reversed order. */
void orc_ntt_forward(uint32_t* a, uint32_t N, uint32_t q, uint32_t psi) {
    int logn = ilog2(N);
    uint32_t t = N;
    for (uint32_t m = 1; m < N; m <<= 1) {
        t >>= 1;
        for (uint32_t i = 0; i < m; ++i) {
            uint64_t S = orc_powmod(psi, orc_brv(m + i, logn), q);
            uint32_t j1 = 2 * i * t;
            for (uint32_t j = j1; j < j1 + t; ++j) {
                uint64_t U = a[j], V = mulmod(a[j + t], S, q);
                a[j] = (uint32_t)((U + V) % q);
                a[j + t] = (uint32_t)((U + q - V) % q);
            }
        }
    }
}

/* In place: bit-reversed evaluations -> natural-order coefficients (times N^-1). */
void orc_ntt_inverse(uint32_t* a, uint32_t N, uint32_t q, uint32_t psi) {
    int logn = ilog2(N);
    uint32_t psi_inv = orc_powmod(psi, q - 2, q);
    uint32_t t = 1;
    for (uint32_t m = N >> 1; m >= 1; m >>= 1) {
        for (uint32_t i = 0; i < m; ++i) {
            uint64_t S = orc_powmod(psi_inv, orc_brv(m + i, logn), q);
            uint32_t j1 = 2 * i * t;
            for (uint32_t j = j1; j < j1 + t; ++j) {
                uint64_t U = a[j], V = a[j + t];
                a[j] = (uint32_t)((U + V) % q);
                a[j + t] = (uint32_t)mulmod((U + q - V) % q, S, q);
            }
        }
        t <<= 1;
        if (m == 1) break;
    }
    uint64_t n_inv = orc_powmod(N % q, q - 2, q);
    for (uint32_t j = 0; j < N; ++j) a[j] = (uint32_t)mulmod(a[j], n_inv, q);
}

/* ---- batched driver: rows [batch][L][N], one transform per task, pthreads ---- */
typedef struct {
    int dir; const uint32_t* in; uint32_t* out; uint32_t N;
    const uint32_t* primes; const uint32_t* psis; uint32_t L;
    uint64_t first, last;
} job_t;

static void* run_job(void* arg) {
    job_t* j = (job_t*)arg;
    for (uint64_t r = j->first; r < j->last; ++r) {
        uint32_t l = (uint32_t)(r % j->L);
        uint32_t* row = j->out + r * j->N;
        if (j->in != j->out) memcpy(row, j->in + r * j->N, sizeof(uint32_t) * j->N);
        if (j->dir >= 0) orc_ntt_forward(row, j->N, j->primes[l], j->psis[l]);
        else orc_ntt_inverse(row, j->N, j->primes[l], j->psis[l]);
    }
    return NULL;
}

/* dir = +1 forward, -1 inverse.  in may equal out.  Returns 0. */
int orc_ntt_batch(int dir, const uint32_t* in, uint32_t* out, uint32_t N,
                  const uint32_t* primes, const uint32_t* psis, uint32_t L,
                  uint32_t batch, int nthreads) {
    uint64_t rows = (uint64_t)batch * L;
    if (nthreads < 1) nthreads = 1;
    if ((uint64_t)nthreads > rows) nthreads = (int)(rows ? rows : 1);
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * nthreads);
    job_t* jobs = (job_t*)malloc(sizeof(job_t) * nthreads);
    for (int t = 0; t < nthreads; ++t) {
        jobs[t] = (job_t){dir, in, out, N, primes, psis, L,
                          rows * t / nthreads, rows * (t + 1) / nthreads};
        pthread_create(&th[t], NULL, run_job, &jobs[t]);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    free(th); free(jobs);
    return 0;
}
