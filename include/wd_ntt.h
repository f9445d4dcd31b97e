/*
 * wd_ntt.h -- C ABI of libwdntt.so: batched negacyclic RNS NTT / INTT on B200 (sm_100a).
 *
 * This is the boundary of the WarpDrive hot path: the forward
 * and inverse Number Theoretic Transform over RNS-decomposed CKKS polynomials
 * (section II-B1 Eq.(1); PAPER.md:56 ring R_Q = Z_Q[X]/(X^N+1);
 * PAPER.md:334-352 section IV-C "PE kernel": one launch covers every
 * polynomial and limb), with the plan precompute of PAPER.md:358 section IV-D1.
 *
 * Conventions:
 *   * data layout  [batch][L][N] uint32, row-major: row (b, l) is the residue of
 *     polynomial b modulo primes[l]; rows contiguous, N words each.
 *   * forward      out[i] = sum_j in[j] * psi_l^((2*brv_N(i)+1)*j) mod q_l
 *                  (negacyclic, reading C-1; output in BIT-REVERSED order, C-3)
 *   * inverse      the exact inverse: bit-reversed in, natural order out,
 *                  N^-1 applied (reading C-6)
 *   * psi_l        the minimal primitive 2N-th root of unity mod q_l (C-4)
 *   * values       inputs must be canonical in [0, q_l); outputs are canonical.
 *                  A non-canonical input gives an unspecified result but never
 *                  a fault (reading C-7).
 * No floating point anywhere on the path.
 *
 * Ownership and execution: device pointers are caller-owned (torch tensors),
 * 16-byte aligned.  in == out (in place) is allowed, other overlap is undefined.
 * Calls are stream-ordered and asynchronous on `stream` (a cudaStream_t; NULL =
 * legacy default stream), perform no host synchronisation and no allocation,
 * and are re-entrant across host threads.  A plan is bound to the device that
 * was current at create time and is immutable after creation except for the
 * mode knob; destroy it only after all work using it has completed.
 *
 * Errors: functions returning int return WD_OK (0) or a WD_E* code, and also
 * record it in a thread-local slot read by wd_ntt_last_error().  Asynchronous
 * device faults surface at the caller's next synchronisation on the stream.
 */
#ifndef WD_NTT_H
#define WD_NTT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct wd_ntt_plan wd_ntt_plan;        /* opaque */
typedef struct CUstream_st* wd_stream_t;       /* == cudaStream_t */

/* error codes */
#define WD_OK            0
#define WD_EINVAL        1   /* NULL / misaligned pointer, bad size, wrong device      */
#define WD_EPRIME        2   /* a modulus is not prime, >= 2^30, or != 1 (mod 2N)       */
#define WD_EUNSUPPORTED  3   /* N outside [2, 2^17], L outside [1, 4096], mode n/a      */
#define WD_ECUDA         4   /* CUDA runtime error (no device, launch failure, ...)     */
#define WD_ENOMEM        5   /* device or host allocation failed                        */

/* execution modes (wd_ntt_plan_set_mode) */
#define WD_MODE_AUTO     0   /* library default for this N: = WD_MODE_CUDA on B200       */
#define WD_MODE_CUDA     1   /* CUDA-core radix-2^k butterflies only (WD-BO role): the     *
                              * TMEM-resident kernels "tm" at N = 2^13..2^16 when their    *
                              * rounds of rows are >= 85% full (one row per SM, four per   *
                              * SM at 2^13), else v8 / v5 / v1 (wd_ntt_last_kernel names   *
                              * the one a call ran)                   */
#define WD_MODE_TENSOR   2   /* tcgen05 kind::i8 inner DFTs + CUDA-core epilogue        */
#define WD_MODE_FUSED    3   /* both paths concurrently on the same SMs (WD-FUSE role)  */
#define WD_MODE_CUDA_GEMM 4  /* inner DFTs as 32-bit GEMMs on the CUDA cores (WD-CUDA,   *
                              * PAPER.md:322/401), N = 2^16 only     */
#define WD_MODE_FTC      5   /* WD-FTC: the batch *
                              * split at a polynomial boundary, WD-Tensor on a tensor_share *
                              * of the polynomials and WD-CUDA on the rest, the two running *
                              * concurrently on the same GPU (an internal forked stream,    *
                              * joined back into the caller's stream), N = 2^16 only       */
#define WD_MODE_TC4      6   /* 4-step tcgen05 kernel, warp-specialised: TMA producer, one   *
                              * MMA-issuing thread, CUDA-core epilogue warps working on     *
                              * other tiles at the same time, *
                              * N = 2^16 only                                              */

/*
 * wd_ntt_plan_create -- PAPER.md:358 (initialisation phase: moduli, twiddles
 * precomputed and uploaded ahead of time).
 *   N       transform length, a power of two in [2, 2^17]
 *   primes  host array of L moduli; each must be prime, < 2^30 and = 1 mod 2N
 *           (read during the call only; the caller keeps ownership)
 *   L       number of RNS limbs, 1 <= L <= 4096
 * Returns a plan owning its device tables (16*N*L bytes: forward and inverse
 * psi-power tables in bit-reversed order with Shoup companions; the round-1
 * tensor modes TENSOR / FUSED / CUDA_GEMM / FTC add about 8*N*L more, built on
 * their first wd_ntt_plan_set_mode / wd_ntt_plan_autotune), or NULL with
 * wd_ntt_last_error() set to WD_EINVAL / WD_EPRIME / WD_EUNSUPPORTED / WD_ECUDA /
 * WD_ENOMEM (host or device allocation failure: never an exception).
 * Argument validation happens before any CUDA call, so the WD_EINVAL /
 * WD_EPRIME / WD_EUNSUPPORTED paths work on a machine without a GPU.
 */
wd_ntt_plan* wd_ntt_plan_create(uint32_t N, const uint32_t* primes, uint32_t L);

/* Frees the plan's device tables.  NULL is a no-op.  Caller must have
 * synchronised all work using the plan. */
void wd_ntt_plan_destroy(wd_ntt_plan* plan);

/*
 * wd_ntt_forward / wd_ntt_inverse -- PAPER.md:85-91 (Eq.(1) and its inverse),
 * batched over all (polynomial, limb) rows in ONE launch.
 *   in, out  device pointers to batch*L*N uint32 words, layout [batch][L][N],
 *            16-byte aligned; in == out allowed
 *   batch    number of polynomials (a ciphertext is 2 polynomials);
 *            0 is a successful no-op
 *   stream   cudaStream_t the work is enqueued on
 * Returns WD_OK, WD_EINVAL (NULL plan/pointer, misalignment, wrong device),
 * WD_EUNSUPPORTED (mode not available for this N) or WD_ECUDA (launch error).
 */
int wd_ntt_forward(const wd_ntt_plan* plan, const uint32_t* in, uint32_t* out,
                   uint32_t batch, wd_stream_t stream);
int wd_ntt_inverse(const wd_ntt_plan* plan, const uint32_t* in, uint32_t* out,
                   uint32_t batch, wd_stream_t stream);

/*
 * wd_ntt_forward_host / wd_ntt_inverse_host -- the same transforms on HOST
 * buffers (end-to-end path): copies host->device, transforms, copies back,
 * pipelined in chunks over internal streams so the H2D copy of chunk k+1,
 * the kernel of chunk k and the D2H copy of chunk k-1 overlap.
 *   h_in, h_out  host pointers, batch*L*N words (pinned memory recommended;
 *                pageable works but serialises); h_in == h_out allowed
 *   d_work       caller-owned device scratch of >= batch*L*N words, 16-B aligned
 *   stream       the call is ordered after prior work on `stream`, and work
 *                enqueued on `stream` afterwards is ordered after its end
 * Asynchronous like the device calls: h_out is valid after the caller
 * synchronises `stream`.
 */
int wd_ntt_forward_host(const wd_ntt_plan* plan, const uint32_t* h_in, uint32_t* h_out,
                        uint32_t batch, uint32_t* d_work, wd_stream_t stream);
int wd_ntt_inverse_host(const wd_ntt_plan* plan, const uint32_t* h_in, uint32_t* h_out,
                        uint32_t batch, uint32_t* d_work, wd_stream_t stream);

/*
 * wd_ntt_pointwise_inverse -- SURVEY.md 8 row f1 (NEXT #1): out = INTT(a o b),
 * the negacyclic product of two polynomials given in the NTT domain
 * (PAPER.md:63 HMULT tensor product + PAPER.md:85 "convert polynomial
 * multiplication into point-wise multiplication").  Same layout/stream rules;
 * out may alias a or b.
 */
int wd_ntt_pointwise_inverse(const wd_ntt_plan* plan, const uint32_t* a, const uint32_t* b,
                             uint32_t* out, uint32_t batch, wd_stream_t stream);

/*
 * wd_rescale -- SURVEY.md 8 row f4 (NEXT #4), the CKKS rescale of PAPER.md:81
 * ("RSCALE(ct0) = (a0', b0') in R^2_{Q_{l-1}}"), reading C-18:
 * a' = round(a / q_last) for every polynomial, q_last = the plan's LAST prime,
 * i.e. a'_i = floor((A + floor(q_last/2)) / q_last) mod q_i for the integer
 * (CRT) value A of each coefficient.
 *   in     device, [batch][L][N] NTT-domain residues over the plan's primes
 *          (the forward's bit-reversed order), canonical
 *   out    device, [batch][L-1][N] NTT-domain residues over primes[0..L-2],
 *          canonical; must not overlap `in` or `work`
 *   work   caller-owned device scratch of >= batch*N words (16-B aligned)
 * Three launches: gather the last limb, its INTT, then one forward-NTT launch
 * over all batch*(L-1) output rows with the rescale arithmetic fused into its
 * load and store (PE kernel).  Needs L >= 2, N >= 2^12 and
 * q_last distinct from the other primes (else WD_EUNSUPPORTED); pointer errors
 * give WD_EINVAL.  Stream-ordered and asynchronous like the transforms.
 */
int wd_rescale(const wd_ntt_plan* plan, const uint32_t* in, uint32_t* out, uint32_t batch,
               uint32_t* work, wd_stream_t stream);

/*
 * ModUp / ModDown -- SURVEY.md 8 row f3 (NEXT #3): the KeySwitch basis changes
 * around the NTT (Table III, Fig. 4 "PE kernel"
 * for ModUp and ModDown), in the standard RNS-CKKS form (DESIGN.md reading
 * C-19).  A conversion object pairs a plan over the ciphertext basis
 * Q = {q_0..q_{a-1}} with a plan over the special basis P = {p_0..p_{k-1}}
 * (same N >= 2^12, same device, all a + k primes distinct, a, k <= 64).
 *   BConv_{Q->P}(x)_j = sum_i [x_i (Q/q_i)^-1]_{q_i} (Q/q_i) mod p_j
 *   wd_modup:   in  [batch][a][N]   NTT domain over Q
 *               out [batch][a+k][N] NTT domain over Q then P: the Q limbs of
 *               `in` unchanged, the P limbs NTT_P(BConv(INTT_Q(in)))
 *               work >= batch*a*N words
 *   wd_moddown: in  [batch][a+k][N] NTT domain over Q then P
 *               out [batch][a][N]   (in_Q - NTT_Q(BConv_{P->Q}(INTT_P(in_P)))) * P^-1
 *               work >= batch*(a+k)*N words
 * out must not overlap in or work.  Three launches each (plus one 2-D copy in
 * ModUp), every polynomial of the batch in each.  Errors as for the
 * transforms; wd_rns_conv_create returns NULL (WD_EINVAL: NULL plan or a
 * repeated prime; WD_EUNSUPPORTED: N/device mismatch, N < 2^12, > 64 limbs;
 * WD_ENOMEM).  The conversion object references the two plans: destroy it
 * before them.
 */
typedef struct wd_rns_conv wd_rns_conv;
/*
 * Limb-sharded ModUp (SURVEY.md 8 rows e + f3: the one step of the path with a real exchange).
 * Rank g holds a shard of the Q limbs; plan_q covers that shard and q_all (a_all primes,
 * host array, read during the call) is the whole basis Q.  wd_modup_partial INTTs the local
 * limbs and writes this shard's share of BConv_{Q->P} with the whole-Q constants as
 * canonical residues in 64-bit words, partial [batch][k][N] (device).  The caller sums the
 * shards' partials (an integer all-reduce, e.g. NCCL ncclSum on int64), then
 * wd_modup_finish reduces the sums mod p_j into out_p [batch][k][N] and NTTs them: the P
 * limbs of ModUp, identical on every rank.  ModDown needs no exchange when the P limbs are
 * replicated: wd_moddown on a shard conversion object produces the local Q limbs.
 * wd_modup itself refuses a shard object (WD_EINVAL).  work >= batch*a_local*N words.
 */
wd_rns_conv* wd_rns_conv_create_shard(const wd_ntt_plan* plan_q_local, const wd_ntt_plan* plan_p,
                                      const uint32_t* q_all, uint32_t a_all);
int wd_modup_partial(const wd_rns_conv* conv, const uint32_t* in_local, uint64_t* partial,
                     uint32_t batch, uint32_t* work, wd_stream_t stream);
int wd_modup_finish(const wd_rns_conv* conv, const uint64_t* sum, uint32_t* out_p,
                    uint32_t batch, wd_stream_t stream);
wd_rns_conv* wd_rns_conv_create(const wd_ntt_plan* plan_q, const wd_ntt_plan* plan_p);
void wd_rns_conv_destroy(wd_rns_conv* conv);
int wd_modup(const wd_rns_conv* conv, const uint32_t* in, uint32_t* out, uint32_t batch,
             uint32_t* work, wd_stream_t stream);
int wd_moddown(const wd_rns_conv* conv, const uint32_t* in, uint32_t* out, uint32_t batch,
               uint32_t* work, wd_stream_t stream);

/* ---- queries and knobs ---- */
uint32_t wd_ntt_plan_n(const wd_ntt_plan* plan);
uint32_t wd_ntt_plan_limbs(const wd_ntt_plan* plan);
/* psi actually used for limb `limb` (0 if out of range) -- reading C-4 */
uint32_t wd_ntt_plan_psi(const wd_ntt_plan* plan, uint32_t limb);

/* Host-only helpers of the plan precompute (no GPU needed):
 * wd_ntt_root(q, N): the minimal primitive 2N-th root the plan would use, 0
 * if q fails the prime checks; wd_ntt_check_prime(q, N): WD_OK or WD_EPRIME. */
uint32_t wd_ntt_root(uint32_t q, uint32_t N);
int      wd_ntt_check_prime(uint32_t q, uint32_t N);

/* Select the execution path.  tensor_share in [0,1] is, in WD_MODE_FUSED,
 * the fraction of rows whose column phase runs on the tensor-core warps
 * while the CUDA-core warps run the row phase (the rest of the rows run
 * entirely on the CUDA-core warps).  In WD_MODE_FTC it is the
 * fraction of polynomials given to WD-Tensor (default 0.7, the best of 0.5 / 0.6 / 0.7
 * measured at config 3).  Ignored otherwise; < 0 keeps the plan's default.  Returns WD_OK,
 * WD_EINVAL or WD_EUNSUPPORTED.  Not thread-safe against concurrent calls
 * using the same plan. */
int wd_ntt_plan_set_mode(wd_ntt_plan* plan, int mode, float tensor_share);
int wd_ntt_plan_get_mode(const wd_ntt_plan* plan);

/* Row a9's split "chosen from measurement" (the WD-FUSE ratio follows
 * the units' measured throughput): times one forward + inverse over `batch` polynomials of
 * scratch data (allocated and freed inside the call, zero residues) for every execution path
 * available at this N -- WD_MODE_CUDA, and for N = 2^16 also WD_MODE_FUSED (phase-split
 * pipeline and row splits with tensor_share 0.25 / 0.5 / 0.75), WD_MODE_TENSOR,
 * WD_MODE_CUDA_GEMM, WD_MODE_FTC (at the plan's FTC share) and WD_MODE_TC4 -- with CUDA events on
 * `stream`, and sets the plan to the fastest (building the tensor tables of N = 2^16 first).
 * Writes that path's milliseconds per forward + inverse to *best_ms if best_ms != NULL.
 * Synchronises `stream`.  Returns WD_OK, WD_EINVAL (NULL plan, batch == 0, wrong device) or
 * WD_ECUDA (allocation or launch failure; the plan's mode is then unchanged).  The candidates
 * are timed with an explicit mode each; the plan's mode is written once, at the end, so other
 * streams launching with this plan meanwhile run in the old mode or the new one.  Two concurrent
 * autotune / set_mode calls on one plan are not supported. */
int wd_ntt_plan_autotune(wd_ntt_plan* plan, uint32_t batch, wd_stream_t stream, float* best_ms);

/* Kernel launches issued by the last forward/inverse call on this thread. */
uint32_t wd_ntt_last_launches(void);

/* Name of the kernel family the last forward/inverse call on this thread dispatched to (a static
 * string, never NULL; "" before the first call): "tm" (TMEM-resident rows, N = 2^16), "v8/cl1",
 * "v8/cl2", "v8/cl4", "v8/cl8" (v8 with 1..8-CTA clusters per row), "v5", "v1", "small", "tc4", "tensor",
 * "fused", "cuda_gemm", "ftc".  Diagnostics for benches and tests: which path AUTO took. */
const char* wd_ntt_last_kernel(void);

/* Diagnostics only: while dev_buf (device memory, 20480 uint64 words) is set, every WD_MODE_TC4 launch
 * records clock64() timestamps of CTA 0's pipeline events into it (loads, MMAs, accumulator
 * hand-over, staging hand-over, stores; ntt_tc4.cuh TR_*).  NULL switches it off.  Process-wide. */
void wd_ntt_debug_tc4_trace(void* dev_buf);

int         wd_ntt_last_error(void);
const char* wd_ntt_strerror(int code);
const char* wd_ntt_version(void);

#ifdef __cplusplus
}
#endif
#endif /* WD_NTT_H */
