// wd_ntt.cu -- libwdntt.so: plan precompute, C ABI and dispatch (b).
//
// The ABI is declared and documented in include/wd_ntt.h.  Everything on the call path is
// asynchronous on the caller's stream; the only host<->device copies are the one-time table
// uploads of plan creation and the explicit host-buffer entry points.  The
// kernels live in the k_*.cu translation units behind launch.h; this file holds no device code.
// Environment knobs (WD_NTT_KERNEL, WD_NTT_CL, WD_NTT_LM: A/B runs only) are read once, when a
// plan is created, never on the launch path.
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
#include "launch.h"
#include "plan_math.h"

using namespace wd;

namespace {
thread_local int g_last_error = WD_OK;
thread_local uint32_t g_last_launches = 0;
thread_local const char* g_last_kernel = "";
int set_err(int e) { g_last_error = e; return e; }
}  // namespace

namespace wd {
int build_tensor_tables(TensorTables& tc, uint32_t logN, const std::vector<uint32_t>& primes,
                        const std::vector<uint32_t>& psis);
void free_tensor_tables(TensorTables& t);
}  // namespace wd

struct wd_ntt_plan {
    uint32_t N = 0, logN = 0, L = 0;
    int device = -1;
    int sm_count = 148;
    // A/B knobs, read from the environment once at creation: kernel generation (0 = AUTO; 1, 5, 8
    // force v1, v5, v8), v8 cluster size (0 = AUTO), limb-major row walk
    int kernel_ver = 0;
    int v8_cl = 0;
    uint32_t limb_major = 1;
    int v8_tma = 1;               // v8 column-phase feed (launch.h launch_v8; WD_NTT_V8_TMA)
    V8Occ occ;                     // v8 resident clusters per CL (grid sizing without per-launch queries)
    std::vector<uint32_t> primes, psi;
    uint2* d_fwd = nullptr;        // [L][N]  (psi^brv(i), Shoup)
    uint2* d_inv = nullptr;        // [L][N]  (psi^-brv(i), Shoup)
    LimbConst* d_lc = nullptr;     // [L]
    // N = 2^17 forward through tm (ntt_tmr.cuh H17): the two 2^16 halves as a virtual plan of 2 L limbs,
    // limb' = 2 l + h: [L][2][2^16] re-indexed forward twiddles (local index 2^k + g of half h = Psi[2^(k+1)
    // + h 2^k + g]) and [2 L] LimbConst carrying the first layer's (Psi[1], Shoup) in pad_[0..1]
    uint2* d_fwd17 = nullptr;
    LimbConst* d_lc17 = nullptr;
    uint4* d_rs = nullptr;         // [L] RESCALE constants vs the last prime (ntt_rns.cuh); L >= 2
    uint32_t rs_thr = 0;           // q_last - floor(q_last / 2)
    bool rs_ok = false;            // L >= 2 and q_last differs from every other prime
    TensorTables tc;               // round-1 tensor-path tables (N = 2^16), built on first use
    Tc4Tables t4;                  // 4-step tcgen05 kernel tables (N = 2^16), built on first use
    std::mutex tc_mu;
    int mode = WD_MODE_AUTO;
    float tensor_share = -1.0f;    // FUSED: share of rows whose column phase runs on tcgen05 (< 0: default)
    float ftc_share = 0.7f;        // FTC: polynomials on WD-Tensor (best of 0.5/0.6/0.7 at config 3)
    cudaStream_t hs[3] = {nullptr, nullptr, nullptr};   // host-path pipeline streams
    cudaEvent_t he[4] = {nullptr, nullptr, nullptr, nullptr};
    cudaStream_t fs = nullptr;     // FTC fork stream and its fork / join events
    cudaEvent_t fe[2] = {nullptr, nullptr};
    std::mutex ftc_mu;             // orders fork/join event use across host threads
    std::mutex host_mu;            // the host-buffer pipeline's streams / events are per plan
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

bool tensor_mode(int mode) {
    return mode == WD_MODE_TENSOR || mode == WD_MODE_FUSED || mode == WD_MODE_CUDA_GEMM || mode == WD_MODE_FTC;
}

int ensure_tc4_tables(wd_ntt_plan* p) {
    std::lock_guard<std::mutex> lk(p->tc_mu);
    if (p->t4.ok) return WD_OK;
    if (p->logN != 16) return WD_EUNSUPPORTED;
    int e;
    try {
        e = build_tc4_tables(p->t4, p->primes, p->psi);
    } catch (const std::bad_alloc&) {
        e = WD_ENOMEM;
    }
    if (e != WD_OK) { cudaGetLastError(); free_tc4_tables(p->t4); return e == WD_ENOMEM ? WD_ENOMEM : WD_ECUDA; }
    return WD_OK;
}

// the round-1 tensor tables (TENSOR / FUSED / CUDA_GEMM / FTC), built when one of those modes is first
// selected (they roughly double a plan's device footprint, so AUTO / CUDA plans never pay for them)
int ensure_tensor_tables(wd_ntt_plan* p) {
    std::lock_guard<std::mutex> lk(p->tc_mu);
    if (p->tc.ok) return WD_OK;
    if (p->logN != 16) return WD_EUNSUPPORTED;
    int e;
    try {
        e = build_tensor_tables(p->tc, p->logN, p->primes, p->psi);
    } catch (const std::bad_alloc&) {
        e = WD_ENOMEM;
    }
    if (e != WD_OK) { cudaGetLastError(); free_tensor_tables(p->tc); return e == WD_ENOMEM ? WD_ENOMEM : WD_ECUDA; }
    return WD_OK;
}

// AUTO / CUDA: the measured default CUDA-core kernel per N and row count
int launch_cuda_core(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, cudaStream_t s) {
    const uint32_t logN = p->logN, sm = (uint32_t)p->sm_count;
    if (logN < 12) { launch_v1(logN, fwd, a, rows, s); g_last_kernel = "small"; return 1; }
    int ver = p->kernel_ver;
    // N = 2^13..2^16: tm, the TMEM-resident kernels.  They process rows in rounds of `unit` (one row per
    // SM; four per SM at 2^13), so a last, partly filled round leaves SMs idle for a whole row time.
    //  * a small remainder (<= unit / 4 rows): tm runs the full rounds and v8, with the most CTAs per row,
    //    the remaining schedule slots right after it (the same limb-major slot -> row map);
    //  * otherwise tm alone when its rounds are at least 85% full, else v8, whose 4 CTAs per SM absorb
    //    such a tail (scripts/gpu_tm_rows*.sh, profiles/r02/tm/)
    // N = 2^17 forward: tm on the two 2^16 halves of every row (ntt_tmr.cuh H17; 2 rows per 2^17 row),
    // when those half-row rounds are at least 85% full.  Out of place only: both halves read the whole
    // input row (the first layer pairs them) on different SMs at different times, so in place one half's
    // output could overwrite input the other still has to read.  The inverse stays on v8 (its last layer
    // joins the halves).
    if ((ver == 0 || ver == 20) && logN == 17 && fwd && p->d_fwd17 && a.in != a.out && !a.in2 && !a.aux && !a.cpy &&
        !a.in_ls && !a.out_ls && !a.slot0 && !a.nb_total) {
        const uint64_t r2 = 2ull * rows, u = (uint64_t)sm;
        if ((ver == 20 || (r2 >= u && r2 * 20 >= u * ((r2 + u - 1) / u) * 17)) && r2 <= 0x7fffffffull) {
            NttArgs ah = a;
            ah.L = 2 * a.L; ah.tw = p->d_fwd17; ah.lc = p->d_lc17;
            const int n = launch_tmr17(ah, (uint32_t)r2, p->sm_count, s);
            if (n > 0) { g_last_kernel = "tm17"; return n; }
        }
    }
    bool tm_tail = false;
    uint64_t tm_unit = 0;
    if (ver == 0 && logN >= 13 && logN <= 16) {
        tm_unit = (uint64_t)sm * (logN == 13 ? 4 : 1);
        const uint64_t tail = rows % tm_unit;
        if (rows >= tm_unit && tail * 4 <= tm_unit) { ver = 20; tm_tail = tail != 0; }
        else if ((uint64_t)rows * 20 >= tm_unit * ((rows + tm_unit - 1) / tm_unit) * 17) ver = 20;
    }
    if (ver == 0) {
        if ((logN == 15 || logN == 16) && rows < sm / 4) ver = 5;        // v5: the row in a cluster's DSMEM
        else if (rows >= sm || logN >= 15) ver = 8;
        else ver = 1;                                                   // N <= 2^14, few rows
    }
    if (ver == 20 && logN >= 13 && logN <= 16) {                      // tm: TMEM-resident rows
        if (tm_tail) {
            const uint32_t tail = (uint32_t)(rows % tm_unit);
            NttArgs am = a;
            am.nb_total = rows / a.L;                                   // the whole batch's slot map
            const int n = launch_tmr(logN, fwd, am, rows - tail, p->sm_count, s);
            if (n > 0) {
                NttArgs at = am;
                at.slot0 = rows - tail;
                launch_v8(logN, fwd, at, tail, std::min(8, 1 << ((int)logN - 12)), 0, p->occ, p->v8_tma, s);
                g_last_kernel = "tm+v8";
                return n + 1;
            }
        } else {
            const int n = launch_tmr(logN, fwd, a, rows, p->sm_count, s);
            if (n > 0) { g_last_kernel = "tm"; return n; }
        }
        ver = 8;
    }
    if (ver == 5 && logN >= 14) { launch_v5(logN, fwd, a, rows, p->sm_count, s); g_last_kernel = "v5"; return 1; }
    if (ver == 1 || ver == 5) { launch_v1(logN, fwd, a, rows, s); g_last_kernel = "v1"; return 1; }
    int cl = p->v8_cl;
    if (!cl) {
        cl = 2;
        // few rows (<= half the SM count, e.g. one ciphertext at L = 36): 8-CTA clusters put ~4 CTAs
        // per SM to work on them (config 2: 2105 -> 2485 KOPS, profiles/r01/f4)
        if (logN >= 15 && rows * 8 <= sm * 4) cl = 8;
        // N = 2^13, 2^14 with many rows: the whole row per CTA (s13 +8.6%, s14 +3.7%)
        else if (logN <= 14 && rows >= 8u * sm) cl = 1;
        // between half and one SM count of rows: 4-CTA clusters (config 5 sweep)
        else if (logN >= 15 && rows <= sm) cl = 4;
    }
    launch_v8(logN, fwd, a, rows, cl, 0, p->occ, p->v8_tma, s);
    {
        const int cm = std::max(1, std::min(cl, 1 << std::min<int>(3, (int)logN - 12)));   // launch_v8's clamp
        g_last_kernel = cm == 8 ? "v8/cl8" : cm == 4 ? "v8/cl4" : cm == 2 ? "v8/cl2" : "v8/cl1";
    }
    return 1;
}

// v8 with a RESCALE / ModDown store map (EPI 1 / 2) or a plain v8 launch at the default cluster size
void launch_v8_default(const wd_ntt_plan* p, bool fwd, const NttArgs& a, uint32_t rows, int epi, cudaStream_t s) {
    launch_v8(p->logN, fwd, a, rows, p->logN > 12 ? 2 : 1, epi, p->occ, p->v8_tma, s);
}

int effective_mode(const wd_ntt_plan* p) { return p->mode == WD_MODE_AUTO ? WD_MODE_CUDA : p->mode; }

// one transform call in an explicit mode (the plan's own mode for the ABI calls; autotune passes its
// candidates here instead of rewriting the plan's mode while other streams may be launching)
int run_mode(const wd_ntt_plan* p, int mode, float share, bool fwd, const uint32_t* in, const uint32_t* in2,
             uint32_t* out, uint32_t batch, cudaStream_t s) {
    g_last_launches = 0;
    if (!p || !in || !out) return set_err(WD_EINVAL);
    if (((uintptr_t)in | (uintptr_t)out | (uintptr_t)in2) & 15) return set_err(WD_EINVAL);
    if (batch == 0) return set_err(WD_OK);
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != p->device) return set_err(WD_EINVAL);
    const uint64_t rows64 = (uint64_t)batch * p->L;
    if (rows64 > 0x7fffffffull) return set_err(WD_EINVAL);
    const uint32_t rows = (uint32_t)rows64;
    NttArgs a;
    a.in = in; a.in2 = in2; a.out = out; a.tw = fwd ? p->d_fwd : p->d_inv; a.lc = p->d_lc; a.L = p->L;
    a.limb_major = p->limb_major;
    if (mode == WD_MODE_AUTO) mode = WD_MODE_CUDA;
    int launches = 0;
    if (in2 != nullptr || mode == WD_MODE_CUDA) {
        launches = launch_cuda_core(p, fwd, a, rows, s);
    } else if (mode == WD_MODE_TC4) {
        if (!p->t4.ok) return set_err(WD_EUNSUPPORTED);
        if (fwd) { launches = launch_tc4(fwd, a, p->t4, rows, p->sm_count, s); g_last_kernel = "tc4"; }
        else launches = launch_cuda_core(p, fwd, a, rows, s);          // inverse kernel: not yet built
        if (launches == -2) return set_err(WD_ECUDA);
        if (launches < 0) return set_err(WD_EUNSUPPORTED);
    } else {
        if (!p->tc.ok) return set_err(WD_EUNSUPPORTED);
        if (mode == WD_MODE_CUDA_GEMM) {
            launch_wdcuda(fwd, a, p->tc, rows, p->sm_count, s);
            launches = 1;
            g_last_kernel = "cuda_gemm";
        } else if (mode == WD_MODE_TENSOR) {
            launches = launch_tensor(fwd, a, p->tc, rows, p->sm_count, s);
            g_last_kernel = "tensor";
        } else if (mode == WD_MODE_FUSED) {
            launches = launch_fused(fwd, a, p->tc, rows, p->sm_count, share, s);
            g_last_kernel = "fused";
        } else if (mode == WD_MODE_FTC) {
            g_last_kernel = "ftc";
            // WD-FTC: split at a polynomial boundary (rows stay limb-aligned), WD-Tensor on the first
            // bt polynomials in a forked stream, WD-CUDA on the rest in `s`, then join.
            const uint32_t bt = std::min<uint32_t>(batch, (uint32_t)std::lround(p->ftc_share * batch));
            NttArgs ac = a;
            const size_t off = (size_t)bt * p->L * p->N;
            ac.in = a.in + off; ac.out = a.out + off;
            if (bt == 0) {
                launch_wdcuda(fwd, ac, p->tc, rows, p->sm_count, s);
                launches = 1;
            } else if (bt == batch) {
                launches = launch_tensor(fwd, a, p->tc, rows, p->sm_count, s);
            } else {
                wd_ntt_plan* pm = const_cast<wd_ntt_plan*>(p);   // the mutex only, never the plan state
                std::lock_guard<std::mutex> lk(pm->ftc_mu);
                cudaEventRecord(p->fe[0], s);
                cudaStreamWaitEvent(p->fs, p->fe[0], 0);
                const int n1 = launch_tensor(fwd, a, p->tc, bt * p->L, p->sm_count, p->fs);
                launch_wdcuda(fwd, ac, p->tc, (batch - bt) * p->L, p->sm_count, s);
                cudaEventRecord(p->fe[1], p->fs);
                cudaStreamWaitEvent(s, p->fe[1], 0);
                launches = n1 + 1;
            }
        } else {
            return set_err(WD_EUNSUPPORTED);
        }
        if (launches < 0) return set_err(WD_EUNSUPPORTED);
    }
    if (cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    g_last_launches = (uint32_t)launches;
    return set_err(WD_OK);
}

int run(const wd_ntt_plan* p, bool fwd, const uint32_t* in, const uint32_t* in2, uint32_t* out, uint32_t batch,
        cudaStream_t s) {
    if (!p) return set_err(WD_EINVAL);
    return run_mode(p, p->mode, p->tensor_share, fwd, in, in2, out, batch, s);
}

int run_host(const wd_ntt_plan* pc, bool fwd, const uint32_t* h_in, uint32_t* h_out, uint32_t batch,
             uint32_t* d_work, cudaStream_t s) {
    if (!pc || !h_in || !h_out || !d_work || ((uintptr_t)d_work & 15)) return set_err(WD_EINVAL);
    if (batch == 0) return set_err(WD_OK);
    wd_ntt_plan* p = const_cast<wd_ntt_plan*>(pc);   // the per-plan pipeline streams / mutex only
    std::lock_guard<std::mutex> lk(p->host_mu);
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != p->device) return set_err(WD_EINVAL);
    const size_t row_words = (size_t)p->L * p->N;
    // chunk boundaries are multiples of g polynomials, g the smallest count whose words are a
    // multiple of 4 (every chunk's device offset stays 16-byte aligned, as run() requires)
    uint32_t g = 1;
    while ((g * row_words) % 4) ++g;
    // chunks of >= g polynomials: H2D(k+1) || kernel(k) || D2H(k-1).  The first H2D and the last D2H
    // are not overlapped, so a call costs ~(nch+1)/nch of one copy direction: 8 chunks for small
    // jobs, up to 32 chunks of ~32 MB for large ones.
    const size_t total_bytes = (size_t)batch * row_words * 4;
    const uint32_t want = (uint32_t)std::min<size_t>(32, std::max<size_t>(8, total_bytes >> 25));
    const uint32_t units = (batch + g - 1) / g;
    const uint32_t nch = std::max<uint32_t>(1, std::min<uint32_t>(units, want));
    cudaEventRecord(p->he[3], s);
    uint32_t total = 0;
    uint32_t b0 = 0;
    int err = WD_OK;
    for (uint32_t k = 0; k < nch && err == WD_OK; ++k) {
        const uint32_t b1 = std::min<uint32_t>(batch, (uint32_t)((uint64_t)units * (k + 1) / nch) * g);
        if (b1 <= b0) continue;
        const uint32_t nb = b1 - b0;
        cudaStream_t st = p->hs[k % 3];
        if (k < 3) cudaStreamWaitEvent(st, p->he[3], 0);
        const size_t off = (size_t)b0 * row_words, bytes = (size_t)nb * row_words * 4;
        cudaMemcpyAsync(d_work + off, h_in + off, bytes, cudaMemcpyHostToDevice, st);
        err = run(p, fwd, d_work + off, nullptr, d_work + off, nb, st);
        if (err != WD_OK) break;                 // nothing more is enqueued; the join below still runs
        total += g_last_launches;
        cudaMemcpyAsync(h_out + off, d_work + off, bytes, cudaMemcpyDeviceToHost, st);
        b0 = b1;
    }
    // join: the caller's stream waits for every pipeline stream, also after an error, so work
    // already in flight stays ordered before anything the caller enqueues next
    for (int i = 0; i < 3; ++i) {
        cudaEventRecord(p->he[i], p->hs[i]);
        cudaStreamWaitEvent(s, p->he[i], 0);
    }
    if (err != WD_OK) return set_err(err);
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
        cudaFree(p->d_fwd17); cudaFree(p->d_lc17);
        free_tensor_tables(p->tc);
        free_tc4_tables(p->t4);
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

    // ---- host precompute (a1): psi, bit-reversed psi-power tables + Shoup companions.  Host
    // allocation failures (about 16 N L bytes here) return NULL with WD_ENOMEM, never throw.
    std::vector<uint2> fwd, inv;
    std::vector<LimbConst> lc;
    try {
    p->primes.assign(primes, primes + L);
    fwd.resize((size_t)L * N); inv.resize((size_t)L * N); lc.resize(L);
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
    } catch (const std::bad_alloc&) {
        delete p; set_err(WD_ENOMEM); return nullptr;
    }

    // ---- device upload (the only H2D copy of the plan's life)
    if (cudaGetDevice(&p->device) != cudaSuccess) { cudaGetLastError(); p->device = -1; delete p; set_err(WD_ECUDA); return nullptr; }
    cudaDeviceGetAttribute(&p->sm_count, cudaDevAttrMultiProcessorCount, p->device);
    // A/B knobs: read here once, never on the launch path.  Unknown generations keep AUTO.
    if (const char* ev = getenv("WD_NTT_KERNEL")) {
        const int v = ev[0] == 'v' ? atoi(ev + 1) : (ev[0] == 't' && ev[1] == 'm') ? 20 : 0;
        if (v == 1 || v == 5 || v == 8 || v == 20) p->kernel_ver = v;
    }
    if (const char* ev = getenv("WD_NTT_CL")) p->v8_cl = atoi(ev) >= 8 ? 8 : atoi(ev) >= 4 ? 4 : atoi(ev) >= 2 ? 2 : 1;
    if (const char* ev = getenv("WD_NTT_LM")) p->limb_major = atoi(ev) != 0;
    if (const char* ev = getenv("WD_NTT_V8_TMA")) p->v8_tma = atoi(ev) & 7;
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
    if (p->logN == 17) {   // the virtual half plan of the tm forward (same table bytes as d_fwd)
        try {
            const uint32_t H = N / 2;
            std::vector<uint2> h17((size_t)L * N);
            std::vector<LimbConst> l17(2 * (size_t)L);
            for (uint32_t l = 0; l < L; ++l) {
                const uint2* f = fwd.data() + (size_t)l * N;
                for (uint32_t hh = 0; hh < 2; ++hh) {
                    uint2* d = h17.data() + ((size_t)l * 2 + hh) * H;
                    d[0] = make_uint2(0, 0);
                    for (uint32_t k = 0; (1u << k) < H; ++k)
                        for (uint32_t g = 0; g < (1u << k); ++g) d[(1u << k) + g] = f[(2u << k) + (hh << k) + g];
                    LimbConst c = lc[l];
                    c.pad_[0] = f[1].x; c.pad_[1] = f[1].y;
                    l17[2 * l + hh] = c;
                }
            }
            if (cudaMalloc(&p->d_fwd17, tb) != cudaSuccess || cudaMalloc(&p->d_lc17, sizeof(LimbConst) * 2 * L) != cudaSuccess ||
                cudaMemcpy(p->d_fwd17, h17.data(), tb, cudaMemcpyHostToDevice) != cudaSuccess ||
                cudaMemcpy(p->d_lc17, l17.data(), sizeof(LimbConst) * 2 * L, cudaMemcpyHostToDevice) != cudaSuccess) {
                cudaGetLastError(); free_plan(p); set_err(WD_ENOMEM); return nullptr;
            }
        } catch (const std::bad_alloc&) {
            free_plan(p); set_err(WD_ENOMEM); return nullptr;
        }
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
    for (auto& s : p->hs) if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess) { free_plan(p); set_err(WD_ECUDA); return nullptr; }
    for (auto& e : p->he) if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) { free_plan(p); set_err(WD_ECUDA); return nullptr; }
    if (cudaStreamCreateWithFlags(&p->fs, cudaStreamNonBlocking) != cudaSuccess) { free_plan(p); set_err(WD_ECUDA); return nullptr; }
    for (auto& e : p->fe) if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) { free_plan(p); set_err(WD_ECUDA); return nullptr; }
    if (prep_cc(p->logN) || prep_v8(p->logN, p->sm_count, &p->occ) || prep_rns() ||
        (p->logN >= 13 && p->logN <= 17 && prep_tmr()) ||
        (p->logN == 16 && (prep_tensor() || prep_wdcuda() || prep_tc4()))) {
        cudaGetLastError(); free_plan(p); set_err(WD_ECUDA); return nullptr;
    }
    p->mode = WD_MODE_AUTO;
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
    launch_rs_gather(in, work, N, L, batch, p->sm_count, s);
    // K2: INTT of the last limb (a 1-limb view of the plan's tables), in place in work
    NttArgs ai;
    ai.in = work; ai.in2 = nullptr; ai.out = work; ai.tw = p->d_inv + (size_t)(L - 1) * N; ai.lc = p->d_lc + (L - 1); ai.L = 1;
    uint32_t launches = 1 + (uint32_t)launch_cuda_core(p, false, ai, batch, s);
    // K3: forward NTT of every output row with the rescale load / store maps (v8, EPI = 1)
    NttArgs af;
    af.in = work; af.in2 = nullptr; af.out = out; af.tw = p->d_fwd; af.lc = p->d_lc; af.L = L - 1;
    af.aux = in; af.rs = p->d_rs; af.rs_thr = p->rs_thr; af.Lfull = L;
    const uint32_t rows = batch * (L - 1);
    launch_v8_default(p, true, af, rows, 1, s);
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
    if (pq->logN >= 12) {
        // v8 copies the Q limbs (NTT domain, unchanged) into out as it stages them: one read of
        // the input instead of two (the separate 2-D copy cost ~0.4 ms at config 3)
        ai.cpy = out; ai.cpy_ls = a + k;
        launch_v8_default(pq, false, ai, batch * a, 0, s);
        launches = 1;
    } else {
        launches = (uint32_t)launch_cuda_core(pq, false, ai, batch * a, s);
        // the Q limbs pass through unchanged (NTT domain)
        if (cudaMemcpy2DAsync(out, (size_t)(a + k) * N * 4, in, (size_t)a * N * 4, (size_t)a * N * 4, batch,
                              cudaMemcpyDeviceToDevice, s) != cudaSuccess) { cudaGetLastError(); return set_err(WD_ECUDA); }
    }
    // K2: BConv Q -> P into the P section of out (coefficient domain)
    BconvTab t{c->d_up_src, c->d_up_w, c->d_up_dst, a, k};
    launch_bconv(work, a, out, a + k, a, t, N, batch, pq->sm_count, s);
    // K3: forward NTT of the P section in place (rows strided by a + k)
    NttArgs af;
    af.in = out + (size_t)a * N; af.in2 = nullptr; af.out = out + (size_t)a * N; af.tw = pp->d_fwd; af.lc = pp->d_lc;
    af.L = k; af.in_ls = a + k; af.out_ls = a + k;
    launch_v8_default(pp, true, af, batch * k, 0, s);
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
    launch_bconv_partial(work, a, partial, t, pq->N, batch, pq->sm_count, s);
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
    launch_reduce64(sum, out_p, c->d_up_dst, pp->L, pp->N, rows, pp->sm_count, s);
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
    launch_v8_default(pp, false, ai, batch * k, 0, s);
    // K2: BConv P -> Q (coefficient domain) -> wq
    BconvTab t{c->d_dn_src, c->d_dn_w, c->d_dn_dst, k, a};
    launch_bconv(wp, k, wq, a, 0, t, N, batch, pq->sm_count, s);
    // K3: forward NTT over Q with the store map out = (in_Q - NTT(wq)) * P^-1 (v8, EPI = 2)
    NttArgs af;
    af.in = wq; af.in2 = nullptr; af.out = out; af.tw = pq->d_fwd; af.lc = pq->d_lc; af.L = a;
    af.aux = in; af.rs = c->d_pinv; af.Lfull = a + k;
    launch_v8_default(pq, true, af, batch * a, 2, s);
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
    if (!p || mode < WD_MODE_AUTO || mode > WD_MODE_TC4) return set_err(WD_EINVAL);
    if (tensor_share > 1.0f) return set_err(WD_EINVAL);
    if (mode == WD_MODE_TC4) {
        if (p->logN != 16) return set_err(WD_EUNSUPPORTED);
        const int e = ensure_tc4_tables(p);
        if (e != WD_OK) return set_err(e);
    }
    if (tensor_mode(mode)) {
        if (p->logN != 16) return set_err(WD_EUNSUPPORTED);
        const int e = ensure_tensor_tables(p);
        if (e != WD_OK) return set_err(e);
    }
    p->mode = mode;
    if (tensor_share >= 0.0f) {
        if (mode == WD_MODE_FTC) p->ftc_share = tensor_share;
        else p->tensor_share = tensor_share;
    }
    return set_err(WD_OK);
}
int wd_ntt_plan_get_mode(const wd_ntt_plan* p) { return p ? effective_mode(p) : -1; }

// Times every execution path the plan supports on `batch` scratch polynomials and keeps the fastest.
// Candidates run through run_mode with an explicit mode: the plan's mode changes once, at the end.
int wd_ntt_plan_autotune(wd_ntt_plan* p, uint32_t batch, wd_stream_t st, float* best_ms) {
    if (!p || batch == 0) return set_err(WD_EINVAL);
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev != p->device) return set_err(WD_EINVAL);
    if ((uint64_t)batch * p->L > 0x7fffffffull) return set_err(WD_EINVAL);
    if (p->logN == 16) {
        int e = ensure_tensor_tables(p);
        if (e == WD_OK) e = ensure_tc4_tables(p);
        if (e != WD_OK) return set_err(e);
    }
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
    if (p->logN == 16 && p->tc.ok) {
        for (float sh : {-1.0f, 0.25f, 0.5f, 0.75f}) cands.push_back({WD_MODE_FUSED, sh});
        cands.push_back({WD_MODE_TENSOR, p->tensor_share});
        cands.push_back({WD_MODE_CUDA_GEMM, p->tensor_share});
        cands.push_back({WD_MODE_FTC, p->tensor_share});
    }
    if (p->logN == 16 && p->t4.ok) cands.push_back({WD_MODE_TC4, p->tensor_share});
    int best = -1;
    float best_t = 0.0f;
    for (size_t i = 0; i < cands.size(); ++i) {
        const int m = cands[i].mode;
        const float sh = cands[i].share;
        auto pair = [&]() {
            return run_mode(p, m, sh, true, x, nullptr, y, batch, s) == WD_OK &&
                   run_mode(p, m, sh, false, y, nullptr, x, batch, s) == WD_OK;
        };
        bool ok = pair();                                // one warm-up pair, then 3 timed pairs
        float t = 0.0f;
        if (ok) {
            cudaEventRecord(e0, s);
            for (int k = 0; k < 3 && ok; ++k) ok = pair();
            cudaEventRecord(e1, s);
            ok = ok && cudaEventSynchronize(e1) == cudaSuccess && cudaEventElapsedTime(&t, e0, e1) == cudaSuccess;
        }
        if (!ok) {
            if (cudaGetLastError() != cudaSuccess || m == WD_MODE_CUDA) { cleanup(); return set_err(WD_ECUDA); }
            continue;                                    // this path is unsupported here: skip it
        }
        t /= 3.0f;
        if (best < 0 || t < best_t) { best = (int)i; best_t = t; }
    }
    cleanup();
    p->mode = cands[best].mode;
    if (cands[best].mode == WD_MODE_FUSED) p->tensor_share = cands[best].share;
    if (best_ms) *best_ms = best_t;
    return set_err(WD_OK);
}

uint32_t wd_ntt_last_launches(void) { return g_last_launches; }
const char* wd_ntt_last_kernel(void) { return g_last_kernel; }

void wd_ntt_debug_tc4_trace(void* dev_buf) { tc4_set_trace(dev_buf); }

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
