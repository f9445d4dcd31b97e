#!/usr/bin/env python
"""bench.py -- batched negacyclic RNS NTT/INTT throughput on B200 (BASELINE.json metric).

Contract (task statement / DESIGN.md "Measurement"):
  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl wd|reference] [--mode auto|cuda|tensor|fused|cuda_gemm|ftc]
A STEP = one pass of the whole hot path over one batch: forward NTT of every
(polynomial, limb) row, then the inverse NTT of the result (config 3 of
BASELINE.json: N=2^16, L=36, 64 ciphertexts = 128 polynomials = 4608 rows per
direction).  value = KOPS = 1e-3 x single-prime N-point transforms per second
(SURVEY.md reading C-9), counting both directions, summed over all ranks
(weak scaling: every rank owns its own 64-ciphertext batch; the limbs and
ciphertexts are independent so there is no collective inside the step).
Inputs (1.2 GB) are larger than L2 (126 MB), so no explicit flush is needed.
Rank 0 prints ONE JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
if "WORLD_SIZE" in os.environ:            # under torchrun: NCCL communicator lines for the driver's rank check
    os.environ.setdefault("NCCL_DEBUG", "INFO")
    os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")

CONFIGS = {
    # name: (logN, L, ciphertexts)
    "c1": (12, 4, None),       # 1 polynomial (configs[0]; oracle in seconds)
    "c2": (16, 36, 1),
    "c3": (16, 36, 64),        # headline (BASELINE.json metric / configs[2])
    "c4": (17, 48, 32),
    # batch-1 small cases (config 5's "batch 1" end): kernel-selection data, not bench lines
    "t15": (15, 36, 1),
    "t16": (16, 16, 1),
    "t17": (17, 36, 1),
}
# config 5 (the N sweep, BASELINE configs[4]) at batch 128 polynomials, 16 limbs: parity cases
# and kernel-selection data, not bench lines
for _lg in range(12, 18):
    CONFIGS["s%d" % _lg] = (_lg, 16, 64)
CONFIG_NAMES = {"c1": "config1 (BASELINE configs[0])", "c2": "config2 (one ciphertext)",
                "c3": "config3 (BASELINE configs[2], headline)", "c4": "config4 per-GPU shard"}
CONFIG_NAMES.update({"t15": "config5 point N=2^15, L=36, one ciphertext", "t16": "config5 point N=2^16, L=16, one ciphertext",
                    "t17": "config5 point N=2^17, L=36, one ciphertext"})
CONFIG_NAMES.update({"s%d" % _lg: "config5 sweep point N=2^%d, L=16, 128 polynomials" % _lg for _lg in range(12, 18)})
METRIC = "NTT KOPS (N=2^16, L=36) at 1/2/4/8 B200; % of HBM / int8 tensor roofline"
FALLBACK_HBM_GBS = 6650.0
BFLY_PER_CLK_SM = 13.57       # measured: scripts/int_probe.cu ct_bfly_hi, 4 CTAs/SM (profiles/r01/int_probe.jsonl)


def i8_peak():
    """Measured tcgen05 kind::i8 peak (scripts/tc4_probe.cu, committed under profiles/r02)."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "r02", "peaks_i8.json")))
        return float(d["int8_tcgen05_peak_TMAC_per_s"]), float(d.get("n64_TMAC_per_s", 0.0)), "measured"
    except Exception:
        return 2250.0, 0.0, "nominal (4.5 POPS dense int8)"


# int8 tensor MACs per N-point transform, per mode: every radix-16 byte-plane GEMM stage multiplies
# 16 coefficients x 4 data bytes by 16 outputs x 4 byte planes, i.e. 256 MACs per output element
# (SURVEY.md 8 row a5); N = 2^16 has 4 such stages (TENSOR, tc4 forward), FUSED runs the column
# phase's two stages on tcgen05 (rows with the tensor share), WD-CUDA / CUDA none.
def tensor_macs_per_transform(mode: str, n: int, fwd: bool) -> float:
    if n != 1 << 16:
        return 0.0
    stages = {"tensor": 4, "tc4": 4 if fwd else 0, "fused": 2, "ftc": 4 * 0.7}.get(mode, 0)
    return 256.0 * n * stages


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except Exception:
        return {"hbm_gbs": FALLBACK_HBM_GBS, "bf16_tflops": 1590.0}, "fallback"


class ClockSampler:
    """Samples SM clock and throttle reasons with NVML during the timed region."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
        0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
        0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, dev_index: int, period: float = 0.01):
        self.samples, self.reasons, self.stop_ev = [], set(), threading.Event()
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None
        self.period = period
        self.th = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        while not self.stop_ev.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.nv:
            self.th.start()
        return self

    def __exit__(self, *a):
        self.stop_ev.set()
        if self.nv:
            self.th.join()

    def summary(self):
        s = sorted(self.samples)
        return {"sm_mhz": (s[len(s) // 2] if s else None), "sm_max_mhz": self.max_mhz,
                "samples": len(s), "reasons": sorted(self.reasons)}


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def oracle_kops(logn: int, L: int, seconds: float = 12.0):
    """Time the CPU oracle (as it stands) on a bounded sample of the workload."""
    import oracle
    from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs
    threads = oracle.default_threads()
    primes = inputs.bench_primes(L)
    n = 1 << logn
    x = inputs.uniform_residues(primes, n, 1, inputs.SEED_BASE + 2)[0]      # one polynomial, all limbs
    for q in primes:
        oracle.psi_min(q, n)                                                 # psi search: plan time, not timed
    done, t0 = 0, time.perf_counter()
    while True:
        k = max(1, min(L, threads))
        rows = x[:k][None]
        y = oracle.ntt_forward(rows, primes[:k], threads=threads)
        oracle.ntt_inverse(y, primes[:k], threads=threads)
        done += 2 * k
        el = time.perf_counter() - t0
        if el >= seconds:
            break
    return {"value": done / el / 1e3, "unit": "KOPS", "cores": threads, "kind": "oracle",
            "sample": "%d N=2^%d transforms (fwd+inv pairs over the first %d limbs of one polynomial of the "
                      "workload, %d threads) in %.1f s on %s" % (done, logn, min(L, threads), threads, el,
                                                                   cpu_model())}


def run_reference(args):
    """--impl reference: the oracle on the host cores, same metric/config (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    logn, L, nct = CONFIGS[args.config]
    import oracle
    from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs
    oracle.build()
    threads = oracle.default_threads()
    primes = inputs.bench_primes(L)
    n = 1 << logn
    x = inputs.uniform_residues(primes, n, 1, inputs.SEED_BASE + 2)[0]
    for q in primes:
        oracle.psi_min(q, n)
    k = max(1, min(L, threads))             # rows per step: one bounded sample of the workload
    def step():
        y = oracle.ntt_forward(x[:k][None], primes[:k], threads=threads)
        oracle.ntt_inverse(y, primes[:k], threads=threads)
    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    el = time.perf_counter() - t0
    v = 2 * k * args.steps / el / 1e3
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "KOPS", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": el / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": "N=2^%d L=%d, bounded sample: %d rows fwd+inv per step" % (logn, L, k),
                   "N": n, "L": L},
        "cpu_baseline": {"value": v, "unit": "KOPS", "cores": threads, "kind": "oracle",
                         "sample": "%d rows (N=2^%d) forward+inverse per step, %d threads, %s" % (k, logn, threads,
                                                                                                  cpu_model())},
        "e2e": {"value": v, "unit": "KOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def run_rescale(args):
    """--op rescale: CKKS RESCALE (wd_rescale, row f4) of a batch of polynomials, config shape
    (default c3: N=2^16, L=36 -> 35 limbs, 128 polynomials).  One step = one rescale of every
    polynomial; value = polynomials rescaled per second.  Roofline: HBM, algorithmic bytes =
    read L*N*4 + write (L-1)*N*4 per polynomial (the work buffer round trip of the last limb,
    4*N*4 bytes, is overhead, not algorithmic)."""
    import torch
    from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
    torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", "0")))
    logn, L, nct = CONFIGS[args.config]
    n = 1 << logn
    batch = 1 if nct is None else 2 * nct
    primes = inputs.bench_primes(L)
    plan = wdntt.Plan(n, primes)
    x = inputs.uniform_residues_torch(primes, n, batch, inputs.SEED_BASE + 2, device="cuda")
    out = torch.empty((batch, L - 1, n), dtype=x.dtype, device="cuda")
    work = torch.empty((batch, n), dtype=x.dtype, device="cuda")
    sp = torch.cuda.current_stream().cuda_stream
    for _ in range(max(3, args.warmup)):
        wdntt.wd_rescale(plan.handle, x, out, batch, work, sp)
    torch.cuda.synchronize()
    launches = 0
    with ClockSampler(0) as clk:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.steps):
            wdntt.wd_rescale(plan.handle, x, out, batch, work, sp)
            launches += wdntt.wd_ntt_last_launches()
        e1.record()
        torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.steps
    pk, pk_kind = peaks()
    hbm = float(pk.get("hbm_gbs", FALLBACK_HBM_GBS))
    alg = batch * n * 4.0 * (2 * L - 1)
    line = {"metric": "CKKS RESCALE throughput (N=2^%d, L=%d -> %d)" % (logn, L, L - 1),
            "value": batch / (ms / 1e3), "unit": "polynomials/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic (splitmix64 uniform residues)",
            "us_per_ciphertext": 2 * ms * 1e3 / batch,
            "config": {"workload": "%s: rescale of %d polynomials" % (CONFIG_NAMES[args.config], batch),
                       "N": n, "L": L, "polys": batch},
            "roofline": {"bound": "hbm", "kernel": "whole op (3 launches)", "achieved": alg / (ms / 1e3) / 1e9,
                         "peak": hbm, "unit": "GB/s", "frac": alg / (ms / 1e3) / 1e9 / hbm, "traffic": None,
                         "peak_kind": pk_kind, "algorithmic_bytes_per_step": alg},
            "gpu_launches": launches, "clocks": clk.summary()}
    print(json.dumps(line), flush=True)


def run_modupdown(args):
    """--op modup|moddown: the KeySwitch basis changes (row f3) at the config shape (default c3:
    N=2^16, a = L = 36 ciphertext limbs, k = --k special primes, 128 polynomials).  One step = one
    ModUp (a -> a+k limbs) or ModDown (a+k -> a) of every polynomial; value = polynomials/s.
    Roofline: HBM, algorithmic bytes = read + write of the polynomial (ModUp: a*N*4 in,
    (a+k)*N*4 out; ModDown: (a+k)*N*4 in, a*N*4 out)."""
    import torch
    from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
    torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", "0")))
    logn, a, nct = CONFIGS[args.config]
    n = 1 << logn
    batch = 1 if nct is None else 2 * nct
    allp = inputs.bench_primes(a + args.k)
    qs, ps = allp[:a], allp[a:]
    pq, pp = wdntt.Plan(n, qs), wdntt.Plan(n, ps)
    conv = wdntt.RnsConv(pq, pp)
    up = args.op == "modup"
    lin, lout = (a, a + args.k) if up else (a + args.k, a)
    x = inputs.uniform_residues_torch(qs if up else allp, n, batch, inputs.SEED_BASE + 2, device="cuda")
    out = torch.empty((batch, lout, n), dtype=x.dtype, device="cuda")
    work = torch.empty((batch, a + args.k, n), dtype=x.dtype, device="cuda")
    sp = torch.cuda.current_stream().cuda_stream
    fn = wdntt.wd_modup if up else wdntt.wd_moddown
    for _ in range(max(3, args.warmup)):
        fn(conv.handle, x, out, batch, work, sp)
    torch.cuda.synchronize()
    launches = 0
    with ClockSampler(0) as clk:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.steps):
            fn(conv.handle, x, out, batch, work, sp)
            launches += wdntt.wd_ntt_last_launches()
        e1.record()
        torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.steps
    pk, pk_kind = peaks()
    hbm = float(pk.get("hbm_gbs", FALLBACK_HBM_GBS))
    alg = batch * n * 4.0 * (lin + lout)
    line = {"metric": "CKKS %s throughput (N=2^%d, %d -> %d limbs)" % ("ModUp" if up else "ModDown", logn, lin, lout),
            "value": batch / (ms / 1e3), "unit": "polynomials/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic (splitmix64 uniform residues)",
            "config": {"workload": "%s: %s of %d polynomials, a=%d, k=%d" % (CONFIG_NAMES[args.config], args.op, batch,
                                                                           a, args.k), "N": n, "polys": batch},
            "roofline": {"bound": "hbm", "kernel": "whole op", "achieved": alg / (ms / 1e3) / 1e9, "peak": hbm,
                         "unit": "GB/s", "frac": alg / (ms / 1e3) / 1e9 / hbm, "traffic": None, "peak_kind": pk_kind,
                         "algorithmic_bytes_per_step": alg},
            "gpu_launches": launches, "clocks": clk.summary()}
    print(json.dumps(line), flush=True)


def run_polymul(args):
    """--op polymul: the negacyclic polynomial product c = INTT(NTT(a) o NTT(b)) mod (X^N + 1, q_l)
    of SURVEY.md 8 row f1 (the HMULT tensor-product step), at the config shape (default c3:
    N=2^16, L=36, 128 polynomial pairs).  One step = two forward launches and one fused
    pointwise-product + inverse launch over every pair; value = polynomial products per second.
    Roofline: HBM, algorithmic bytes = read a and b, write c (12*N bytes per row); the three
    launches move 28*N bytes per row (the NTT-domain operands round-trip through HBM)."""
    import torch
    from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
    torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", "0")))
    logn, L, nct = CONFIGS[args.config]
    n = 1 << logn
    batch = 1 if nct is None else 2 * nct
    primes = inputs.bench_primes(L)
    plan = wdntt.Plan(n, primes)
    xa = inputs.uniform_residues_torch(primes, n, batch, inputs.SEED_BASE + 2, device="cuda")
    xb = inputs.uniform_residues_torch(primes, n, batch, inputs.SEED_BASE + 3, device="cuda")
    ya, yb, c = torch.empty_like(xa), torch.empty_like(xa), torch.empty_like(xa)
    sp = torch.cuda.current_stream().cuda_stream

    def step():
        wdntt.wd_ntt_forward(plan.handle, xa, ya, batch, sp)
        n0 = wdntt.wd_ntt_last_launches()
        wdntt.wd_ntt_forward(plan.handle, xb, yb, batch, sp)
        n1 = wdntt.wd_ntt_last_launches()
        wdntt.wd_ntt_pointwise_inverse(plan.handle, ya, yb, c, batch, sp)
        return n0 + n1 + wdntt.wd_ntt_last_launches()

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize()
    launches = 0
    with ClockSampler(0) as clk:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.steps):
            launches += step()
        e1.record()
        torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.steps
    pk, pk_kind = peaks()
    hbm = float(pk.get("hbm_gbs", FALLBACK_HBM_GBS))
    alg = batch * L * n * 12.0
    line = {"metric": "negacyclic polynomial multiply throughput (N=2^%d, L=%d)" % (logn, L),
            "value": batch / (ms / 1e3), "unit": "polynomial products/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic (splitmix64 uniform residues)",
            "config": {"workload": "%s: %d polynomial pairs, NTT(a), NTT(b), fused pointwise product + INTT"
                                   % (CONFIG_NAMES[args.config], batch), "N": n, "L": L, "polys": batch},
            "roofline": {"bound": "hbm", "kernel": "whole op (3 launches)", "achieved": alg / (ms / 1e3) / 1e9,
                         "peak": hbm, "unit": "GB/s", "frac": alg / (ms / 1e3) / 1e9 / hbm, "traffic": None,
                         "peak_kind": pk_kind, "algorithmic_bytes_per_step": alg},
            "gpu_launches": launches, "clocks": clk.summary()}
    print(json.dumps(line), flush=True)


def run_shard(args):
    """--shard limbs (SURVEY.md 8 row e; BASELINE configs[3]: N=2^17, L=48, limbs sharded over 2/4/8
    GPUs).  Rank g owns limbs [g L / G, (g+1) L / G) of ONE batch and builds its own plan over those
    primes; the NTT has no collective (limbs are independent).  Reported separately:
      value           the resident-shard rate: every rank transforms its shard, inputs already in
                      HBM, K steps of forward + inverse, barrier + max over ranks
      scatter_gather  the same step with NCCL moving the data: rank 0 holds the whole batch, scatters
                      the limb slices, every rank transforms, rank 0 gathers the results"""
    import torch
    import torch.distributed as dist
    from paper_conf_hpca_fanzzfzdtksy25_b200 import dist as wdist
    from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local), rank=rank, world_size=world,
                            init_method="env://" if "MASTER_ADDR" in os.environ else "tcp://127.0.0.1:%d" % (29500 + os.getpid() % 1000))
    logn, L, nct = CONFIGS[args.config]
    n = 1 << logn
    batch = 1 if nct is None else 2 * nct
    primes = inputs.bench_primes(L)
    spans = [wdist.limb_range(L, world, g) for g in range(world)]
    l0, l1 = spans[rank]
    lg = l1 - l0
    plan = wdntt.Plan(n, primes[l0:l1])
    plan.set_mode(args.mode, args.share)
    full = inputs.uniform_residues_torch(primes, n, batch, inputs.SEED_BASE + 3, device="cuda")
    x = full[:, l0:l1].contiguous()
    y, z = torch.empty_like(x), torch.empty_like(x)
    sp = torch.cuda.current_stream().cuda_stream
    stream = torch.cuda.current_stream()

    def step():
        wdntt.wd_ntt_forward(plan.handle, x, y, batch, sp)
        a = wdntt.wd_ntt_last_launches()
        wdntt.wd_ntt_inverse(plan.handle, y, z, batch, sp)
        return a + wdntt.wd_ntt_last_launches()

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize()
    assert torch.equal(z, x), "round trip failed"
    dist.barrier()
    torch.cuda.synchronize()
    launches = 0
    with ClockSampler(local) as clk:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            launches += step()
        e1.record(stream)
        torch.cuda.synchronize()
    t = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device="cuda")
    dist.barrier()
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())
    kops = 2 * batch * L * args.steps / (ms / 1e3) / 1e3

    # ---- scatter + transform + gather through NCCL (rank 0 owns the whole batch; dist.py helpers,
    # the same code the gloo CPU tests run)
    sg_steps = max(1, min(args.steps, 5))
    src_full = full if rank == 0 else None
    result = {}

    def sg_step():
        xl = wdist.scatter_limbs(src_full, L, n, batch, src=0)
        wdntt.wd_ntt_forward(plan.handle, xl, y, batch, sp)
        wdntt.wd_ntt_inverse(plan.handle, y, z, batch, sp)
        result["full"] = wdist.gather_limbs(z, L, n, batch, dst=0)

    sg_step()
    torch.cuda.synchronize()
    if rank == 0:
        assert torch.equal(result["full"], full), "scatter/gather round trip failed"
    dist.barrier()
    torch.cuda.synchronize()
    g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    g0.record(stream)
    for _ in range(sg_steps):
        sg_step()
    g1.record(stream)
    torch.cuda.synchronize()
    tg = torch.tensor([g0.elapsed_time(g1)], dtype=torch.float64, device="cuda")
    dist.all_reduce(tg, op=dist.ReduceOp.MAX)
    sg_ms = float(tg.item())
    if rank == 0:
        pk, pk_kind = peaks()
        hbm = float(pk.get("hbm_gbs", FALLBACK_HBM_GBS))
        per_rank_ms = ms / args.steps / 2
        alg = 8.0 * n * batch * lg
        line = {
            "metric": METRIC, "value": kops, "unit": "KOPS", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic (splitmix64 uniform residues, SURVEY.md 8.d)",
            "config": {"workload": "%s: N=2^%d, L=%d limbs of %d polynomials sharded over %d GPU(s) (%s limbs per "
                                   "rank), forward+inverse per step" % (CONFIG_NAMES.get(args.config, args.config), logn,
                                                                         L, batch, world, "/".join(
                                                                             str(b_ - a_) for a_, b_ in spans)),
                       "N": n, "L": L, "polys": batch, "mode": args.mode, "parallelism": "limb shards, no collective in the NTT",
                       "l2": "shard %.2f GB per rank" % (batch * lg * n * 4 / 1e9)},
            "roofline": {"bound": "hbm", "kernel": "forward+inverse average (rank 0)",
                         "achieved": alg / (per_rank_ms / 1e3) / 1e9, "peak": hbm, "unit": "GB/s",
                         "frac": alg / (per_rank_ms / 1e3) / 1e9 / hbm, "traffic": None, "peak_kind": pk_kind},
            "scatter_gather": {"value": 2 * batch * L * sg_steps / (sg_ms / 1e3) / 1e3, "unit": "KOPS",
                               "ms_per_step": sg_ms / sg_steps, "bytes_scattered_per_step": batch * L * n * 4,
                               "bytes_gathered_per_step": batch * L * n * 4,
                               "api": "torch.distributed scatter/gather (NCCL) around wd_ntt_forward/inverse"},
            "gpu_launches": launches, "clocks": clk.summary(),
            "e2e": {"value": 2 * batch * L * sg_steps / (sg_ms / 1e3) / 1e3, "unit": "KOPS",
                    "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0,
                    "note": "device-resident full batch on rank 0; the data movement is the NCCL scatter + gather"},
        }
        print(json.dumps(line), flush=True)
    dist.destroy_process_group()


def main():
    if os.environ.get("WD_BENCH_WATCHDOG"):                    # debugging hangs: dump all stacks, exit
        import faulthandler
        faulthandler.dump_traceback_later(float(os.environ["WD_BENCH_WATCHDOG"]), exit=True)
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="wd", choices=["wd", "reference"])
    ap.add_argument("--mode", default="auto", choices=["auto", "cuda", "tensor", "fused", "cuda_gemm", "ftc", "tc4"])
    ap.add_argument("--shard", default="none", choices=["none", "limbs"],
                    help="limbs: under torchrun every rank owns L/G limbs of ONE batch (config 4's split); "
                         "reports the resident-shard rate and the scatter + gather end to end separately")
    ap.add_argument("--share", type=float, default=-1.0, help="tensor share for --mode fused / ftc")
    ap.add_argument("--config", default="c3", choices=sorted(CONFIGS))
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--graph", default="auto", choices=["auto", "on", "off"],
                    help="time each direction's K launches as one CUDA graph (auto: L2-resident configs)")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--op", default="ntt", choices=["ntt", "rescale", "modup", "moddown", "polymul"],
                    help="ntt: the headline forward+inverse step; rescale: SURVEY.md 8 row f4; "
                         "modup / moddown: row f3 (KeySwitch basis changes); polymul: row f1")
    ap.add_argument("--k", type=int, default=1, help="special primes for --op modup/moddown (PAPER.md Table III: K=1)")
    args = ap.parse_args()
    if args.op == "rescale":
        run_rescale(args)
        return
    if args.op in ("modup", "moddown"):
        run_modupdown(args)
        return
    if args.op == "polymul":
        run_polymul(args)
        return

    if args.impl == "reference":
        run_reference(args)
        return
    if args.shard == "limbs":
        run_shard(args)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    logn, L, nct = CONFIGS[args.config]
    n = 1 << logn
    batch = 1 if nct is None else 2 * nct            # polynomials (1 ciphertext = 2 polynomials)
    primes = inputs.bench_primes(L)
    rows = batch * L
    plan = wdntt.Plan(n, primes)
    plan.set_mode(args.mode, args.share)
    x = inputs.uniform_residues_torch(primes, n, batch, inputs.SEED_BASE + 2 + 97 * rank, device="cuda")
    y = torch.empty_like(x)
    z = torch.empty_like(x)
    stream = torch.cuda.current_stream()
    sp = stream.cuda_stream

    kern = {}

    def step():
        wdntt.wd_ntt_forward(plan.handle, x, y, batch, sp)
        lf = wdntt.wd_ntt_last_launches()
        kern["forward"] = wdntt.wd_ntt_last_kernel()
        wdntt.wd_ntt_inverse(plan.handle, y, z, batch, sp)
        kern["inverse"] = wdntt.wd_ntt_last_kernel()
        return lf + wdntt.wd_ntt_last_launches()

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize()
    assert torch.equal(z, x), "round trip failed"

    # ---- timed region: K steps, per-launch events on the launching stream
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches = 0
    # Latency-bound (L2-resident) configs: the K launches of each direction are captured in one
    # CUDA graph each, so the timed region measures the GPU rather than the host's launch rate
    # (the harness rule: capture launch-bound inner loops in CUDA graphs).  Large configs keep
    # eager per-launch events.
    use_graph = args.graph == "on" or (args.graph == "auto" and rows * n * 4 <= 126e6)
    if use_graph:
        cs = torch.cuda.Stream()
        cs.wait_stream(stream)
        gf, gi = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
        with torch.cuda.graph(gf, stream=cs):
            for _ in range(args.steps):
                wdntt.wd_ntt_forward(plan.handle, x, y, batch, cs.cuda_stream)
                launches += wdntt.wd_ntt_last_launches()
        with torch.cuda.graph(gi, stream=cs):
            for _ in range(args.steps):
                wdntt.wd_ntt_inverse(plan.handle, y, z, batch, cs.cuda_stream)
                launches += wdntt.wd_ntt_last_launches()
        gf.replay(); gi.replay()                     # warm the graphs
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        with ClockSampler(local) as clk:
            t_start = torch.cuda.Event(enable_timing=True)
            t_mid = torch.cuda.Event(enable_timing=True)
            t_end = torch.cuda.Event(enable_timing=True)
            t_start.record(stream)
            gf.replay()
            t_mid.record(stream)
            gi.replay()
            t_end.record(stream)
            torch.cuda.synchronize()
        ms = t_start.elapsed_time(t_end)
        fwd_ms = t_start.elapsed_time(t_mid) / args.steps
        inv_ms = t_mid.elapsed_time(t_end) / args.steps
        assert torch.equal(z, x), "round trip failed (graph)"
    else:
      with ClockSampler(local) as clk:
        t_start = torch.cuda.Event(enable_timing=True)
        t_end = torch.cuda.Event(enable_timing=True)
        t_start.record(stream)
        for k in range(args.steps):
            ev[k][0].record(stream)
            wdntt.wd_ntt_forward(plan.handle, x, y, batch, sp)
            launches += wdntt.wd_ntt_last_launches()
            ev[k][1].record(stream)
            wdntt.wd_ntt_inverse(plan.handle, y, z, batch, sp)
            launches += wdntt.wd_ntt_last_launches()
            ev[k][2].record(stream)
        t_end.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    if not use_graph:
        ms = t_start.elapsed_time(t_end)
        fwd_ms = float(np.mean([e[0].elapsed_time(e[1]) for e in ev]))
        inv_ms = float(np.mean([e[1].elapsed_time(e[2]) for e in ev]))
    t = torch.tensor([ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    total_transforms = 2 * rows * args.steps * world
    kops = total_transforms / (ms_max / 1e3) / 1e3

    # ---- end to end through the host-buffer C-ABI calls (pinned host memory)
    e2e = None
    if args.e2e_steps > 0:
        hx = torch.empty(x.shape, dtype=torch.int32, pin_memory=True)
        hx.copy_(x)
        hy = torch.empty_like(hx, pin_memory=True)
        work = y                                  # device scratch: the bench's own output buffer
        def e2e_step():
            wdntt.wd_ntt_forward_host(plan.handle, hx, hy, batch, work, sp)
            wdntt.wd_ntt_inverse_host(plan.handle, hy, hy, batch, work, sp)      # in place on the host
        e2e_step()
        torch.cuda.synchronize()
        assert torch.equal(hy, hx), "host-buffer round trip failed"
        if world > 1:
            dist.barrier()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        for _ in range(args.e2e_steps):
            e2e_step()
        a1.record(stream)
        torch.cuda.synchronize()
        te = torch.tensor([a0.elapsed_time(a1)], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        bytes_step = 2 * rows * n * 4            # two host calls, each copies the batch in and out
        e2e = {"value": 2 * rows * args.e2e_steps * world / (float(te.item()) / 1e3) / 1e3, "unit": "KOPS",
               "h2d_bytes_per_step": bytes_step, "d2h_bytes_per_step": bytes_step,
               "steps": args.e2e_steps, "api": "wd_ntt_forward_host + wd_ntt_inverse_host (pinned host buffers)"}
        # the PCIe bound: the same bytes as bare pinned copies, H2D and D2H on two streams at once
        s_h, s_d = torch.cuda.Stream(), torch.cuda.Stream()
        c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        c0.record(stream)
        s_h.wait_stream(stream); s_d.wait_stream(stream)
        for _ in range(2):
            with torch.cuda.stream(s_h):
                work.copy_(hx, non_blocking=True)
            with torch.cuda.stream(s_d):
                hy.copy_(x, non_blocking=True)
        stream.wait_stream(s_h); stream.wait_stream(s_d)
        c1.record(stream)
        torch.cuda.synchronize()
        copy_ms = c0.elapsed_time(c1)            # 2 x batch bytes each way = one e2e step's copies
        e2e["pcie_bound"] = {"value": 2 * rows / (copy_ms / 1e3) / 1e3, "unit": "KOPS",
                             "copy_ms_per_step": copy_ms,
                             "note": "bare pinned H2D || D2H of one step's bytes, no kernels"}
        e2e["frac_of_pcie_bound"] = e2e["value"] / world / e2e["pcie_bound"]["value"]
        del hx, hy

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    pk, pk_kind = peaks()
    hbm = float(pk.get("hbm_gbs", FALLBACK_HBM_GBS))
    sms = torch.cuda.get_device_properties(local).multi_processor_count
    dom_ms, dom_name = (fwd_ms, "forward") if fwd_ms >= inv_ms else (inv_ms, "inverse")
    alg_bytes = 8.0 * n * rows                       # read 4N + write 4N bytes per transform
    achieved = alg_bytes / (dom_ms / 1e3) / 1e9
    # DRAM traffic of the dominant launch: NOT measured in this run (that needs ncu); taken from the
    # committed ncu --set full capture of the same launch and labelled with its source
    traffic, traffic_src = None, None
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        key = "%s_%s_%s" % (args.config, args.mode, dom_name)
        traffic = tr.get(key)
        traffic_src = tr.get("_source", {}).get(key) if traffic is not None else None
    except Exception:
        pass
    i8_pk, i8_pk64, i8_kind = i8_peak()
    macs_f = tensor_macs_per_transform(args.mode, n, True) * rows
    macs_i = tensor_macs_per_transform(args.mode, n, False) * rows
    tmacs = max(macs_f / (fwd_ms / 1e3), macs_i / (inv_ms / 1e3)) / 1e12
    line = {
        "metric": METRIC, "value": kops, "unit": "KOPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic (splitmix64 uniform residues, SURVEY.md 8.d)",
        "config": {"workload": "%s: N=2^%d, L=%d, %s polynomials per GPU, forward+inverse per step"
                               % (CONFIG_NAMES[args.config], logn, L, batch), "N": n, "L": L, "polys_per_gpu": batch,
                   "rows_per_direction_per_gpu": rows, "mode": args.mode,
                   "l2": ("inputs %.2f GB > 126 MB L2, no flush needed" % (rows * n * 4 / 1e9)
                          if rows * n * 4 > 126e6 else "inputs %.1f MB are L2-resident (latency-bound small case)"
                          % (rows * n * 4 / 1e6)),
                   "parallelism": "limb/ciphertext independent, weak scaling, no collective",
                   "timing": ("one CUDA graph of K launches per direction (launch-bound config)" if use_graph
                              else "eager launches, CUDA events around every launch")},
        "fwd_kops": rows * world / (fwd_ms / 1e3) / 1e3, "inv_kops": rows * world / (inv_ms / 1e3) / 1e3,
        "fwd_ms": fwd_ms, "inv_ms": inv_ms,
        "kernels": kern,
        "roofline": {"bound": "hbm", "kernel": "%s (%s)" % (dom_name, kern.get(dom_name, "?")), "achieved": achieved,
                     "peak": hbm, "unit": "GB/s",
                     "frac": achieved / hbm, "traffic": traffic, "traffic_source": traffic_src,
                     "peak_kind": "%s (MEASURED_PEAKS.json hbm_gbs copy bandwidth)" % pk_kind,
                     "algorithmic_bytes_per_launch": alg_bytes},
        # int8 tensor pipe: algorithmic byte-plane MACs of the launch / time / the measured kind::i8 peak
        # (M=128 N=256 back-to-back MMAs; the N=64 tile shape of the NTT stages peaks at n64_peak)
        "roofline_tensor": {"bound": "tensor", "achieved": tmacs, "peak": i8_pk, "unit": "TMAC/s (int8)",
                            "frac": tmacs / i8_pk, "n64_peak": i8_pk64, "peak_kind": i8_kind,
                            "macs_per_launch": {"forward": macs_f, "inverse": macs_i},
                            "note": "0 for modes without tcgen05 work (cuda = tm / v8 butterflies)"},
        # the bound that actually limits a Shoup-butterfly kernel on B200: the fma pipe (IMAD.HI at
        # quarter rate + 2 IMAD per butterfly); peak = the measured butterfly rate of a pure
        # register-resident butterfly loop (scripts/int_probe.cu, profiles/r01/int_probe.jsonl:
        # 13.6 butterflies/clk/SM) x SMs x the SM clock measured during the timed region
        "roofline_alu": {"bound": "alu", "kernel": "%s (%s)" % (dom_name, kern.get(dom_name, "?")),
                         "achieved": (n // 2) * logn * rows / (dom_ms / 1e3) / 1e9,
                         "peak": BFLY_PER_CLK_SM * sms * (clk.summary()["sm_mhz"] or 1965) / 1e3,
                         "unit": "G butterflies/s",
                         "frac": (n // 2) * logn * rows / (dom_ms / 1e3) / 1e9
                                 / (BFLY_PER_CLK_SM * sms * (clk.summary()["sm_mhz"] or 1965) / 1e3),
                         "note": "algorithmic butterflies (N/2 log2 N per transform); the WD-CUDA and tensor "
                                 "modes do other work per element, for them this is a normalised rate"},
        "gpu_launches": launches,
        "clocks": clk.summary(),
        "e2e": e2e,
    }
    if not args.no_cpu and world == 1:
        line["cpu_baseline"] = oracle_kops(logn, L, args.cpu_seconds)
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
