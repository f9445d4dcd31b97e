"""Run tc4_probe.cu on a B200: int8 tcgen05 peak and the SWIZZLE_64B TMA -> UMMA layout check.
Prints JSON lines (profiles/r02/tc4_probe.jsonl)."""
import ctypes
import json
import os
import subprocess
import sys

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(HERE, "tc4_probe.so")
src = os.path.join(HERE, "tc4_probe.cu")
if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17", "-Xcompiler",
                           "-fPIC", "-shared", "-o", so, src, "-lcuda"])
lib = ctypes.CDLL(so)
lib.peak_i8.restype = ctypes.c_float
lib.peak_i8.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int]
lib.sw64_check.restype = ctypes.c_int

SM = 148
for n in (256, 128, 64):
    iters = 20000
    ms = lib.peak_i8(n, SM, iters)
    macs = SM * iters * 128 * n * 32
    print(json.dumps({"probe": "peak_i8", "M": 128, "N": n, "K": 32, "ctas": SM, "iters": iters, "ms": ms,
                      "TMAC_per_s": macs / (ms / 1e3) / 1e12, "TOPS": 2 * macs / (ms / 1e3) / 1e12,
                      "mac_per_clk_per_sm_at_1965": macs / (ms / 1e3) / SM / 1.965e9}), flush=True)

rng = np.random.default_rng(7)
G = rng.integers(0, 2**32, size=(128, 256), dtype=np.uint64).astype(np.uint32)
B = rng.integers(0, 256, size=(64, 64), dtype=np.uint8)          # [n][k]
for variant, e in ((1, 0), (3, 0), (3, 5), (3, 15), (2, 0)):
    D = np.zeros((128, 64), dtype=np.int32)
    Ad = np.zeros(8192, dtype=np.uint8)
    err = lib.sw64_check(variant, e, G.ctypes.data, B.ctypes.data, D.ctypes.data, Ad.ctypes.data)
    if variant == 1:
        A = G[:, 0:16]
    else:
        A = np.concatenate([G[:, 8 * e:8 * e + 8], G[:, 128 + 8 * e:128 + 8 * e + 8]], axis=1)
    Ab = A.copy().view(np.uint8).reshape(128, 64)
    ref = Ab.astype(np.int64) @ B.astype(np.int64).T
    ok = bool(np.array_equal(D.astype(np.int64), ref))
    # the smem image expected from the 64B swizzle: 16-byte chunk c of row m at chunk c ^ ((m >> 1) & 3)
    exp = np.zeros(8192, dtype=np.uint8)
    for m in range(128):
        for c in range(4):
            if variant == 3:
                off = (m >> 3) * 512 + c * 128 + (m & 7) * 16
            else:
                off = m * 64 + (c ^ ((m >> 1) & 3)) * 16
            exp[off:off + 16] = Ab[m, c * 16:c * 16 + 16]
    print(json.dumps({"probe": "sw64_tma_umma", "variant": variant, "e": e, "err": err, "exact": ok,
                      "smem_matches_xor_model": bool(np.array_equal(exp, Ad)),
                      "mismatch": int((D.astype(np.int64) != ref).sum())}), flush=True)
