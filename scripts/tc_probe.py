"""Run the tensor-path probes on a B200 (see tc_probe.cu).  Prints JSON lines."""
import ctypes
import json
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(HERE, "tc_probe.so")
if not os.path.exists(so):
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-Xcompiler", "-fPIC",
                           "-shared", "-o", so, os.path.join(HERE, "tc_probe.cu")])
lib = ctypes.CDLL(so)
lib.probe_mma.restype = ctypes.c_int
lib.probe_tmem_a.restype = ctypes.c_int
lib.probe_mma_loop.restype = ctypes.c_float
lib.probe_mma_loop.argtypes = [ctypes.c_int] * 4
lib.probe_int.restype = ctypes.c_float
lib.probe_int.argtypes = [ctypes.c_int] * 3
lib.probe_copy.restype = ctypes.c_float
lib.probe_copy.argtypes = [ctypes.c_size_t, ctypes.c_int, ctypes.c_int]

rng = np.random.default_rng(1)
A = rng.integers(0, 256, size=(128, 64), dtype=np.uint8)
B = rng.integers(0, 256, size=(64, 64), dtype=np.uint8)     # [n][k]
D = np.zeros((128, 64), dtype=np.int32)
e = lib.probe_mma(A.ctypes.data, B.ctypes.data, D.ctypes.data)
ref = A.astype(np.int64) @ B.astype(np.int64).T
ok = bool(np.array_equal(D.astype(np.int64), ref))
res = {"probe": "mma_i8_128x64x64", "err": e, "exact": ok}
if not ok:
    res["mismatch"] = int((D != ref).sum())
    res["D00"] = D[:2, :4].tolist()
    res["ref00"] = ref[:2, :4].tolist()
    # try to guess the layout issue: correlate with transposes
    res["eq_T"] = bool(np.array_equal(D.astype(np.int64), (A.astype(np.int64) @ B.astype(np.int64))))
print(json.dumps(res), flush=True)

B4 = rng.integers(0, 256, size=(4, 64, 64), dtype=np.uint8)
D4 = np.zeros((128, 64), dtype=np.int32)
e = lib.probe_mask(A.ctypes.data, B4.ctypes.data, D4.ctypes.data)
res = {"probe": "mma_mask", "err": e}
for g in range(4):
    refg = A[32 * g:32 * g + 32].astype(np.int64) @ B4[g].astype(np.int64).T
    res["group%d_exact" % g] = bool(np.array_equal(D4[32 * g:32 * g + 32], refg))
    res["group%d_matches_B3" % g] = bool(np.array_equal(D4[32 * g:32 * g + 32], A[32*g:32*g+32].astype(np.int64) @ B4[3].astype(np.int64).T))
print(json.dumps(res), flush=True)
D5 = np.zeros((128, 64), dtype=np.int32)
e = lib.probe_tmem_a(A.ctypes.data, B.ctypes.data, D5.ctypes.data)
print(json.dumps({"probe": "mma_a_from_tmem", "err": e, "exact": bool(np.array_equal(D5.astype(np.int64), ref)),
                  "D00": D5[:1, :4].tolist(), "ref00": ref[:1, :4].tolist()}), flush=True)
import sys
if "--mask-only" in sys.argv:
    sys.exit(0)
SM = 148
for blocks_per_sm in (1, 2, 4):
    blocks = SM * blocks_per_sm
    it = 2000
    for do_ld, do_mma in ((0, 1), (1, 0), (1, 1)):
        ms = lib.probe_mma_loop(blocks, it, do_ld, do_mma)
        per_iter_ns = ms * 1e6 / it
        elems = blocks * 128 * 16 * it       # 128 rows x 16 u32 outputs per tile-iteration
        print(json.dumps({"probe": "mma_loop", "blocks": blocks, "ld": do_ld, "mma": do_mma, "ms": ms,
                          "ns_per_iter_per_cta_wave": per_iter_ns,
                          "Gelem_per_s": elems / (ms / 1e3) / 1e9,
                          "tmem_read_TBps": (blocks * 128 * 64 * 4 * it * do_ld) / (ms / 1e3) / 1e12}),
              flush=True)

for threads, bps in ((256, 8), (512, 4), (1024, 2)):
    it = 2000
    ms = lib.probe_int(SM * bps, threads, it)
    bfly = SM * bps * threads * 32 * it
    print(json.dumps({"probe": "int_bfly", "threads": threads, "blocks": SM * bps, "ms": ms,
                      "Gbfly_per_s": bfly / (ms / 1e3) / 1e9}), flush=True)

for mb in (16, 48, 96, 2048):
    b = mb << 20
    ms = lib.probe_copy(b, SM * 4, 5)
    print(json.dumps({"probe": "copy", "MB": mb, "ms": ms, "GBps_rw": 2 * b / (ms / 1e3) / 1e9}), flush=True)
