"""Integer-pipe throughput probes (scripts/int_probe.cu) on a B200: ops per clock per SM."""
import ctypes
import json
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(HERE, "int_probe.so")
if not os.path.exists(so):
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-Xcompiler", "-fPIC",
                           "-shared", "-o", so, os.path.join(HERE, "int_probe.cu")])
lib = ctypes.CDLL(so)
lib.int_probe.restype = ctypes.c_float
lib.int_probe.argtypes = [ctypes.c_int] * 3
names = ["imad_hi", "imad_wide_both", "imad_lo", "shoup_hi", "lop3_iadd3", "ct_bfly_hi", "iadd3", "ct_bfly_mul64"]
for m, n in enumerate(names):
    for ctas in (4, 8):
        r = lib.int_probe(m, 4000, ctas)
        print(json.dumps({"probe": n, "ctas_per_sm": ctas, "ops_per_clk_per_sm": round(r, 2)}), flush=True)
