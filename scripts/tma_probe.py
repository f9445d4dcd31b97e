"""TMA throughput by box shape (tma_probe.cu).  JSON lines: GB/s aggregate over 148 CTAs (1 per SM)."""
import ctypes, json, os, subprocess
HERE = os.path.dirname(os.path.abspath(__file__))
so, src = os.path.join(HERE, "tma_probe.so"), os.path.join(HERE, "tma_probe.cu")
if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17", "-Xcompiler",
                           "-fPIC", "-shared", "-o", so, src, "-lcuda"])
lib = ctypes.CDLL(so)
lib.tma_probe.restype = ctypes.c_float
lib.tma_probe.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_uint32]
names = {0: "ld 2D 128w x16 (512B rows)", 1: "ld 2D 16w x128 SW64 (64B rows)", 2: "ld 3D 8w x128 x2 SW32 (32B rows)",
         3: "ld 5D canonical (16B rows)", 4: "ld 1D bulk 8KB", 10: "st 2D 128w x16", 11: "st 2D 16w x128 SW64",
         12: "st 2D 32w x128 SW128 (16KB)", 14: "st 1D bulk 8KB"}
for where, rows in (("L2", 32768), ("HBM", 524288)):
    for mode in (0, 1, 2, 3, 4, 10, 11, 12, 14):
        tiles = 2000
        ms = lib.tma_probe(mode, 148, tiles, rows)
        nbytes = 148 * tiles * (16384 if mode == 12 else 8192)
        print(json.dumps({"probe": "tma", "where": where, "mode": names[mode], "ms": ms,
                          "GBps": nbytes / (ms / 1e3) / 1e9 if ms > 0 else None}), flush=True)
