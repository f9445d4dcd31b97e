import sys, os, ctypes
sys.path.insert(0, '/root/repo')
import torch
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
cudart = ctypes.CDLL('libcudart.so.12')
cudart.cudaGetErrorString.restype = ctypes.c_char_p
primes = inputs.bench_primes(2)
p = wdntt.Plan(1 << 16, primes, mode="tc4")
x = torch.zeros((1, 2, 1 << 16), dtype=torch.int32, device="cuda")
try:
    p.forward(x, x)
except Exception as e:
    print("err", e)
e = cudart.cudaGetLastError()
print("cudaGetLastError", e, cudart.cudaGetErrorString(e))
