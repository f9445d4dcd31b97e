"""Two forward+inverse steps at N=2^16, L=36, B polynomials (argv: B mode) -- for ncu captures."""
import sys, os
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
B = int(sys.argv[1]) if len(sys.argv) > 1 else 128
mode = sys.argv[2] if len(sys.argv) > 2 else "auto"
logn = int(sys.argv[3]) if len(sys.argv) > 3 else 16
L = int(sys.argv[4]) if len(sys.argv) > 4 else 36
N = 1 << logn
primes = inputs.bench_primes(L)
x = inputs.uniform_residues_torch(primes, N, B, inputs.SEED_BASE + 2, device="cuda")
y, z = torch.empty_like(x), torch.empty_like(x)
p = wdntt.Plan(N, primes, mode=mode)
for _ in range(2):
    p.forward(x, y)
    p.inverse(y, z)
torch.cuda.synchronize()
assert torch.equal(z, x)
print("done", mode, B)
