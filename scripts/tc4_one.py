"""One tc4 forward (plus one warm-up) at N=2^16, L=36, batch B (argv[1], default 32) for ncu captures."""
import sys, os
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
N, L = 1 << 16, 36
B = int(sys.argv[1]) if len(sys.argv) > 1 else 32
mode = sys.argv[2] if len(sys.argv) > 2 else "tc4"
fwd = (sys.argv[3] != "inv") if len(sys.argv) > 3 else True
primes = inputs.bench_primes(L)
x = inputs.uniform_residues_torch(primes, N, B, inputs.SEED_BASE + 2, device="cuda")
y = torch.empty_like(x)
p = wdntt.Plan(N, primes, mode=mode)
for _ in range(2):
    (p.forward if fwd else p.inverse)(x, y)
torch.cuda.synchronize()
print("done", mode, B)
