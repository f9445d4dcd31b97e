"""Forward / inverse ms of one (logN, L, ciphertexts) point under the current environment (AUTO).
usage: python scripts/point_time.py LOGN L NCT [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt  # noqa: E402

logn, L, nct = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 20
n, b = 1 << logn, 2 * nct
primes = inputs.bench_primes(L)
plan = wdntt.Plan(n, primes)
x = inputs.uniform_residues_torch(primes, n, b, inputs.SEED_BASE + 5, device="cuda")
y, z = torch.empty_like(x), torch.empty_like(x)
sp = torch.cuda.current_stream().cuda_stream
for _ in range(3):
    wdntt.wd_ntt_forward(plan.handle, x, y, b, sp)
    wdntt.wd_ntt_inverse(plan.handle, y, z, b, sp)
torch.cuda.synchronize()
assert torch.equal(z, x)
ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
ev[0].record()
for _ in range(reps):
    wdntt.wd_ntt_forward(plan.handle, x, y, b, sp)
ev[1].record()
for _ in range(reps):
    wdntt.wd_ntt_inverse(plan.handle, y, z, b, sp)
ev[2].record()
torch.cuda.synchronize()
f, i = ev[0].elapsed_time(ev[1]) / reps, ev[1].elapsed_time(ev[2]) / reps
print("logN=%d L=%d ct=%d env=%s fwd %.4f ms inv %.4f ms KOPS %.0f" % (
    logn, L, nct, os.environ.get("WD_NTT_V8_TMA", "-"), f, i, 2 * b * L / (f + i)))
