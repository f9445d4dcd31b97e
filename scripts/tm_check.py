"""A/B of the TMEM-resident kernel "tm" against v8 (N = 2^16 by default): bit-exact agreement (and
sampled rows vs the oracle) at several batch sizes, in place, then forward / inverse ms of both at
128 polynomials.  usage: python scripts/tm_check.py [L] [reps] [logN]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt  # noqa: E402

L = int(sys.argv[1]) if len(sys.argv) > 1 else 36
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
logn = int(sys.argv[3]) if len(sys.argv) > 3 else 16
n = 1 << logn
primes = inputs.bench_primes(L)


def mk(kern):
    os.environ["WD_NTT_KERNEL"] = kern
    p = wdntt.Plan(n, primes)
    os.environ.pop("WD_NTT_KERNEL")
    return p


pt, p8 = mk("tm"), mk("v8")
sp = torch.cuda.current_stream().cuda_stream
ok = True
for b in (1, 2, 3, 5, 128):
    x = inputs.uniform_residues_torch(primes, n, b, inputs.SEED_BASE + 7 + b, device="cuda")
    yt, y8, zt = torch.empty_like(x), torch.empty_like(x), torch.empty_like(x)
    wdntt.wd_ntt_forward(pt.handle, x, yt, b, sp)
    wdntt.wd_ntt_forward(p8.handle, x, y8, b, sp)
    wdntt.wd_ntt_inverse(pt.handle, yt, zt, b, sp)
    torch.cuda.synchronize()
    f_eq, rt = torch.equal(yt, y8), torch.equal(zt, x)
    # sampled rows vs the oracle
    xs = x.cpu().numpy().view(np.uint32).reshape(b, L, n)
    ys = yt.cpu().numpy().view(np.uint32).reshape(b, L, n)
    idx = [(0, 0), (b - 1, L - 1), (b // 2, L // 2)]
    o_ok = all(np.array_equal(oracle.ntt_forward_row(xs[i, l], primes[l]), ys[i, l]) for i, l in idx)
    oi_ok = all(np.array_equal(oracle.ntt_inverse_row(ys[i, l], primes[l]), xs[i, l]) for i, l in idx)
    # in place
    w = x.clone()
    wdntt.wd_ntt_forward(pt.handle, w, w, b, sp)
    torch.cuda.synchronize()
    ip_f = torch.equal(w, y8)
    wdntt.wd_ntt_inverse(pt.handle, w, w, b, sp)
    torch.cuda.synchronize()
    ip_i = torch.equal(w, x)
    assert wdntt.wd_ntt_last_kernel() == "tm", wdntt.wd_ntt_last_kernel()
    print("batch %3d: fwd==v8 %s  roundtrip %s  oracle fwd %s inv %s  in-place fwd %s inv %s" % (
        b, f_eq, rt, o_ok, oi_ok, ip_f, ip_i), flush=True)
    ok &= f_eq and rt and o_ok and oi_ok and ip_f and ip_i


def timeit(plan, b):
    x = inputs.uniform_residues_torch(primes, n, b, inputs.SEED_BASE + 5, device="cuda")
    y, z = torch.empty_like(x), torch.empty_like(x)
    for _ in range(3):
        wdntt.wd_ntt_forward(plan.handle, x, y, b, sp)
        wdntt.wd_ntt_inverse(plan.handle, y, z, b, sp)
    torch.cuda.synchronize()
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
    return f, i, 2 * b * L / (f + i)


for b in (128, 2):
    for name, pl in (("v8", p8), ("tm", pt), ("v8", p8), ("tm", pt)):
        f, i, k = timeit(pl, b)
        print("%s logN %d batch %3d L %d: fwd %.4f ms inv %.4f ms KOPS %.0f" % (name, logn, b, L, f, i, k), flush=True)
print("ALL OK" if ok else "MISMATCH")
