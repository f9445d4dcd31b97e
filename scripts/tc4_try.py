"""tc4 bring-up: forward vs the oracle on growing shapes, then timing at config 3 (prints lines)."""
import sys, os, time
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt

N = 1 << 16
def check(L, batch, seed=1, inplace=False):
    primes = inputs.bench_primes(L)
    x = inputs.uniform_residues(primes, N, batch, seed)
    p = wdntt.Plan(N, primes, mode="tc4")
    d = torch.from_numpy(x.view(np.int32)).cuda()
    y = d if inplace else torch.empty_like(d)
    t0 = time.time()
    p.forward(d, y)
    torch.cuda.synchronize()
    yh = y.cpu().numpy().view(np.uint32)
    ref = oracle.ntt_forward(x, primes)
    ok = np.array_equal(yh, ref)
    bad = int((yh != ref).sum())
    rows_bad = int((yh != ref).any(axis=2).sum())
    print("L=%d batch=%d inplace=%s ok=%s bad_words=%d bad_rows=%d/%d (%.2fs)" % (L, batch, inplace, ok, bad, rows_bad, L * batch, time.time() - t0), flush=True)
    if not ok:
        r = np.argwhere((yh != ref).any(axis=2))[0]
        b, l = r
        diff = np.nonzero(yh[b, l] != ref[b, l])[0]
        print("  first bad row", (b, l), "first bad idx", diff[:16].tolist(), "n", len(diff), flush=True)
        print("  got", yh[b, l, diff[:4]].tolist(), "want", ref[b, l, diff[:4]].tolist(), flush=True)
    p.close()
    return ok

ok = check(1, 1)
ok = check(3, 2) and ok
ok = check(5, 67, seed=2) and ok
ok = check(36, 8, seed=3, inplace=True) and ok
# timing at config 3 vs v8
L, batch = 36, 128
primes = inputs.bench_primes(L)
x = inputs.uniform_residues_torch(primes, N, batch, inputs.SEED_BASE + 2, device="cuda")
y = torch.empty_like(x); y2 = torch.empty_like(x)
for mode in ("cuda", "tc4"):
    p = wdntt.Plan(N, primes, mode=mode)
    for _ in range(3):
        p.forward(x, y)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        p.forward(x, y)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 20
    print("mode %s fwd %.4f ms  %.0f KOPS(fwd only)  HBM frac %.3f" % (mode, ms, L * batch / ms, L * batch * 8 * N / (ms / 1e3) / 6552e9), flush=True)
    if mode == "cuda":
        y2.copy_(y)
    else:
        print("tc4 == cuda at config 3:", bool(torch.equal(y, y2)), flush=True)
    p.close()
