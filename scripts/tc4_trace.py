"""Pipeline timeline of CTA 0 of one tc4 forward (config-3 shape unless argv[1] gives the batch)."""
import sys, os
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
N, L = 1 << 16, 36
B = int(sys.argv[1]) if len(sys.argv) > 1 else 128
primes = inputs.bench_primes(L)
x = inputs.uniform_residues_torch(primes, N, B, inputs.SEED_BASE + 2, device="cuda")
y = torch.empty_like(x)
p = wdntt.Plan(N, primes, mode="tc4")
p.forward(x, y); torch.cuda.synchronize()
tr = torch.zeros(53248, dtype=torch.int64, device="cuda")
wdntt._lib.wd_ntt_debug_tc4_trace(tr.data_ptr())
p.forward(x, y); torch.cuda.synchronize()
wdntt._lib.wd_ntt_debug_tc4_trace(None)
t = tr.cpu().numpy().astype(np.int64)
rows = B * L
n = (rows + 147) // 148   # rows of CTA 0 (approx)
load, mma, acc, stg, store = t[0:4096], t[4096:8192], t[8192:12288], t[12288:16384], t[16384:20480]
t0 = mma[0]
def rel(a): return (a - t0)
nt = int((mma > 0).sum()); nl = int((load > 0).sum()); ns = int((store > 0).sum())
print("tiles", nt, "loads", nl, "stores", ns, "total cycles %d" % (mma[nt - 1] - t0))
# per-pass summary: 32 tiles / pass, 16 loads / pass, 16 stores / pass
for p_ in range(min(nt // 32, 12)):
    m = mma[32 * p_:32 * p_ + 32]; a = acc[32 * p_:32 * p_ + 32]
    l = load[16 * p_:16 * p_ + 16]; st = store[16 * p_:16 * p_ + 16]; sg = stg[16 * p_:16 * p_ + 16]
    print("pass %2d  mma1 %7d..%7d (d %5d)  mma2 %7d..%7d (d %5d)  acc-mma lag s1 %5d s2 %5d  load0 %7d  st0 %7d stg-lag %5d"
          % (p_, rel(m[0]), rel(m[15]), (m[15] - m[0]) // 15, rel(m[16]), rel(m[31]), (m[31] - m[16]) // 15,
             np.median(a[:16] - m[:16]), np.median(a[16:] - m[16:]), rel(l[0]), rel(st[0]), np.median(st - sg)))
d = np.diff(mma[:nt])
print("MMA issue interval: median %d  mean %d  p90 %d" % (np.median(d), d.mean(), np.percentile(d, 90)))
lag = acc[:nt] - mma[:nt]
print("acc observed - MMA issued: median %d p10 %d p90 %d" % (np.median(lag), np.percentile(lag, 10), np.percentile(lag, 90)))
det = t[20480:53248].reshape(4096, 8)
for p_ in (2, 3):
    print("pass", p_, "(tile: operand ready -> acc slot free -> MMA issued -> owner observes acc)")
    for k in range(32):
        tt = 32 * p_ + k
        print("  tile %2d  opnd %7d  slot +%5d  issue +%5d  observed +%5d" % (k, det[tt, 6] - t0, mma[tt] - det[tt, 6] - 0, 0, acc[tt] - mma[tt]))
np.save("gpurun_out/tc4_trace.npy", t)
