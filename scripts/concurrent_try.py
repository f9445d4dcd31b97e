"""WD-FUSE on B200 as two kernels sharing every SM: tc4 (tensor) on a share of the polynomials in
one stream, v8 (CUDA cores, one CTA per SM via WD_NTT_V8_CTAS=1) on the rest in another."""
import os, sys
os.environ.setdefault("WD_NTT_V8_CTAS", "1")
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
N, L, B = 1 << 16, 36, 128
primes = inputs.bench_primes(L)
x = inputs.uniform_residues_torch(primes, N, B, inputs.SEED_BASE + 2, device="cuda")
y = torch.empty_like(x); yref = torch.empty_like(x)
pt = wdntt.Plan(N, primes, mode="tc4")
pc = wdntt.Plan(N, primes, mode="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
main = torch.cuda.current_stream()
pc.forward(x, yref); torch.cuda.synchronize()
def run(bt):
    s1.wait_stream(main); s2.wait_stream(main)
    if bt > 0:
        wdntt.wd_ntt_forward(pt.handle, x[:bt], y[:bt], bt, s1.cuda_stream)
    if bt < B:
        wdntt.wd_ntt_forward(pc.handle, x[bt:], y[bt:], B - bt, s2.cuda_stream)
    main.wait_stream(s1); main.wait_stream(s2)
for bt in (0, 128, 32, 48, 64, 80, 96):
    for _ in range(3): run(bt)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10): run(bt)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 10
    ok = bool(torch.equal(y, yref))
    print("tc4 polys %3d / v8 polys %3d: %.4f ms per forward of 128 polys (%.0f KOPS fwd)  exact=%s" % (bt, B - bt, ms, B * L / ms, ok), flush=True)
