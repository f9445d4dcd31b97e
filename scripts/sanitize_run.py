"""Drive every launch path of libwdntt.so once on small shapes, for compute-sanitizer
(memcheck / racecheck / synccheck).  Usage: python scripts/sanitize_run.py [group ...]
Groups: v8 v8feeds tm cc cl small tensor fused ftc gemm tc4 rns host.  Each group prints one line; the round trip
is checked (INTT(NTT(x)) == x) so a wrong result under the sanitizer is visible too."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt  # noqa: E402


def rt(plan, n, primes, batch, seed=11):
    x = torch.from_numpy(inputs.uniform_residues(primes, n, batch, seed).view(np.int32)).cuda()
    y = torch.empty_like(x)
    z = torch.empty_like(x)
    plan.forward(x, y)
    plan.inverse(y, z)
    torch.cuda.synchronize()
    assert torch.equal(z, x), "round trip failed"


def group_v8():
    for logn, L, batch in ((16, 2, 2), (16, 4, 25), (16, 8, 40), (15, 3, 50), (17, 2, 2), (17, 3, 30),
                           (13, 4, 300), (14, 2, 600), (12, 4, 2)):
        pr = inputs.bench_primes(L)
        p = wdntt.Plan(1 << logn, pr)
        rt(p, 1 << logn, pr, batch)
        p.close()


def group_v8feeds():
    # every v8 column feed (WD_NTT_V8_TMA is read at plan creation) and cluster size at N = 2^14, 2^16
    for feed in ("0", "1", "2", "4", "7"):
        for logn, cl, batch in ((16, "2", 30), (16, "1", 30), (14, "4", 300)):
            os.environ["WD_NTT_V8_TMA"], os.environ["WD_NTT_CL"] = feed, cl
            pr = inputs.bench_primes(2)
            p = wdntt.Plan(1 << logn, pr)
            rt(p, 1 << logn, pr, batch)
            p.close()
    os.environ.pop("WD_NTT_V8_TMA"); os.environ.pop("WD_NTT_CL")


def group_tm():
    # tm, the TMEM-resident kernel (N = 2^16): fewer rows than SMs, and CTAs with 2 and 3 rows (both
    # TMEM layouts, the row mbarrier handoff, the cross-row TMA / cp.async prefetches)
    os.environ["WD_NTT_KERNEL"] = "tm"
    for L, batch in ((2, 3), (4, 40), (3, 100)):
        pr = inputs.bench_primes(L)
        p = wdntt.Plan(1 << 16, pr)
        rt(p, 1 << 16, pr, batch)
        assert wdntt.wd_ntt_last_kernel() == "tm"
        p.close()
    os.environ.pop("WD_NTT_KERNEL")


def group_cc():
    for logn, L, batch in ((12, 2, 3), (13, 2, 3), (14, 2, 3)):
        pr = inputs.bench_primes(L)
        p = wdntt.Plan(1 << logn, pr)
        rt(p, 1 << logn, pr, batch)
        p.close()


def group_cl():
    for logn, L, batch in ((15, 2, 2), (16, 2, 3)):
        pr = inputs.bench_primes(L)
        p = wdntt.Plan(1 << logn, pr)
        rt(p, 1 << logn, pr, batch)
        p.close()


def group_small():
    for logn in (4, 8, 11):
        pr = inputs.bench_primes(2)
        p = wdntt.Plan(1 << logn, pr)
        rt(p, 1 << logn, pr, 3)
        p.close()


def _mode(name, share=-1.0, batch=3, L=3):
    pr = inputs.bench_primes(L)
    p = wdntt.Plan(1 << 16, pr)
    p.set_mode(name, share)
    rt(p, 1 << 16, pr, batch)
    p.close()


def group_tensor():
    _mode("tensor")


def group_fused():
    _mode("fused")


def group_ftc():
    _mode("ftc", 0.5, batch=4)


def group_gemm():
    _mode("cuda_gemm")


def group_tc4():
    if "tc4" in getattr(wdntt, "MODES", {}):
        _mode("tc4", batch=2, L=3)


def group_rns():
    n = 1 << 16
    pr = inputs.bench_primes(5)
    p = wdntt.Plan(n, pr)
    x = torch.from_numpy(inputs.uniform_residues(pr, n, 2, 3).view(np.int32)).cuda()
    p.rescale(x)
    a = torch.from_numpy(inputs.uniform_residues(pr, n, 2, 4).view(np.int32)).cuda()
    b = torch.from_numpy(inputs.uniform_residues(pr, n, 2, 5).view(np.int32)).cuda()
    p.pointwise_inverse(a, b)
    qs, ps = pr[:4], pr[4:]
    pq, pp = wdntt.Plan(n, qs), wdntt.Plan(n, ps)
    conv = wdntt.RnsConv(pq, pp)
    xq = torch.from_numpy(inputs.uniform_residues(qs, n, 2, 6).view(np.int32)).cuda()
    up = conv.modup(xq)
    conv.moddown(up)
    torch.cuda.synchronize()
    conv.close(); pq.close(); pp.close(); p.close()


def group_host():
    n = 1 << 14
    pr = inputs.bench_primes(3)
    p = wdntt.Plan(n, pr)
    x = inputs.uniform_residues(pr, n, 5, 9)
    hx = torch.from_numpy(x.view(np.int32)).pin_memory()
    hy = torch.empty_like(hx).pin_memory()
    work = torch.empty(hx.shape, dtype=torch.int32, device="cuda")
    wdntt.wd_ntt_forward_host(p.handle, hx, hy, 5, work)
    wdntt.wd_ntt_inverse_host(p.handle, hy, hy, 5, work)
    torch.cuda.synchronize()
    assert torch.equal(hy, hx)
    p.close()


GROUPS = {k[6:]: v for k, v in globals().items() if k.startswith("group_")}

if __name__ == "__main__":
    names = sys.argv[1:] or list(GROUPS)
    for g in names:
        GROUPS[g]()
        print("sanitize group %s: ok" % g, flush=True)
