import os, sys, numpy as np, torch
sys.path.insert(0, '.')
os.environ['WD_NTT_KERNEL'] = sys.argv[1] if len(sys.argv) > 1 else 'v7'
from paper_conf_hpca_fanzzfzdtksy25_b200 import wdntt as wd, inputs
import oracle
P = inputs.bench_primes(4)
for logn in (16,):
    n = 1 << logn
    for kind in ('delta', 'rand'):
        x = inputs.uniform_residues(P[:1], n, 1, 7) if kind == 'rand' else inputs.structured('delta', P[:1], n)
        plan = wd.Plan(n, P[:1], mode='cuda')
        xd = torch.from_numpy(x.view(np.int32).copy()).cuda(); yd = torch.empty_like(xd)
        plan.forward(xd, yd); torch.cuda.synchronize()
        y = yd.cpu().numpy().view(np.uint32).reshape(-1)
        ref = oracle.ntt_forward(x, P[:1]).reshape(-1)
        bad = np.nonzero(y != ref)[0]
        print(kind, logn, 'bad', len(bad), bad[:20], y[:8], ref[:8])
        # inverse of the oracle output
        rd = torch.from_numpy(ref.view(np.int32).copy().reshape(x.shape)).cuda(); zd = torch.empty_like(rd)
        plan.inverse(rd, zd); torch.cuda.synchronize()
        z = zd.cpu().numpy().view(np.uint32).reshape(-1)
        bad = np.nonzero(z != x.reshape(-1))[0]
        print(' inv bad', len(bad), bad[:20])
