"""Multi-process (gloo, world size 2, CPU) tests of the limb-sharding host logic
(SURVEY.md 8 row e, T6).  The per-rank transform is the CPU oracle standing in
for the GPU kernel (NCCL cannot put two ranks on one GPU, and this box has none);
the result must be byte-identical to the unsharded oracle output."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_hpca_fanzzfzdtksy25_b200 import dist as wdist
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_limb_range_partitions():
    for L in (1, 5, 36, 48, 60):
        for G in (1, 2, 3, 4, 8):
            spans = [wdist.limb_range(L, G, g) for g in range(G)]
            assert spans[0][0] == 0 and spans[-1][1] == L
            assert all(spans[i][1] == spans[i + 1][0] for i in range(G - 1))
            sz = [b - a for a, b in spans]
            assert max(sz) - min(sz) <= 1


def _worker(rank, world, port, n, L, batch, out_q):
    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    primes = inputs.bench_primes(L)
    x = None
    if rank == 0:
        x = torch.from_numpy(inputs.uniform_residues(primes, n, batch, 99).view(np.int32))

    def transform(xl, pr):
        y = oracle.ntt_forward(xl.numpy().view(np.uint32), pr, threads=1)
        return torch.from_numpy(y.view(np.int32))

    y = wdist.sharded_transform(x, primes, n, batch, transform)
    if rank == 0:
        ref = oracle.ntt_forward(x.numpy().view(np.uint32), primes, threads=2)
        out_q.put(bool(np.array_equal(y.numpy().view(np.uint32), ref)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("L", [5, 6])
def test_sharded_equals_unsharded_gloo(L):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, 256, L, 2, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
        assert p.exitcode == 0
    assert q.get(timeout=5) is True


# -------------------------------------------------- limb-sharded ModUp: the all-reduce exchange
def _modup_worker(rank, world, port, n, out_q):
    import oracle
    from oracle import rns
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    qs = inputs.bench_primes(5)
    ps = [786433, 805961729]
    x = inputs.uniform_residues(qs, n, 2, 123)                  # every rank can build the same input
    l0, l1 = wdist.limb_range(len(qs), world, rank)
    x_local = torch.from_numpy(np.ascontiguousarray(x[:, l0:l1]).view(np.int32))

    def partial_fn(xl):
        coeff = oracle.ntt_inverse(xl.numpy().view(np.uint32), qs[l0:l1], threads=1)
        return torch.from_numpy(rns.bconv_partial(coeff, qs[l0:l1], qs, ps).astype(np.int64))

    def finish_fn(total):
        t = total.numpy().astype(np.uint64)
        for j, p in enumerate(ps):
            t[:, j] %= p
        return torch.from_numpy(oracle.ntt_forward(t.astype(np.uint32), ps, threads=1).view(np.int32))

    up_p = wdist.sharded_modup(x_local, partial_fn, finish_fn)
    ref = rns.modup(x, qs, ps)[:, len(qs):]
    out_q.put((rank, bool(np.array_equal(up_p.numpy().view(np.uint32), ref))))
    dist.barrier()
    dist.destroy_process_group()


def test_sharded_modup_allreduce_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_modup_worker, args=(r, 2, port, 128, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
        assert p.exitcode == 0
    res = sorted(q.get(timeout=5) for _ in range(2))
    assert res == [(0, True), (1, True)]
