"""GPU parity of the RNS operations around the NTT vs oracle/rns.py.

RESCALE is exact integer arithmetic with one canonical answer, so every comparison is
bit-exact: against the step-by-step RNS oracle everywhere, and against the big-int CRT
definition (round(A / q_last)) on the small cases.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from oracle import rns  # noqa: E402
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs  # noqa: E402

P = inputs.bench_primes(110)
SMALL = [786433, 269221889, 537133057, 805961729]


@pytest.fixture(scope="module")
def wd():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_hpca_fanzzfzdtksy25_b200 import wdntt
    return wdntt


def to_dev(x: np.ndarray):
    return torch.from_numpy(np.ascontiguousarray(x).view(np.int32)).cuda()


def to_host(t) -> np.ndarray:
    return t.cpu().numpy().view(np.uint32)


def gpu_rescale(wd, plan, x):
    o = plan.rescale(to_dev(x))
    torch.cuda.synchronize()
    return to_host(o)


@pytest.mark.parametrize("logn,L,batch", [(12, 2, 3), (12, 5, 2), (13, 4, 3), (14, 3, 2), (15, 3, 2), (16, 4, 2),
                                          (17, 3, 1)])
def test_rescale_vs_rns_oracle(wd, logn, L, batch):
    n = 1 << logn
    primes = P[:L]
    x = inputs.uniform_residues(primes, n, batch, 8000 + logn * 10 + L)
    plan = wd.Plan(n, primes)
    assert np.array_equal(gpu_rescale(wd, plan, x), rns.rescale_rns(x, primes)), (logn, L)


def test_rescale_vs_definition_small(wd):
    n = 1 << 12
    primes = [P[3], SMALL[1], P[0]]
    x = inputs.uniform_residues(primes, n, 2, 8100)
    plan = wd.Plan(n, primes)
    assert np.array_equal(gpu_rescale(wd, plan, x), rns.rescale_definition(x, primes))


@pytest.mark.parametrize("primes", [[SMALL[0], P[1], SMALL[3], P[2]], [P[5], SMALL[2], SMALL[0]], [SMALL[0], P[7]]])
def test_rescale_prime_sizes(wd, primes):
    n = 1 << 16
    x = inputs.uniform_residues(primes, n, 2, 8200 + len(primes))
    plan = wd.Plan(n, primes)
    assert np.array_equal(gpu_rescale(wd, plan, x), rns.rescale_rns(x, primes))
    for kind in ("zeros", "qm1", "alt"):
        s = inputs.structured(kind, primes, n)
        assert np.array_equal(gpu_rescale(wd, plan, s), rns.rescale_rns(s, primes)), kind


def test_rescale_many_rows(wd):
    # more output rows than resident CTAs: every CTA walks several rows
    n, primes = 1 << 13, P[:9]
    x = inputs.uniform_residues(primes, n, 90, 8300)
    plan = wd.Plan(n, primes)
    assert np.array_equal(gpu_rescale(wd, plan, x), rns.rescale_rns(x, primes))


def test_rescale_full_size_sampled(wd):
    # BASELINE config 3 shape (N = 2^16, L = 36, 128 polynomials): sampled polynomials vs the oracle
    n, L, batch = 1 << 16, 36, 128
    primes = P[:L]
    x = inputs.uniform_residues_torch(primes, n, batch, inputs.SEED_BASE + 2, device="cuda")
    plan = wd.Plan(n, primes)
    o = plan.rescale(x)
    torch.cuda.synchronize()
    for b in (0, 77, 127):
        xb = to_host(x[b:b + 1])
        assert np.array_equal(to_host(o[b:b + 1]), rns.rescale_rns(xb, primes)), b


def test_rescale_errors(wd):
    n = 1 << 12
    x = to_dev(inputs.uniform_residues(P[:1], n, 1, 1))
    plan1 = wd.Plan(n, P[:1])
    with pytest.raises(wd.WdNttError):
        wd.wd_rescale(plan1.handle, x, x, 1, x)               # L = 1: nothing to divide by
    plan = wd.Plan(n, P[:3])
    y = to_dev(inputs.uniform_residues(P[:3], n, 1, 2))
    out = torch.empty((1, 2, n), dtype=torch.int32, device="cuda")
    work = torch.empty((1, n), dtype=torch.int32, device="cuda")
    wd.wd_rescale(plan.handle, y, out, 0, work)                # batch 0: no-op
    with pytest.raises(wd.WdNttError):
        wd.wd_rescale(plan.handle, y, out, 1, None)            # no work buffer
    dup = wd.Plan(n, [P[0], P[1], P[0]])                       # q_last repeated: no inverse
    with pytest.raises(wd.WdNttError):
        wd.wd_rescale(dup.handle, to_dev(inputs.uniform_residues([P[0], P[1], P[0]], n, 1, 3)), out, 1, work)


# ---------------------------------------------------------------- ModUp / ModDown (row f3)
QS = [P[0], P[1], P[2], SMALL[2]]
PS = [P[40], SMALL[3], P[41]]


@pytest.mark.parametrize("logn,a,k,batch", [(12, 4, 3, 2), (13, 3, 1, 3), (16, 4, 3, 2), (17, 2, 2, 1)])
def test_modup_moddown_vs_oracle(wd, logn, a, k, batch):
    n = 1 << logn
    qs, ps = QS[:a], PS[:k]
    if logn == 17:                                   # q = 1 mod 2^18 needed: bench primes only
        qs, ps = P[:a], P[40:40 + k]
    pq, pp = wd.Plan(n, qs), wd.Plan(n, ps)
    conv = wd.RnsConv(pq, pp)
    x = inputs.uniform_residues(qs, n, batch, 8400 + logn)
    up = conv.modup(to_dev(x))
    torch.cuda.synchronize()
    assert np.array_equal(to_host(up), rns.modup(x, qs, ps)), ("modup", logn)
    e = inputs.uniform_residues(qs + ps, n, batch, 8500 + logn)
    dn = conv.moddown(to_dev(e))
    torch.cuda.synchronize()
    assert np.array_equal(to_host(dn), rns.moddown(e, qs, ps)), ("moddown", logn)


def test_modup_moddown_keyswitch_shape(wd):
    # the paper's KeySwitch shape (Table III: N = 2^16, l = 34 ... 36 limbs, K = 1 special prime)
    # with a batch of 8 polynomials: ModUp 36 -> 37 limbs, ModDown 37 -> 36
    n, a, k, batch = 1 << 16, 36, 1, 8
    qs, ps = P[:a], P[50:50 + k]
    pq, pp = wd.Plan(n, qs), wd.Plan(n, ps)
    conv = wd.RnsConv(pq, pp)
    x = inputs.uniform_residues(qs, n, batch, 8600)
    up = to_host(conv.modup(to_dev(x)))
    dn = to_host(conv.moddown(to_dev(up)))
    torch.cuda.synchronize()
    for b in (0, 5):
        assert np.array_equal(up[b:b + 1], rns.modup(x[b:b + 1], qs, ps)), b
        assert np.array_equal(dn[b:b + 1], rns.moddown(up[b:b + 1], qs, ps)), b


@pytest.mark.parametrize("logn,a,k,batch", [(13, 6, 4, 3), (14, 9, 2, 2), (12, 37, 1, 2)])
def test_modup_few_targets_many_sources(wd, logn, a, k, batch):
    # rns_bconv_few (S > 4 sources, D <= 4 targets: register accumulation, Barrett every 12
    # terms) and ModUp's Q-limb pass-through fused into the v8 INTT
    n, qs, ps = 1 << logn, P[:a], P[100:100 + k]
    pq, pp = wd.Plan(n, qs), wd.Plan(n, ps)
    conv = wd.RnsConv(pq, pp)
    x = inputs.uniform_residues(qs, n, batch, 8800 + logn)
    up = to_host(conv.modup(to_dev(x)))
    assert np.array_equal(up, rns.modup(x, qs, ps))


def test_modup_many_rows_and_wide_bases(wd):
    n, qs, ps = 1 << 13, P[:20], P[30:46]            # 20 -> 36 limbs; more rows than resident CTAs
    pq, pp = wd.Plan(n, qs), wd.Plan(n, ps)
    conv = wd.RnsConv(pq, pp)
    x = inputs.uniform_residues(qs, n, 12, 8700)
    up = to_host(conv.modup(to_dev(x)))
    assert np.array_equal(up, rns.modup(x, qs, ps))
    dn = to_host(conv.moddown(to_dev(up)))
    assert np.array_equal(dn, rns.moddown(up, qs, ps))


def test_rns_conv_errors(wd):
    n = 1 << 12
    pq = wd.Plan(n, P[:3])
    with pytest.raises(wd.WdNttError):
        wd.RnsConv(pq, wd.Plan(n, [P[2], P[9]]))            # a prime in both bases
    with pytest.raises(wd.WdNttError):
        wd.RnsConv(pq, wd.Plan(1 << 13, P[10:12]))          # N mismatch


def test_sharded_modup_partials(wd):
    # two Q-limb shards on one GPU: partial shares summed (the all-reduce's job) and finished
    # equal the unsharded ModUp's P limbs; ModDown on a shard gives that shard's Q limbs
    n, qs, ps = 1 << 16, P[:6], P[40:42]
    x = inputs.uniform_residues(qs, n, 3, 8800)
    pp = wd.Plan(n, ps)
    total, convs = None, []
    for a0, a1 in [(0, 4), (4, 6)]:
        pq = wd.Plan(n, qs[a0:a1])
        conv = wd.RnsConv(pq, pp, q_all=qs)
        convs.append((a0, a1, conv, pq))
        part = conv.modup_partial(to_dev(np.ascontiguousarray(x[:, a0:a1])))
        total = part if total is None else total + part
    up_p = convs[0][2].modup_finish(total)
    torch.cuda.synchronize()
    full = rns.modup(x, qs, ps)
    assert np.array_equal(to_host(up_p), full[:, len(qs):])
    with pytest.raises(wd.WdNttError):
        convs[0][2].modup(to_dev(np.ascontiguousarray(x[:, 0:4])))   # a shard cannot run the whole ModUp
    ext = inputs.uniform_residues(qs + ps, n, 2, 8900)
    down = rns.moddown(ext, qs, ps)
    for a0, a1, conv, pq in convs:
        loc = np.ascontiguousarray(np.concatenate([ext[:, a0:a1], ext[:, len(qs):]], axis=1))
        got = to_host(conv.moddown(to_dev(loc)))
        assert np.array_equal(got, down[:, a0:a1]), (a0, a1)
