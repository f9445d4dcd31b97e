"""GPU parity: libwdntt.so (through the C ABI) vs the CPU oracle, bit for bit.

Integer transforms have exactly one correct canonical answer,
so every comparison is exact equality.  Small cases compare every row; the
BASELINE.json full-size configs compare sampled rows against the oracle and
check properties that hold at any size (round trip, sum rule) on every row.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs  # noqa: E402

P = inputs.bench_primes(60)


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


def gpu_fwd(wd, plan, x, mode=None):
    d = to_dev(x)
    o = torch.empty_like(d)
    if mode is not None:
        plan.set_mode(mode)
    plan.forward(d, o)
    torch.cuda.synchronize()
    return to_host(o)


def gpu_inv(wd, plan, y):
    d = to_dev(y)
    o = torch.empty_like(d)
    plan.inverse(d, o)
    torch.cuda.synchronize()
    return to_host(o)


# -------------------------------------------------------------- config 1 (BASELINE configs[0])
def test_config1_n4096_l4(wd):
    primes = P[:4]
    x = inputs.uniform_residues(primes, 1 << 12, 1, inputs.SEED_BASE + 0)
    plan = wd.Plan(1 << 12, primes)
    for l, q in enumerate(primes):
        assert plan.psi(l) == oracle.psi_min(q, 1 << 12)
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes))
    z = gpu_inv(wd, plan, y)
    assert np.array_equal(z, x)
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes))


# -------------------------------------------------------------- every supported N, full rows
@pytest.mark.parametrize("logn", list(range(1, 18)))
def test_all_sizes_vs_oracle(wd, logn):
    n = 1 << logn
    primes = [P[0], P[11], P[37]]
    batch = 3 if logn <= 15 else 2
    x = inputs.uniform_residues(primes, n, batch, 1000 + logn)
    plan = wd.Plan(n, primes)
    y = gpu_fwd(wd, plan, x)
    ref = oracle.ntt_forward(x, primes)
    assert np.array_equal(y, ref)
    assert np.array_equal(gpu_inv(wd, plan, y), x)
    yi = gpu_inv(wd, plan, x)
    assert np.array_equal(yi, oracle.ntt_inverse(x, primes))


@pytest.mark.parametrize("logn", [12, 14, 16, 17])
@pytest.mark.parametrize("kind", ["zeros", "qm1", "alt", "delta", "mono1", "mono4095", "ternary", "gauss"])
def test_edge_inputs(wd, logn, kind):
    n = 1 << logn
    primes = [P[0], P[59]]
    x = inputs.structured(kind, primes, n, seed=logn)
    plan = wd.Plan(n, primes)
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes))
    # all-(q-1) in the evaluation domain stresses the inverse's lazy bounds too
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes))


@pytest.mark.parametrize("logn", [12, 16])
def test_in_place_equals_out_of_place(wd, logn):
    n = 1 << logn
    primes = P[:5]
    x = inputs.uniform_residues(primes, n, 2, 7)
    plan = wd.Plan(n, primes)
    d = to_dev(x)
    o = torch.empty_like(d)
    plan.forward(d, o)
    plan.forward(d, d)
    torch.cuda.synchronize()
    assert torch.equal(d, o)
    plan.inverse(d, d)
    torch.cuda.synchronize()
    assert np.array_equal(to_host(d), x)


def test_batch_zero_and_errors(wd):
    plan = wd.Plan(1 << 12, P[:2])
    d = torch.zeros(2 * 4096 + 4, dtype=torch.int32, device="cuda")
    assert wd.wd_ntt_forward(plan.handle, d, d, 0) == 0
    with pytest.raises(wd.WdNttError) as e:
        wd.wd_ntt_forward(plan.handle, d.data_ptr() + 4, d.data_ptr() + 4, 1)
    assert e.value.code == wd.WD_EINVAL


def test_pointwise_inverse_is_negacyclic_product(wd):
    # f1: INTT(NTT(a) o NTT(b)) = a * b mod (X^N + 1, q)
    from oracle import brute
    for logn in (6, 12):
        n = 1 << logn
        primes = P[:3]
        a = inputs.uniform_residues(primes, n, 2, 11)
        b = inputs.uniform_residues(primes, n, 2, 12)
        plan = wd.Plan(n, primes)
        A, B = to_dev(gpu_fwd(wd, plan, a)), to_dev(gpu_fwd(wd, plan, b))
        o = torch.empty_like(A)
        plan.pointwise_inverse(A, B, o)
        torch.cuda.synchronize()
        got = to_host(o)
        fa, fb = oracle.ntt_forward(a, primes), oracle.ntt_forward(b, primes)
        prod = (fa.astype(np.uint64) * fb.astype(np.uint64)) % np.array(primes, np.uint64)[None, :, None]
        assert np.array_equal(got, oracle.ntt_inverse(prod.astype(np.uint32), primes))
        if logn == 6:
            for bi in range(2):
                for l, q in enumerate(primes):
                    assert got[bi, l].tolist() == brute.negacyclic_mul(a[bi, l].tolist(), b[bi, l].tolist(), q)


# -------------------------------------------------------------- BASELINE configs at full size
def _full_size_check(wd, n, L, batch, seed):
    """Every row of the forward AND the inverse against the (multithreaded) oracle, in the launch
    configuration bench.py times (AUTO, out of place), plus the exact round trip on the device."""
    primes = P[:L]
    x = inputs.uniform_residues(primes, n, batch, seed)
    plan = wd.Plan(n, primes)
    d = to_dev(x)
    y = torch.empty_like(d)
    plan.forward(d, y)
    torch.cuda.synchronize()
    yh = to_host(y)
    assert np.array_equal(yh, oracle.ntt_forward(x, primes))
    z = torch.empty_like(y)
    plan.inverse(y, z)
    torch.cuda.synchronize()
    assert torch.equal(z, d)
    # the inverse on its own input distribution (uniform residues read as NTT values)
    plan.inverse(d, z)
    torch.cuda.synchronize()
    assert np.array_equal(to_host(z), oracle.ntt_inverse(x, primes))
    del d, y, z
    torch.cuda.empty_cache()


def test_config2_one_ciphertext(wd):
    _full_size_check(wd, 1 << 16, 36, 2, inputs.SEED_BASE + 1)


def test_config3_headline_64_ciphertexts(wd):
    _full_size_check(wd, 1 << 16, 36, 128, inputs.SEED_BASE + 2)


def test_config4_n131072_l48(wd):
    _full_size_check(wd, 1 << 17, 48, 64, inputs.SEED_BASE + 3)


# -------------------------------------------------------------- AUTO's decision boundaries
# AUTO picks the kernel (v1 / v5 / v8 / tm) and v8's cluster size (8, 4, 2, 1 CTAs per row) from N and
# the row count, with thresholds at SM/4, SM/2, SM, 8 x SM rows and, at N = 2^13..2^16, tm's rounds of
# rows: full rounds with a small remainder run as tm + a v8 tail launch (wd_ntt.cu launch_cuda_core).
# Every N, every threshold +-1, every row of both directions against the oracle.
def _boundary_rows():
    sm = torch.cuda.get_device_properties(0).multi_processor_count if torch.cuda.is_available() else 148
    pts = {1, sm // 4 - 1, sm // 4, sm // 2, sm // 2 + 1, sm - 1, sm, sm + 1, 2 * sm - 1, 2 * sm, 2 * sm + 1,
           4 * sm - 1, 4 * sm, 4 * sm + 1, 8 * sm - 1, 8 * sm}
    return sorted(pts)


@pytest.mark.parametrize("logn", [12, 13, 14, 15, 16, 17])
def test_auto_decision_boundaries(wd, logn):
    n = 1 << logn
    for rows in _boundary_rows():
        primes = [P[(rows + logn) % 60]]
        x = inputs.uniform_residues(primes, n, rows, 7000 + logn * 10007 + rows)
        plan = wd.Plan(n, primes)
        y = gpu_fwd(wd, plan, x)
        sm = torch.cuda.get_device_properties(0).multi_processor_count
        unit = sm * (4 if logn == 13 else 1)     # tm processes rows in rounds of `unit`
        tail = rows % unit
        split = 13 <= logn <= 16 and rows >= unit and tail * 4 <= unit          # full rounds + v8 tail
        tm_alone = 13 <= logn <= 16 and not split and rows * 20 >= unit * (-(-rows // unit)) * 17
        want = "tm+v8" if split and tail else "tm" if split or tm_alone else None
        if logn == 17 and 2 * rows >= sm and 2 * rows * 20 >= sm * (-(-2 * rows // sm)) * 17:
            want = "tm17"                        # the forward on the two 2^16 halves of every row
        got = wd.wd_ntt_last_kernel()
        assert (got == want) if want else not got.startswith("tm"), (logn, rows, got)
        assert np.array_equal(y, oracle.ntt_forward(x, primes)), (logn, rows)
        assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes)), (logn, rows)
        plan.close()


# AUTO's tm + v8-tail split (full rounds of rows on tm, a remainder <= a quarter round on v8 with the
# same limb-major slot map) at row counts that are not multiples of L's: every row of both directions
@pytest.mark.parametrize("logn,L,batch", [(16, 36, 5), (16, 7, 43), (15, 5, 61), (14, 9, 33), (13, 11, 55)])
def test_auto_tm_tail_split(wd, logn, L, batch):
    n = 1 << logn
    sm = torch.cuda.get_device_properties(0).multi_processor_count
    unit = sm * (4 if logn == 13 else 1)
    rows = batch * L
    primes = [P[(11 * i + L) % 60] for i in range(L)]
    x = inputs.uniform_residues(primes, n, batch, 5900 + logn * 7 + batch)
    plan = wd.Plan(n, primes)
    y = gpu_fwd(wd, plan, x)
    tail = rows % unit
    if rows >= unit and 0 < tail * 4 <= unit:
        assert wd.wd_ntt_last_kernel() == "tm+v8", (logn, rows)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), (logn, L, batch)
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes)), (logn, L, batch)
    t = to_dev(x)
    plan.forward(t, t)                                   # in place
    plan.inverse(t, t)
    torch.cuda.synchronize()
    assert np.array_equal(to_host(t), x), (logn, L, batch)
    plan.close()


@pytest.mark.parametrize("logn,L", [(12, 1), (13, 60), (14, 17), (15, 9), (16, 60), (17, 2)])
def test_config5_sweep_batch1(wd, logn, L):
    n = 1 << logn
    primes = P[:L]
    x = inputs.uniform_residues(primes, n, 2, 5000 + logn)   # batch 1 ciphertext
    plan = wd.Plan(n, primes)
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes))


# -------------------------------------------------------------- execution modes (rows a4 / a5 / a9)
def _modes(wd):
    return ["cuda", "tensor", "fused"]


MODES = [("cuda", -1.0), ("tensor", -1.0), ("fused", -1.0), ("fused", 0.0), ("fused", 0.6),
         ("ftc", -1.0), ("ftc", 0.0), ("ftc", 0.5), ("ftc", 1.0)]


@pytest.mark.parametrize("mode,share", MODES)
def test_modes_vs_oracle_n65536(wd, mode, share):
    n = 1 << 16
    primes = [P[0], P[13], P[59]]
    x = inputs.uniform_residues(primes, n, 3, 77)
    plan = wd.Plan(n, primes)
    try:
        plan.set_mode(mode, share)
    except wd.WdNttError as e:
        pytest.fail("mode %s unavailable: %s" % (mode, e))
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), mode
    assert np.array_equal(gpu_inv(wd, plan, y), x), mode
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes)), mode
    q = inputs.structured("qm1", primes, n)
    assert np.array_equal(gpu_fwd(wd, plan, q), oracle.ntt_forward(q, primes)), mode
    assert np.array_equal(gpu_inv(wd, plan, q), oracle.ntt_inverse(q, primes)), mode


@pytest.mark.parametrize("mode,share", MODES[1:])
def test_modes_headline_config(wd, mode, share):
    n, L, batch = 1 << 16, 36, 128
    primes = P[:L]
    x = inputs.uniform_residues_torch(primes, n, batch, inputs.SEED_BASE + 2, device="cuda")
    plan = wd.Plan(n, primes)
    ref_plan = wd.Plan(n, primes, mode="cuda")
    plan.set_mode(mode, share)
    y = torch.empty_like(x)
    yr = torch.empty_like(x)
    plan.forward(x, y)
    ref_plan.forward(x, yr)
    torch.cuda.synchronize()
    assert torch.equal(y, yr)                  # bit-identical across paths, every row
    rows = [0, 1, 35, 36 * 64 + 7, batch * L - 1]
    yh = to_host(y.view(batch * L, n)[torch.as_tensor(rows, device="cuda")])
    xh = to_host(x.view(batch * L, n)[torch.as_tensor(rows, device="cuda")])
    for k, r in enumerate(rows):
        assert np.array_equal(yh[k], oracle.ntt_forward_row(xh[k], primes[r % L]))
    z = torch.empty_like(x)
    plan.inverse(y, z)
    torch.cuda.synchronize()
    assert torch.equal(z, x)


# -------------------------------------------------------------- every CUDA-core kernel generation
# WD_NTT_KERNEL (read at plan creation) forces v1 (one CTA per row), v5 (row in a cluster's DSMEM,
# N >= 2^14) or v8 (the default) regardless of the row count.
@pytest.mark.parametrize("ver", ["v1", "v5", "v8"])
@pytest.mark.parametrize("logn", [12, 13, 14, 15, 16, 17])
def test_cuda_core_generations(wd, ver, logn, monkeypatch):
    monkeypatch.setenv("WD_NTT_KERNEL", ver)
    n = 1 << logn
    primes = [P[0], P[29], P[59]]
    x = inputs.uniform_residues(primes, n, 3, 4000 + logn)
    plan = wd.Plan(n, primes, mode="cuda")
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), (ver, logn)
    assert np.array_equal(gpu_inv(wd, plan, y), x), (ver, logn)
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes)), (ver, logn)
    q = np.repeat(inputs.structured("qm1", primes, n), 3, axis=0)          # same batch as x
    assert np.array_equal(gpu_fwd(wd, plan, q), oracle.ntt_forward(q, primes)), (ver, logn)
    # the pointwise-product inverse (row f1) through the same kernel generation
    a2 = to_dev(x)
    o = torch.empty_like(a2)
    plan.pointwise_inverse(a2, to_dev(q), o)
    torch.cuda.synchronize()
    prod = (x.astype(np.uint64) * q.astype(np.uint64)) % np.array(primes, np.uint64)[None, :, None]
    assert np.array_equal(to_host(o), oracle.ntt_inverse(prod.astype(np.uint32), primes)), (ver, logn)


# v8 at every cluster size (WD_NTT_CL), over more rows than resident clusters and a ragged count
@pytest.mark.parametrize("cl", ["1", "2", "4", "8"])
@pytest.mark.parametrize("logn,batch", [(13, 301), (14, 161), (15, 97), (16, 83), (17, 45)])
def test_v8_cluster_sizes_many_rows(wd, cl, logn, batch, monkeypatch):
    monkeypatch.setenv("WD_NTT_KERNEL", "v8")
    monkeypatch.setenv("WD_NTT_CL", cl)
    n = 1 << logn
    primes = [P[1], P[7], P[30], P[58]]
    x = inputs.uniform_residues(primes, n, batch, 5100 + logn)
    plan = wd.Plan(n, primes, mode="cuda")
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), (cl, logn)
    assert np.array_equal(gpu_inv(wd, plan, y), x), (cl, logn)
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes)), (cl, logn)


# v8's column-phase feeds (WD_NTT_V8_TMA, read at plan creation; default 1): 0 register loads, 1 TMA
# forward, 2 TMA inverse, 4 inverse next-row sub-row prefetch; every cluster size, more rows than
# resident clusters (so the cross-row prefetches run), in place, and a ModUp-style strided section
@pytest.mark.parametrize("feed", ["0", "1", "2", "4", "7"])
@pytest.mark.parametrize("logn,cl", [(13, "2"), (14, "1"), (14, "4"), (15, "8"), (16, "2"), (16, "1")])
def test_v8_column_feeds(wd, feed, logn, cl, monkeypatch):
    monkeypatch.setenv("WD_NTT_KERNEL", "v8")
    monkeypatch.setenv("WD_NTT_CL", cl)
    monkeypatch.setenv("WD_NTT_V8_TMA", feed)
    n = 1 << logn
    primes = [P[2], P[9], P[44]]
    batch = 600 if logn <= 14 else 211
    x = inputs.uniform_residues(primes, n, batch, 5300 + logn)
    plan = wd.Plan(n, primes, mode="cuda")
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), (feed, logn, cl)
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes)), (feed, logn, cl)
    t = to_dev(x)
    plan.forward(t, t)                                   # in place
    plan.inverse(t, t)
    torch.cuda.synchronize()
    assert np.array_equal(to_host(t), x), (feed, logn, cl)


# tm, the TMEM-resident kernels (WD_NTT_KERNEL=tm; AUTO at N = 2^13..2^16 when its row rounds are full): fewer rows than
# SMs (idle CTAs), one row, ragged row counts against the SM count (CTAs with one row more than others),
# both layouts of the TMEM ping-pong (odd and even rows per CTA), the natural row order (WD_NTT_LM=0),
# edge inputs, in place; every row of both directions against the oracle
@pytest.mark.parametrize("logn,L,batch,lm", [(16, 1, 1, "1"), (16, 3, 1, "1"), (16, 36, 5, "1"), (16, 4, 83, "1"),
                                             (16, 60, 7, "1"), (16, 5, 61, "0"), (16, 36, 9, "0"),
                                             (15, 1, 1, "1"), (15, 36, 5, "1"), (15, 4, 83, "1"), (15, 5, 61, "0"),
                                             (14, 2, 1, "1"), (14, 36, 9, "1"), (14, 7, 100, "1"), (14, 3, 97, "0"),
                                             (13, 1, 1, "1"), (13, 36, 9, "1"), (13, 5, 150, "1"), (13, 3, 211, "0")])
def test_tm_kernel(wd, logn, L, batch, lm, monkeypatch):
    monkeypatch.setenv("WD_NTT_KERNEL", "tm")
    monkeypatch.setenv("WD_NTT_LM", lm)
    n = 1 << logn
    primes = [P[(7 * i + L) % 60] for i in range(L)]
    x = inputs.uniform_residues(primes, n, batch, 5500 + L * 131 + batch)
    plan = wd.Plan(n, primes, mode="cuda")
    y = gpu_fwd(wd, plan, x)
    assert wd.wd_ntt_last_kernel() == "tm"
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), (L, batch)
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes)), (L, batch)
    t = to_dev(x)
    plan.forward(t, t)                                   # in place
    torch.cuda.synchronize()
    assert np.array_equal(to_host(t), y), (L, batch)
    plan.inverse(t, t)
    torch.cuda.synchronize()
    assert np.array_equal(to_host(t), x), (L, batch)
    for kind in ("zeros", "qminus1"):
        e = np.zeros_like(x) if kind == "zeros" else np.broadcast_to(
            np.array(primes, dtype=np.uint32)[None, :, None] - 1, x.shape).copy()
        assert np.array_equal(gpu_fwd(wd, plan, e), oracle.ntt_forward(e, primes)), (L, batch, kind)
        assert np.array_equal(gpu_inv(wd, plan, e), oracle.ntt_inverse(e, primes)), (L, batch, kind)
    plan.close()


# N = 2^17 forward on its two 2^16 halves (tm17: AUTO when the half-row rounds are full, or WD_NTT_KERNEL=tm):
# few half-rows, ragged counts, the natural order, in place, edge inputs; the inverse stays on v8
@pytest.mark.parametrize("L,batch,lm,force", [(1, 74, "1", ""), (3, 50, "1", ""), (48, 4, "1", ""), (5, 1, "1", "tm"),
                                              (7, 11, "0", "tm"), (48, 64, "1", "")])
def test_tm17_forward(wd, L, batch, lm, force, monkeypatch):
    if force:
        monkeypatch.setenv("WD_NTT_KERNEL", force)
    monkeypatch.setenv("WD_NTT_LM", lm)
    n = 1 << 17
    primes = [P[(13 * i + L) % 60] for i in range(L)]
    x = inputs.uniform_residues(primes, n, batch, 6100 + L * 17 + batch)
    plan = wd.Plan(n, primes)
    y = gpu_fwd(wd, plan, x)
    sm = torch.cuda.get_device_properties(0).multi_processor_count
    r2 = 2 * batch * L
    if force or (r2 >= sm and r2 * 20 >= sm * (-(-r2 // sm)) * 17):
        assert wd.wd_ntt_last_kernel() == "tm17", wd.wd_ntt_last_kernel()
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), (L, batch)
    t = to_dev(x)
    plan.forward(t, t)                                   # in place
    plan.inverse(t, t)
    torch.cuda.synchronize()
    assert np.array_equal(to_host(t), x), (L, batch)
    if batch * L <= 200:
        for kind in ("zeros", "qminus1"):
            e = np.zeros_like(x) if kind == "zeros" else np.broadcast_to(
                np.array(primes, dtype=np.uint32)[None, :, None] - 1, x.shape).copy()
            assert np.array_equal(gpu_fwd(wd, plan, e), oracle.ntt_forward(e, primes)), (L, batch, kind)
    plan.close()


# Primes across the range the ABI accepts (the lazy bounds [0, 4q) < 2^32 hold for any q < 2^30).
# 786433 = 3 * 2^18 + 1; the others are the first primes = 1 (mod 2^17) above 2^28, 2^29, 1.5*2^29.
@pytest.mark.parametrize("mode", ["cuda", "tensor", "fused", "cuda_gemm"])
def test_prime_sizes_n16(wd, mode):
    n = 1 << 16
    primes = [786433, 269221889, 537133057, 805961729, P[0]]
    for q in primes:
        assert oracle.is_prime(q) and (q - 1) % (2 * n) == 0
    x = inputs.uniform_residues(primes, n, 3, 5200)
    plan = wd.Plan(n, primes, mode=mode)
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), mode
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes)), mode
    q = np.repeat(inputs.structured("qm1", primes, n), 3, axis=0)
    assert np.array_equal(gpu_fwd(wd, plan, q), oracle.ntt_forward(q, primes)), mode
    assert np.array_equal(gpu_inv(wd, plan, q), oracle.ntt_inverse(q, primes)), mode


# Every tensor-using mode at a ragged batch whose limbs change inside a CTA's row range
# (335 rows over 148 CTAs: 2-3 rows each, limb-major), every row against the oracle
@pytest.mark.parametrize("mode,share", [("tensor", -1.0), ("fused", -1.0), ("fused", 0.5), ("cuda_gemm", -1.0),
                                        ("ftc", 0.6)])
def test_tensor_modes_ragged_limbs(wd, mode, share):
    n = 1 << 16
    primes = [P[4], P[21], P[44], 786433, 805961729]
    x = inputs.uniform_residues(primes, n, 67, 5600)
    plan = wd.Plan(n, primes)
    plan.set_mode(mode, share)
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), mode
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes)), mode


# -------------------------------------------------------------- WD-CUDA (row f2): 32-bit GEMM inner DFTs
def test_wd_cuda_gemm_mode(wd):
    n = 1 << 16
    primes = [P[0], P[33], 786433, 269221889, 805961729]
    x = inputs.uniform_residues(primes, n, 3, 5300)
    plan = wd.Plan(n, primes, mode="cuda_gemm")
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes))
    assert np.array_equal(gpu_inv(wd, plan, y), x)
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes))
    q = np.repeat(inputs.structured("qm1", primes, n), 3, axis=0)
    assert np.array_equal(gpu_fwd(wd, plan, q), oracle.ntt_forward(q, primes))
    assert np.array_equal(gpu_inv(wd, plan, q), oracle.ntt_inverse(q, primes))
    with pytest.raises(wd.WdNttError):
        wd.Plan(1 << 15, P[:2], mode="cuda_gemm")          # N = 2^16 only


# -------------------------------------------------------------- WD-FTC (row f2): WD-Tensor || WD-CUDA
@pytest.mark.parametrize("batch,share", [(1, 0.6), (2, 0.5), (7, 0.6), (5, 0.2)])
def test_wd_ftc_mode(wd, batch, share):
    n = 1 << 16
    primes = [P[0], P[33], 786433, 269221889]
    x = inputs.uniform_residues(primes, n, batch, 5400 + batch)
    plan = wd.Plan(n, primes)
    plan.set_mode("ftc", share)
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), (batch, share)
    assert np.array_equal(gpu_inv(wd, plan, y), x)
    assert np.array_equal(gpu_inv(wd, plan, x), oracle.ntt_inverse(x, primes))
    d = to_dev(x)                                       # in place across the split
    plan.forward(d, d)
    torch.cuda.synchronize()
    assert np.array_equal(to_host(d), y)
    with pytest.raises(wd.WdNttError):
        wd.Plan(1 << 15, P[:2], mode="ftc")                # N = 2^16 only


# -------------------------------------------------------------- row a9: split chosen from measurement
@pytest.mark.parametrize("logn,batch", [(16, 16), (14, 8)])
def test_autotune_picks_a_path_and_stays_exact(wd, logn, batch):
    n = 1 << logn
    primes = [P[3], P[17], P[40]]
    plan = wd.Plan(n, primes)
    mode, ms = plan.autotune(batch)
    assert ms > 0
    if logn == 16:
        assert mode in (1, 2, 3, 4, 5)
    else:
        assert mode == 1                                   # only the CUDA-core path below 2^16
    x = inputs.uniform_residues(primes, n, batch, 6100 + logn)
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), (mode, logn)
    assert np.array_equal(gpu_inv(wd, plan, y), x), (mode, logn)


# -------------------------------------------------------------- tc4: the warp-specialised 4-step tcgen05 kernel
# (rows a3, a5, a9; forward; the inverse of a tc4 plan runs on the CUDA-core kernels).  Every row against the
# oracle: few rows (fewer CTAs than SMs), several rows per CTA with limbs changing inside a CTA's range (the
# stage matrices are reloaded), primes across the accepted range, edge inputs, in place.
@pytest.mark.parametrize("L,batch", [(1, 1), (3, 2), (5, 67), (36, 8), (7, 41)])
def test_tc4_forward_vs_oracle(wd, L, batch):
    n = 1 << 16
    primes = P[:L]
    x = inputs.uniform_residues(primes, n, batch, 8000 + 7 * L + batch)
    plan = wd.Plan(n, primes, mode="tc4")
    y = gpu_fwd(wd, plan, x)
    assert np.array_equal(y, oracle.ntt_forward(x, primes)), (L, batch)
    assert np.array_equal(gpu_inv(wd, plan, y), x)


def test_tc4_prime_sizes_and_edges(wd):
    n = 1 << 16
    primes = [786433, 269221889, 537133057, 805961729, P[0]]
    plan = wd.Plan(n, primes, mode="tc4")
    for kind in ("zeros", "qm1", "alt", "delta", "mono1", "gauss"):
        x = np.repeat(inputs.structured(kind, primes, n, seed=3), 3, axis=0)
        assert np.array_equal(gpu_fwd(wd, plan, x), oracle.ntt_forward(x, primes)), kind
    x = inputs.uniform_residues(primes, n, 9, 8100)
    assert np.array_equal(gpu_fwd(wd, plan, x), oracle.ntt_forward(x, primes))


def test_tc4_in_place_and_full_config3(wd):
    n, L, batch = 1 << 16, 36, 128
    primes = P[:L]
    x = inputs.uniform_residues(primes, n, batch, inputs.SEED_BASE + 2)
    plan = wd.Plan(n, primes, mode="tc4")
    d = to_dev(x)
    plan.forward(d, d)                                  # in place over the whole config-3 batch
    torch.cuda.synchronize()
    assert np.array_equal(to_host(d), oracle.ntt_forward(x, primes))
    with pytest.raises(wd.WdNttError):
        wd.Plan(1 << 15, P[:2], mode="tc4")             # N = 2^16 only
