"""GPU tests of the API surface around the transforms (include/wd_ntt.h), bit-exact vs the oracle.

* the host-buffer calls wd_ntt_forward_host / wd_ntt_inverse_host (the e2e path bench.py
  times): chunked H2D || kernel || D2H pipeline over 3 streams, batch sizes below, at and
  above its minimum of 8 chunks, ragged chunk splits, in place on the host;
* reentrancy across streams (SURVEY.md 8.b "Execution": one plan used from several streams
  at once);
* the contract for non-canonical inputs (8.b "Errors": result unspecified, no fault);
* WD_MODE_FTC (its internal fork stream) under calls from several streams at once.
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


def pinned(x: np.ndarray):
    t = torch.empty(x.shape, dtype=torch.int32, pin_memory=True)
    t.copy_(torch.from_numpy(np.ascontiguousarray(x).view(np.int32)))
    return t


@pytest.mark.parametrize("logn,L,batch", [(12, 4, 1), (12, 3, 5), (12, 2, 8), (12, 3, 11),
                                          (16, 2, 3), (17, 1, 9)])
def test_host_api_vs_oracle(wd, logn, L, batch):
    n = 1 << logn
    primes = P[:L]
    x = inputs.uniform_residues(primes, n, batch, 300 + logn + batch)
    plan = wd.Plan(n, primes)
    hx, hy = pinned(x), pinned(np.zeros_like(x))
    work = torch.empty(x.size, dtype=torch.int32, device="cuda")
    s = torch.cuda.current_stream().cuda_stream
    wd.wd_ntt_forward_host(plan.handle, hx, hy, batch, work, s)
    torch.cuda.synchronize()
    got = hy.numpy().view(np.uint32)
    rows = range(batch) if batch * L <= 12 or logn <= 12 else (0, batch - 1)
    for b in rows:
        assert np.array_equal(got[b], oracle.ntt_forward(x[b:b + 1], primes)[0]), (logn, L, batch, b)
    # inverse in place on the host buffer, as bench.py's e2e step does
    wd.wd_ntt_inverse_host(plan.handle, hy, hy, batch, work, s)
    torch.cuda.synchronize()
    assert np.array_equal(hy.numpy().view(np.uint32), x)
    assert np.array_equal(hx.numpy().view(np.uint32), x)      # input untouched


def test_host_api_matches_device_api(wd):
    n, primes, batch = 1 << 16, P[:36], 6
    x = inputs.uniform_residues(primes, n, batch, 321)
    plan = wd.Plan(n, primes)
    d = torch.from_numpy(x.view(np.int32)).cuda()
    ref = torch.empty_like(d)
    plan.forward(d, ref)
    hx, hy = pinned(x), pinned(np.zeros_like(x))
    work = torch.empty_like(d)
    wd.wd_ntt_forward_host(plan.handle, hx, hy, batch, work, torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert torch.equal(hy, ref.cpu())


def test_host_api_batch_zero_and_errors(wd):
    plan = wd.Plan(1 << 12, P[:2])
    h = pinned(np.zeros((1, 2, 4096), np.uint32))
    work = torch.empty(2 * 4096 + 4, dtype=torch.int32, device="cuda")
    s = torch.cuda.current_stream().cuda_stream
    assert wd.wd_ntt_forward_host(plan.handle, h, h, 0, work, s) == 0
    with pytest.raises(wd.WdNttError) as e:       # misaligned device scratch
        wd.wd_ntt_forward_host(plan.handle, h, h, 1, work.data_ptr() + 4, s)
    assert e.value.code == wd.WD_EINVAL


def test_one_plan_many_streams(wd):
    """8.b: calls are stream-ordered and reentrant; the plan is shared read-only."""
    n, primes, batch, ns = 1 << 14, P[:6], 4, 4
    plan = wd.Plan(n, primes)
    xs = [inputs.uniform_residues(primes, n, batch, 400 + k) for k in range(ns)]
    streams = [torch.cuda.Stream() for _ in range(ns)]
    ds = [torch.from_numpy(x.view(np.int32)).cuda() for x in xs]
    fs = [torch.empty_like(d) for d in ds]
    rs = [torch.empty_like(d) for d in ds]
    torch.cuda.synchronize()
    for _ in range(3):
        for st, d, f, r in zip(streams, ds, fs, rs):
            with torch.cuda.stream(st):
                plan.forward(d, f, stream=st.cuda_stream)
                plan.inverse(f, r, stream=st.cuda_stream)
    torch.cuda.synchronize()
    for x, f, r in zip(xs, fs, rs):
        fh = f.cpu().numpy().view(np.uint32)
        assert np.array_equal(fh[0], oracle.ntt_forward(x[:1], primes)[0])
        assert np.array_equal(r.cpu().numpy().view(np.uint32), x)


@pytest.mark.parametrize("logn", [12, 16, 17])
def test_noncanonical_inputs_do_not_fault(wd, logn):
    """8.b: inputs >= q violate the contract; the result is unspecified but nothing faults,
    and the next valid call on the same plan is still exact."""
    n, primes = 1 << logn, P[:3]
    plan = wd.Plan(n, primes)
    bad = torch.full((2, 3, n), -1, dtype=torch.int32, device="cuda")   # 0xFFFFFFFF
    out = torch.empty_like(bad)
    plan.forward(bad, out)
    plan.inverse(bad, out)
    plan.pointwise_inverse(bad, bad, out)
    torch.cuda.synchronize()
    x = inputs.uniform_residues(primes, n, 1, 77)
    d = torch.from_numpy(x.view(np.int32)).cuda()
    y = torch.empty_like(d)
    plan.forward(d, y)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().view(np.uint32), oracle.ntt_forward(x, primes))


def test_ftc_mode_many_streams(wd):
    """WD_MODE_FTC forks its tensor share onto the plan's own stream and joins it back: calls from
    several caller streams at once must stay exact (the fork stream is shared by all of them)."""
    n, primes, batch, ns = 1 << 16, P[:3], 3, 3
    plan = wd.Plan(n, primes, mode="ftc")
    xs = [inputs.uniform_residues(primes, n, batch, 500 + k) for k in range(ns)]
    streams = [torch.cuda.Stream() for _ in range(ns)]
    ds = [torch.from_numpy(x.view(np.int32)).cuda() for x in xs]
    fs = [torch.empty_like(d) for d in ds]
    rs = [torch.empty_like(d) for d in ds]
    torch.cuda.synchronize()
    for _ in range(2):
        for st, d, f, r in zip(streams, ds, fs, rs):
            with torch.cuda.stream(st):
                plan.forward(d, f, stream=st.cuda_stream)
                plan.inverse(f, r, stream=st.cuda_stream)
    torch.cuda.synchronize()
    for x, f, r in zip(xs, fs, rs):
        assert np.array_equal(f.cpu().numpy().view(np.uint32), oracle.ntt_forward(x, primes))
        assert np.array_equal(r.cpu().numpy().view(np.uint32), x)
