"""Pins of the RNS oracle (oracle/rns.py) -- CPU only.

The definition (``rescale_definition``, big-int CRT) is pinned by closed-form cases whose
result is known without any CRT: coefficients built as A = k * q_l + e with a chosen k and
offset e must rescale to exactly k (e in [-h, q_l - h)) or k + 1 (e = q_l - h, the rounding
boundary), h = floor(q_l / 2) (reading C-18).  The RNS algorithm
(``rescale_rns``) is then checked against the definition on seeded random inputs.
"""
import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from oracle import rns  # noqa: E402
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs  # noqa: E402

P = inputs.bench_primes(8)
SMALL = [786433, 269221889, 537133057, 805961729]      # q = 1 mod 2^17, spread over 2^19 .. 2^30


def _residues(vals, primes):
    """Python ints (any sign) -> [L][N] residues."""
    return np.array([[v % int(q) for v in vals] for q in primes], dtype=np.uint32)


@pytest.mark.parametrize("primes", [P[:2], P[:3], [P[0], SMALL[0], P[1], SMALL[2]], SMALL + [P[3]]])
@pytest.mark.parametrize("n", [16, 64])
def test_rescale_definition_closed_form(primes, n):
    rng = np.random.default_rng(len(primes) * 1000 + n)
    ql = int(primes[-1])
    h = ql // 2
    Qp = 1
    for q in primes[:-1]:
        Qp *= int(q)
    ks = [int(rng.integers(0, 1 << 62)) * int(rng.integers(0, 1 << 62)) % Qp for _ in range(n)]
    es = [int(rng.integers(-h, ql - h)) for _ in range(n)]
    es[0], es[1], es[2] = -h, ql - h - 1, 0                      # both edges of the "round to k" range
    vals = [k * ql + e for k, e in zip(ks, es)]
    a = oracle.ntt_forward(_residues(vals, primes)[None], primes)
    got = oracle.ntt_inverse(rns.rescale_definition(a, primes), primes[:-1])[0]
    assert np.array_equal(got, _residues(ks, primes[:-1]))
    # the rounding boundary: e = q_l - h rounds up to k + 1
    vals = [k * ql + (ql - h) for k in ks]
    a = oracle.ntt_forward(_residues(vals, primes)[None], primes)
    got = oracle.ntt_inverse(rns.rescale_definition(a, primes), primes[:-1])[0]
    assert np.array_equal(got, _residues([k + 1 for k in ks], primes[:-1]))


@pytest.mark.parametrize("primes", [P[:2], P[:5], [SMALL[1], P[2], SMALL[3]], [P[4], SMALL[0]]])
@pytest.mark.parametrize("n", [8, 256, 1024])
def test_rescale_rns_matches_definition(primes, n):
    x = inputs.uniform_residues(primes, n, 2, 7000 + n + len(primes))
    assert np.array_equal(rns.rescale_rns(x, primes), rns.rescale_definition(x, primes))


def test_rescale_rns_structured():
    primes = P[:4]
    n = 256
    for kind in ("zeros", "qm1", "alt", "delta"):
        x = inputs.structured(kind, primes, n)
        assert np.array_equal(rns.rescale_rns(x, primes), rns.rescale_definition(x, primes)), kind


# ---------------------------------------------------------------- basis conversion / ModUp / ModDown
# Pinned by the defining property of the fast basis conversion, checked with big-int CRT and
# never by re-evaluating its formula: for every coefficient there is ONE integer u in
# [0, #src) with out_j = A + u*Q (mod p_j) for every target prime p_j.
def _crt(coeffs, primes):
    return rns._crt_values(coeffs, primes)


def _prod(ps):
    r = 1
    for p in ps:
        r *= int(p)
    return r


QS = [P[0], P[1], P[2], SMALL[2]]
PS = [P[5], SMALL[3], P[6]]


@pytest.mark.parametrize("src,dst", [(QS, PS), (PS, QS), (QS[:1], PS[:1]), (QS[:2], PS)])
def test_bconv_lift_property(src, dst):
    n = 64
    x = inputs.uniform_residues(src, n, 2, 7500 + len(src) * 10 + len(dst))
    x[0, :, 0] = 0                                             # A = 0 -> exactly 0 (u = 0)
    out = rns.bconv(x, src, dst)
    Q = _prod(src)
    for b in range(2):
        A = _crt(x[b], src)
        for j in range(n):
            us = [u for u in range(len(src)) if all((A[j] + u * Q) % int(p) == int(out[b, k, j])
                                                   for k, p in enumerate(dst))]
            assert len(us) == 1, (b, j)
        assert np.all(out[0, :, 0] == 0)


def test_bconv_small_values_exact():
    # A < Q / #src: every y_i sum is then below Q ... not guaranteed; instead A = c * prod(others):
    # x is 0 in every limb but one, so the lift is exact (u = 0) and out_j = A mod p_j
    n = 16
    src, dst = QS, PS
    Q = _prod(src)
    for i, q in enumerate(src):
        x = np.zeros((1, len(src), n), dtype=np.uint32)
        x[0, i, :] = np.arange(n) * 12345 % int(q)
        A = _crt(x[0], src)
        out = rns.bconv(x, src, dst)
        for k, p in enumerate(dst):
            assert [int(v) for v in out[0, k]] == [a % int(p) for a in A]
        assert all(a < Q for a in A)


@pytest.mark.parametrize("n", [16, 256])
def test_modup_property(n):
    a = inputs.uniform_residues(QS, n, 2, 7600 + n)
    up = rns.modup(a, QS, PS)
    assert np.array_equal(up[:, :len(QS)], a)
    coeff_q = oracle.ntt_inverse(a, QS)
    coeff_p = oracle.ntt_inverse(np.ascontiguousarray(up[:, len(QS):]), PS)
    Q = _prod(QS)
    for b in range(2):
        A = _crt(coeff_q[b], QS)
        for j in range(n):
            assert any(all((A[j] + u * Q) % int(p) == int(coeff_p[b, k, j]) for k, p in enumerate(PS))
                       for u in range(len(QS)))


@pytest.mark.parametrize("n", [16, 256])
def test_moddown_property(n):
    allp = QS + PS
    a = inputs.uniform_residues(allp, n, 2, 7700 + n)
    down = rns.moddown(a, QS, PS)
    coeff = oracle.ntt_inverse(a, allp)
    cd = oracle.ntt_inverse(down, QS)
    P_ = _prod(PS)
    for b in range(2):
        A = _crt(coeff[b], allp)
        for j in range(n):
            base = (A[j] - A[j] % P_) // P_                    # floor(A / P)
            assert any(all((base - u) % int(q) == int(cd[b, i, j]) for i, q in enumerate(QS))
                       for u in range(len(PS)))


def test_moddown_exact_multiple_of_p():
    # an extended polynomial whose integer value is exactly P * X (X in [0, Q)): its P limbs are
    # 0, so the correction vanishes and ModDown returns X exactly (closed form, no CRT)
    n = 64
    allp = QS + PS
    P_ = _prod(PS)
    rng = np.random.default_rng(78)
    X = [int(rng.integers(0, 1 << 62)) * int(rng.integers(0, 1 << 62)) % _prod(QS) for _ in range(n)]
    coeff = np.array([[(x * P_) % int(q) for x in X] for q in allp], dtype=np.uint32)
    a = oracle.ntt_forward(coeff[None], allp)
    down = oracle.ntt_inverse(rns.moddown(a, QS, PS), QS)[0]
    assert np.array_equal(down, np.array([[x % int(q) for x in X] for q in QS], dtype=np.uint32))


@pytest.mark.parametrize("split", [1, 2, 3])
def test_bconv_partial_shards_sum_to_full(split):
    # limb-sharded ModUp: the shards' partial BConv sums add up (mod p_j) to the full BConv
    n = 32
    x = inputs.uniform_residues(QS, n, 2, 7900 + split)
    full = rns.bconv(x, QS, PS).astype(np.uint64)
    acc = np.zeros_like(full)
    for a0, a1 in [(0, split), (split, len(QS))]:
        acc += rns.bconv_partial(np.ascontiguousarray(x[:, a0:a1]), QS[a0:a1], QS, PS)
    for j, p in enumerate(PS):
        acc[:, j] %= int(p)
    assert np.array_equal(acc, full)
