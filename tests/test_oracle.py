"""Pins for the CPU oracle (oracle/).  CPU only.

The paper prints no NTT test vectors, so the oracle is pinned
by mathematics: the O(N^2) definition, the convolution theorem, closed-form
special cases, exhaustive minimality of psi, a hand-worked example, and the
round trip.  Each is chosen so a plausible slip (dropped twist, wrong
bit-reversal, transposed index, missing N^-1, wrong root) fails one of them.
"""
import json
import os

import numpy as np
import pytest

import oracle
from oracle import brute
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs

GOLD = os.path.join(os.path.dirname(__file__), "golden")
P = inputs.bench_primes(60)


def _rand(n, q, seed):
    return inputs.uniform_residues([q], n, 1, seed)[0, 0]


# ---------------------------------------------------------------- primes / psi
def test_miller_rabin_matches_trial_division():
    # known traps: Carmichael numbers and strong pseudoprimes to small bases
    traps = [561, 1105, 1729, 2047, 3277, 4033, 4681, 25326001, 3215031751, 2152302898747 % (1 << 32)]
    r = inputs.splitmix64(7, 3000)
    cands = [int(v) & 0xFFFFFFFF for v in r[:1500]] + [int(v) & 0xFFFFF for v in r[1500:]]
    for n in traps + cands + list(range(0, 200)):
        assert oracle.is_prime(n) == inputs._is_prime_trial(n), n


def test_bench_prime_list():
    # P[0]=2^30-2^18+1 ... ; every prime = 1 mod 2^18 and < 2^30
    assert P[:3] == [1073479681, 1068236801, 1062469633]
    assert P[0] == (1 << 30) - (1 << 18) + 1
    for q in P:
        assert q < (1 << 30) and q % (1 << 18) == 1 and oracle.is_prime(q)
    assert P == sorted(P, reverse=True)


def _powvec(g, e, q):
    g = g.astype(np.uint64)
    r = np.ones_like(g)
    b = g % np.uint64(q)
    while e:
        if e & 1:
            r = (r * b) % np.uint64(q)
        b = (b * b) % np.uint64(q)
        e >>= 1
    return r


@pytest.mark.parametrize("q,n", [(P[0], 1 << 12), (P[0], 1 << 16), (P[0], 1 << 17),
                                 (P[5], 1 << 16), (97, 16), (17, 4), (P[1], 1 << 10)])
def test_psi_min_is_minimal_primitive_root(q, n):
    psi = oracle.psi_min(q, n)
    assert pow(psi, n, q) == q - 1                      # psi^N = -1: primitive 2N-th root
    g = np.arange(2, psi, dtype=np.uint64)              # exhaustive: nothing smaller works
    assert not np.any(_powvec(g, n, q) == q - 1)


def test_psi_min_survey_constants():
    # SURVEY.md App. A1 (computed there two ways): q = 2^30-2^18+1
    assert oracle.psi_min(P[0], 1 << 12) == 769236
    assert oracle.psi_min(P[0], 1 << 16) == 4051
    assert oracle.psi_min(P[0], 1 << 17) == 25785


# ---------------------------------------------------------------- golden
def test_hand_worked_example():
    g = json.load(open(os.path.join(GOLD, "ntt_n4_q17.json")))
    assert oracle.psi_min(g["q"], g["N"]) == g["psi"]
    out = oracle.ntt_forward_row(np.array(g["x"], np.uint32), g["q"])
    assert out.tolist() == g["ntt"]
    back = oracle.ntt_inverse_row(out, g["q"])
    assert back.tolist() == g["x"]


# ---------------------------------------------------------------- definition
@pytest.mark.parametrize("logn", range(1, 9))
@pytest.mark.parametrize("q", [P[0], P[7], 12289])
def test_forward_matches_definition(logn, q):
    n = 1 << logn
    if (q - 1) % (2 * n):
        pytest.skip("q not NTT-friendly for this N")
    psi = oracle.psi_min(q, n)
    x = _rand(n, q, 100 + logn)
    assert oracle.ntt_forward_row(x, q).tolist() == brute.forward(x.tolist(), q, psi)


def test_forward_matches_definition_n1024():
    q, n = P[2], 1024
    x = _rand(n, q, 5)
    assert oracle.ntt_forward_row(x, q).tolist() == brute.forward(x.tolist(), q, oracle.psi_min(q, n))


@pytest.mark.parametrize("logn", [1, 2, 3, 5, 6])
def test_inverse_matches_definition(logn):
    q, n = P[3], 1 << logn
    y = _rand(n, q, 200 + logn)
    assert oracle.ntt_inverse_row(y, q).tolist() == brute.inverse(y.tolist(), q, oracle.psi_min(q, n))


@pytest.mark.parametrize("logn", [4, 12, 16, 17])
def test_round_trip(logn):
    q, n = P[1], 1 << logn
    x = _rand(n, q, 300 + logn)
    y = oracle.ntt_forward_row(x, q)
    assert np.array_equal(oracle.ntt_inverse_row(y, q), x)
    assert np.array_equal(oracle.ntt_forward_row(oracle.ntt_inverse_row(x, q), q), x)


# ---------------------------------------------------------------- ring structure
@pytest.mark.parametrize("logn", [3, 6, 8])
def test_negacyclic_convolution_theorem(logn):
    q, n = P[4], 1 << logn
    a, b = _rand(n, q, 1), _rand(n, q, 2)
    c = np.array(brute.negacyclic_mul(a.tolist(), b.tolist(), q), dtype=np.uint32)
    lhs = oracle.ntt_forward_row(c, q).astype(np.uint64)
    rhs = (oracle.ntt_forward_row(a, q).astype(np.uint64) *
           oracle.ntt_forward_row(b, q).astype(np.uint64)) % np.uint64(q)
    assert np.array_equal(lhs, rhs)


@pytest.mark.parametrize("logn", [4, 10, 12])
def test_special_cases(logn):
    q, n = P[6], 1 << logn
    psi = oracle.psi_min(q, n)
    one = np.zeros(n, np.uint32); one[0] = 1
    assert np.all(oracle.ntt_forward_row(one, q) == 1)              # delta -> ones
    c = np.zeros(n, np.uint32); c[0] = 123456
    assert np.all(oracle.ntt_forward_row(c, q) == 123456)           # constant -> constant
    X = np.zeros(n, np.uint32); X[1] = 1
    r = oracle.ntt_forward_row(X, q).astype(np.int64)               # X -> the roots of X^N+1
    assert len(set(r.tolist())) == n
    assert all(pow(int(v), n, q) == q - 1 for v in r[: min(n, 64)])
    lg = logn
    expect = [pow(psi, 2 * brute.brv(i, lg) + 1, q) for i in range(n)]
    assert r.tolist() == expect                                       # ...in bit-reversed order
    x = _rand(n, q, 9)
    y = oracle.ntt_forward_row(x, q).astype(np.int64)
    assert int(y.sum()) % q == n * int(x[0]) % q                      # sum rule
    xs = np.zeros(n, np.int64)                                        # X*x mod X^N+1
    xs[1:] = x[:-1]; xs[0] = (q - int(x[-1])) % q
    ys = oracle.ntt_forward_row(xs.astype(np.uint32), q).astype(np.int64)
    assert np.array_equal(ys, (y * np.array(expect, np.int64)) % q)  # shift rule


def test_batch_driver_matches_rows():
    primes = P[:3]
    x = inputs.uniform_residues(primes, 256, 4, 77)
    y = oracle.ntt_forward(x, primes, threads=3)
    for b in range(4):
        for l, q in enumerate(primes):
            assert np.array_equal(y[b, l], oracle.ntt_forward_row(x[b, l], q))
    z = oracle.ntt_inverse(y, primes, threads=2)
    assert np.array_equal(z, x)
