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
