"""CPU oracle for the RNS pieces around the NTT -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu legs may import this
module; the product library shares no code with it.  Polynomials are ``[B][L][N]`` uint32
arrays in the NTT (evaluation) domain of ``oracle.ntt_forward`` (bit-reversed order), the
form the ciphertexts stay in between homomorphic operations.

RESCALE ("RSCALE(ct0) = (a0', b0') in R_{Q_{l-1}}"; reading C-18 of DESIGN.md):
the ciphertext polynomial a over Q_l = q_0 ... q_l is divided by its last prime with
rounding, a' = round(a / q_l) = floor((A + floor(q_l / 2)) / q_l) coefficient-wise, where A
is the integer (CRT) value of a coefficient; the result lives modulo Q_{l-1}.  (The
representative of A does not matter: Q_l / q_l = Q_{l-1}, so changing A by Q_l changes a'
by Q_{l-1}.)

* ``rescale_definition`` writes that definition out: INTT every limb, reconstruct A with
  Python big ints (CRT), divide and round, reduce mod each remaining prime, NTT back.
* ``rescale_rns`` is the RNS algorithm in its usual step order (no big integers):
    1. c   = INTT_{q_l}(a_l)                      (coefficients of the last limb)
    2. r   = (c + h) mod q_l,  h = floor(q_l / 2)
    3. v   = r - h, the residue of A mod q_l in [-h, q_l - h) (centred)
    4. u_i = NTT_{q_i}(v mod q_i)                  for every i < l
    5. a'_i = (a_i - u_i) * q_l^{-1}  mod q_i
  because A - v = (A + h) - r is the multiple of q_l at or below A + h, so (A - v) / q_l is
  floor((A + h) / q_l).
It is pinned to ``rescale_definition`` (and both to closed-form cases) in tests/test_rns_oracle.py.

Parity status: pinned (nothing here is "parity unpinned").
"""
from __future__ import annotations

import numpy as np

from . import ntt_forward, ntt_inverse


def _crt_values(coeffs: np.ndarray, primes) -> list:
    """coeffs [L][N] residues -> list of N Python ints A in [0, prod primes) (plain CRT)."""
    Q = 1
    for q in primes:
        Q *= int(q)
    terms = []
    for q in primes:
        q = int(q)
        Qi = Q // q
        terms.append((q, Qi * pow(Qi % q, -1, q)))
    n = coeffs.shape[1]
    out = []
    for j in range(n):
        acc = 0
        for l, (q, t) in enumerate(terms):
            acc += int(coeffs[l, j]) * t
        out.append(acc % Q)
    return out


def rescale_definition(a: np.ndarray, primes) -> np.ndarray:
    """[B][L][N] NTT-domain polynomials over primes[0..L-1] -> [B][L-1][N], round(A / q_{L-1})."""
    a = np.ascontiguousarray(a, dtype=np.uint32)
    B, L, N = a.shape
    assert L >= 2 and len(primes) == L
    ql = int(primes[-1])
    coeff = ntt_inverse(a, primes)
    res = np.empty((B, L - 1, N), dtype=np.uint32)
    for b in range(B):
        vals = _crt_values(coeff[b], primes)
        for i in range(L - 1):
            qi = int(primes[i])
            res[b, i] = [((A + ql // 2) // ql) % qi for A in vals]
    return ntt_forward(res, primes[:-1])


def rescale_rns(a: np.ndarray, primes) -> np.ndarray:
    """The RNS rescale algorithm, step by step (see module docstring)."""
    a = np.ascontiguousarray(a, dtype=np.uint32)
    B, L, N = a.shape
    assert L >= 2 and len(primes) == L
    ql = int(primes[-1])
    h = ql // 2
    c = ntt_inverse(a[:, L - 1:L, :], [ql])[:, 0, :].astype(np.uint64)         # step 1
    r = (c + h) % ql                                                             # step 2
    v = r.astype(np.int64) - h                                                   # step 3
    out = np.empty((B, L - 1, N), dtype=np.uint32)
    for i in range(L - 1):
        qi = int(primes[i])
        u = ntt_forward((v % qi).astype(np.uint32)[:, None, :], [qi])[:, 0, :]   # step 4
        inv = pow(ql % qi, -1, qi)
        t = (a[:, i, :].astype(np.uint64) + qi - u.astype(np.uint64)) % qi
        out[:, i, :] = (t * inv % qi).astype(np.uint32)                          # step 5
    return out


# ---------------------------------------------------------------------------------------------
# Basis conversion, ModUp, ModDown (Table III and
# PAPER.md:350 Fig. 4 name them as the KeySwitch kernels around the NTT; the paper does not
# restate their formulas, so DESIGN.md reading C-19 takes the standard RNS-CKKS ones of the
# "100x" baseline it compares against): for a source basis {q_i} with product Q,
#   BConv_{Q->P}(x)_j = sum_i [x_i * (Q/q_i)^{-1}]_{q_i} * (Q/q_i)  mod p_j
# which equals (A + u Q) mod p_j for the integer value A of x and one u in [0, #q) (the fast,
# approximate lift: it does not remove the multiple u Q).
#   ModUp(a)   = a on the Q limbs, NTT_P(BConv_{Q->P}(INTT_Q(a))) on the P limbs
#   ModDown(a) = (a_Q - NTT_Q(BConv_{P->Q}(INTT_P(a_P)))) * P^{-1}  on the Q limbs
# All polynomials in and out are NTT-domain (bit-reversed order), [B][limbs][N].

def bconv(x: np.ndarray, src, dst) -> np.ndarray:
    """Coefficient-domain fast basis conversion [B][len(src)][N] -> [B][len(dst)][N] (literal)."""
    x = np.ascontiguousarray(x, dtype=np.uint32)
    B, a, N = x.shape
    assert a == len(src)
    Q = 1
    for q in src:
        Q *= int(q)
    out = np.zeros((B, len(dst), N), dtype=np.uint32)
    ys = []
    for i, q in enumerate(src):
        q = int(q)
        qhat = Q // q
        ys.append((x[:, i, :].astype(object) * pow(qhat % q, -1, q)) % q)       # y_i, exact ints
    for j, p in enumerate(dst):
        p = int(p)
        acc = np.zeros((B, N), dtype=object)
        for i, q in enumerate(src):
            acc = acc + ys[i] * ((Q // int(q)) % p)
        out[:, j, :] = (acc % p).astype(np.uint64).astype(np.uint32)
    return out


def modup(a: np.ndarray, qs, ps) -> np.ndarray:
    """[B][#q][N] NTT over qs -> [B][#q + #p][N] NTT over qs + ps."""
    a = np.ascontiguousarray(a, dtype=np.uint32)
    coeff = ntt_inverse(a, qs)
    ext = ntt_forward(bconv(coeff, qs, ps), ps)
    return np.concatenate([a, ext], axis=1)


def moddown(a: np.ndarray, qs, ps) -> np.ndarray:
    """[B][#q + #p][N] NTT over qs + ps -> [B][#q][N] NTT over qs: (a - BConv(a_P)) / P."""
    a = np.ascontiguousarray(a, dtype=np.uint32)
    nq = len(qs)
    P = 1
    for p in ps:
        P *= int(p)
    cp = ntt_inverse(np.ascontiguousarray(a[:, nq:, :]), ps)
    corr = ntt_forward(bconv(cp, ps, qs), qs)
    out = np.empty((a.shape[0], nq, a.shape[2]), dtype=np.uint32)
    for i, q in enumerate(qs):
        q = int(q)
        t = (a[:, i, :].astype(np.uint64) + q - corr[:, i, :].astype(np.uint64)) % q
        out[:, i, :] = (t * pow(P % q, -1, q) % q).astype(np.uint32)
    return out


def bconv_partial(x: np.ndarray, local_src, all_src, dst) -> np.ndarray:
    """One limb shard's share of BConv_{Q->P} (limb-sharded ModUp, SURVEY.md 8 rows e/f3):
    the terms of ``bconv`` for the source limbs this shard holds, with Q the product of ALL
    source primes; returns [B][len(dst)][N] residues mod p_j (uint64).  Summing the shards'
    results mod p_j gives ``bconv(x_all, all_src, dst)``."""
    x = np.ascontiguousarray(x, dtype=np.uint32)
    B, a, N = x.shape
    assert a == len(local_src)
    Q = 1
    for q in all_src:
        Q *= int(q)
    out = np.zeros((B, len(dst), N), dtype=np.uint64)
    for j, p in enumerate(dst):
        p = int(p)
        acc = np.zeros((B, N), dtype=object)
        for i, q in enumerate(local_src):
            q = int(q)
            y = (x[:, i, :].astype(object) * pow((Q // q) % q, -1, q)) % q
            acc = acc + y * ((Q // q) % p)
        out[:, j, :] = (acc % p).astype(np.uint64)
    return out
