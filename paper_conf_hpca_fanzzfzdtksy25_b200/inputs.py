"""Seeded synthetic inputs shared by the tests, ``bench.py`` and the oracle harness.

This module holds NO arithmetic of the method (no NTT, no modular reduction
beyond drawing a uniform residue, no twiddles).  It is the only code both the
CUDA path's tests and the oracle's tests import, as DESIGN.md section "Inputs"
requires.

* ``splitmix64(seed, n)`` -- the counter-based generator named in SURVEY.md
  section 8.d ("Synthetic inputs"): state_i = seed + (i+1)*0x9E3779B97F4A7C15,
  then the standard splitmix64 finaliser.
* ``uniform_residues(...)`` -- a ``[B][L][N]`` uint32 array with
  ``x = ((r >> 32) * q_l) >> 32``, i.e. uniform in [0, q_l) per limb, the
  distribution of RLWE ciphertext residues (CKKS ciphertexts
  are pairs of uniform-looking polynomials in R_Q).
* ``bench_primes(count)`` -- the prime list P of SURVEY.md 8.c reading C-5:
  the largest primes below 2^30 with q = 1 (mod 2^18), found here by plain
  trial division (independent of both the oracle's and the library's
  Miller-Rabin tests).
* structured parity inputs (zeros, all q-1, delta, monomials, ternary, small
  Gaussian) from SURVEY.md 8.d.
"""
from __future__ import annotations

import math
from functools import lru_cache

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)

SEED_BASE = 0x5EED0000


def splitmix64(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """n outputs of splitmix64 started at ``seed``; element i uses counter offset+i+1."""
    with np.errstate(over="ignore"):
        ctr = np.arange(offset + 1, offset + n + 1, dtype=np.uint64)
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + ctr * GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        z = z ^ (z >> np.uint64(31))
    return z


def uniform_residues(primes, n: int, batch: int, seed: int) -> np.ndarray:
    """[batch][L][n] uint32, element drawn as ((r>>32)*q)>>32 (uniform in [0,q))."""
    primes = np.asarray(primes, dtype=np.uint64)
    L = primes.shape[0]
    r = splitmix64(seed, batch * L * n).reshape(batch, L, n)
    with np.errstate(over="ignore"):
        x = ((r >> np.uint64(32)) * primes[None, :, None]) >> np.uint64(32)
    return x.astype(np.uint32)


def uniform_residues_torch(primes, n: int, batch: int, seed: int, device="cpu", chunk_rows: int = 256):
    """Same values as ``uniform_residues`` (bit for bit), generated with torch int64 ops
    (wrapping multiply; logical shifts emulated by masking) directly on ``device``.
    Returns an int32 tensor [batch][L][n] holding the uint32 residues."""
    import torch

    def lsr(z, s):                       # logical right shift of a 64-bit pattern
        return (z >> s) & ((1 << (64 - s)) - 1)

    def s64(v):                          # uint64 constant -> int64 bit pattern
        return v - (1 << 64) if v >= (1 << 63) else v

    g, c1, c2 = s64(int(GOLDEN)), s64(int(_C1)), s64(int(_C2))
    L = len(primes)
    out = torch.empty((batch, L, n), dtype=torch.int32, device=device)
    flat = out.view(-1)
    q = torch.tensor([int(p) for p in primes], dtype=torch.int64, device=device)
    rows = batch * L
    for r0 in range(0, rows, chunk_rows):
        r1 = min(rows, r0 + chunk_rows)
        ctr = torch.arange(r0 * n + 1, r1 * n + 1, dtype=torch.int64, device=device)
        z = s64(seed & 0xFFFFFFFFFFFFFFFF) + ctr * g
        z = (z ^ lsr(z, 30)) * c1
        z = (z ^ lsr(z, 27)) * c2
        z = z ^ lsr(z, 31)
        ql = q[(torch.arange(r0, r1, device=device) % L)].repeat_interleave(n)
        x = (lsr(z, 32) * ql) >> 32
        flat[r0 * n:r1 * n] = (x - ((x >> 31) << 32)).to(torch.int32)   # uint32 bits in int32
    return out


def structured(kind: str, primes, n: int, seed: int = 1) -> np.ndarray:
    """[1][L][n] structured inputs for parity edge cases."""
    primes = np.asarray(primes, dtype=np.int64)
    L = primes.shape[0]
    out = np.zeros((1, L, n), dtype=np.int64)
    if kind == "zeros":
        pass
    elif kind == "qm1":                 # all q-1: stresses the lazy-reduction bounds
        out[:] = (primes - 1)[None, :, None]
    elif kind == "alt":                 # alternating 0 / q-1
        out[:, :, 1::2] = (primes - 1)[None, :, None]
    elif kind == "delta":               # the constant polynomial 1
        out[:, :, 0] = 1
    elif kind.startswith("mono"):       # X^k, k given as mono<k>
        k = int(kind[4:]) % n
        out[:, :, k] = 1
    elif kind == "ternary":             # {-1,0,1} mod q (secret-key-like)
        r = splitmix64(seed, L * n).reshape(1, L, n)
        t = (r % np.uint64(3)).astype(np.int64) - 1
        out = np.where(t < 0, primes[None, :, None] - 1, t)
    elif kind == "gauss":               # rounded Gaussian sigma=3.2 via CLT of 12 uniforms
        r = splitmix64(seed, L * n * 12).reshape(1, L, n, 12)
        u = (r >> np.uint64(11)).astype(np.float64) / float(1 << 53)
        g = np.rint((u.sum(axis=-1) - 6.0) * 3.2).astype(np.int64)
        out = np.mod(g, primes[None, :, None])
    else:
        raise ValueError(kind)
    return out.astype(np.uint32)


@lru_cache(maxsize=1)
def _small_primes() -> np.ndarray:
    lim = 1 << 16                       # covers sqrt(2^32)
    s = np.ones(lim + 1, dtype=bool)
    s[:2] = False
    for i in range(2, math.isqrt(lim) + 1):
        if s[i]:
            s[i * i::i] = False
    return np.nonzero(s)[0].astype(np.int64)


def _is_prime_trial(n: int) -> bool:
    """Trial division by every prime <= sqrt(n) (n < 2^32)."""
    if n < 2:
        return False
    sp = _small_primes()
    sp = sp[sp <= math.isqrt(n)]
    return bool(np.all(n % sp != 0)) or n in set(sp.tolist())


@lru_cache(maxsize=None)
def _bench_primes_cached(count: int, log_mod: int, bits: int):
    step = 1 << log_mod
    out = []
    k = ((1 << bits) - 1) // step
    while len(out) < count and k > 0:
        q = k * step + 1
        if q < (1 << bits) and _is_prime_trial(q):
            out.append(q)
        k -= 1
    if len(out) < count:
        raise ValueError("not enough primes")
    return tuple(out)


def bench_primes(count: int, log_mod: int = 18, bits: int = 30) -> list[int]:
    """Largest ``count`` primes q < 2^bits with q = 1 (mod 2^log_mod).

    With log_mod=18 every prime is NTT-friendly for every N <= 2^17.
    """
    return list(_bench_primes_cached(count, log_mod, bits))
