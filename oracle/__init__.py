"""CPU oracle for the batched negacyclic RNS NTT/INTT -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
and ``--impl reference`` legs may import this package.  The product library
(``paper_conf_hpca_fanzzfzdtksy25_b200``) never imports it and shares no code
with it.

Contents:
* ``ntt_oracle.c`` -- plain C merged-psi Cooley-Tukey / Gentleman-Sande with
  ``(uint64)a*b % q`` and powmod twiddles (see its header for citations);
* ``brute.py`` -- pure-Python big-int O(N^2) evaluation of the definition and a
  schoolbook negacyclic product, for pinning the C code on small N;
* this module -- builds ``liboracle.so`` with gcc and wraps it for numpy.

Parity status: every function here is pinned (tests/test_oracle.py); nothing
is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from functools import lru_cache

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ntt_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc -O2, pthreads) if missing or stale."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-pthread",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


@lru_cache(maxsize=1)
def _lib():
    lib = ctypes.CDLL(build())
    u32, u64, i32 = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    p32 = ctypes.POINTER(ctypes.c_uint32)
    lib.orc_powmod.argtypes = [u32, u64, u32]; lib.orc_powmod.restype = u32
    lib.orc_is_prime.argtypes = [u32]; lib.orc_is_prime.restype = i32
    lib.orc_psi_min.argtypes = [u32, u32]; lib.orc_psi_min.restype = u32
    lib.orc_brv.argtypes = [u32, i32]; lib.orc_brv.restype = u32
    lib.orc_ntt_forward.argtypes = [p32, u32, u32, u32]; lib.orc_ntt_forward.restype = None
    lib.orc_ntt_inverse.argtypes = [p32, u32, u32, u32]; lib.orc_ntt_inverse.restype = None
    lib.orc_ntt_batch.argtypes = [i32, p32, p32, u32, p32, p32, u32, u32, i32]
    lib.orc_ntt_batch.restype = i32
    return lib


def _p32(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))


def powmod(a: int, e: int, q: int) -> int:
    return int(_lib().orc_powmod(a, e, q))


def is_prime(n: int) -> bool:
    return bool(_lib().orc_is_prime(n))


@lru_cache(maxsize=None)
def psi_min(q: int, n: int) -> int:
    """Minimal primitive 2N-th root of unity mod q (SURVEY.md reading C-4)."""
    return int(_lib().orc_psi_min(q, n))


def brv(i: int, logn: int) -> int:
    return int(_lib().orc_brv(i, logn))


def default_threads() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def _batch(direction: int, x: np.ndarray, primes, threads: int | None) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.uint32)
    if x.ndim == 1:
        x = x[None, None, :]
    elif x.ndim == 2:
        x = x[None, :, :]
    B, L, N = x.shape
    pr = np.ascontiguousarray(np.asarray(primes, dtype=np.uint32))
    assert pr.shape == (L,)
    psis = np.array([psi_min(int(q), N) for q in pr], dtype=np.uint32)
    out = np.empty_like(x)
    _lib().orc_ntt_batch(direction, _p32(x), _p32(out), N, _p32(pr), _p32(psis), L, B,
                         threads or default_threads())
    return out


def ntt_forward(x: np.ndarray, primes, threads: int | None = None) -> np.ndarray:
    """[B][L][N] (or [L][N], [N]) natural-order residues -> bit-reversed NTT, same shape as 3-D."""
    return _batch(+1, x, primes, threads)


def ntt_inverse(y: np.ndarray, primes, threads: int | None = None) -> np.ndarray:
    """Exact inverse of ntt_forward (bit-reversed in, natural out, N^-1 applied)."""
    return _batch(-1, y, primes, threads)


def ntt_forward_row(x: np.ndarray, q: int) -> np.ndarray:
    """One transform of one row (1-D) with the oracle's own psi."""
    a = np.ascontiguousarray(x, dtype=np.uint32).copy()
    _lib().orc_ntt_forward(_p32(a), a.shape[0], q, psi_min(q, a.shape[0]))
    return a


def ntt_inverse_row(y: np.ndarray, q: int) -> np.ndarray:
    a = np.ascontiguousarray(y, dtype=np.uint32).copy()
    _lib().orc_ntt_inverse(_p32(a), a.shape[0], q, psi_min(q, a.shape[0]))
    return a
