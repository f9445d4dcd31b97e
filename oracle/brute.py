"""Pure-Python big-int brute force of the definitions -- TEST INFRASTRUCTURE ONLY.

These are the definitions of SURVEY.md 8.c written out literally, O(N^2), for
N up to ~1024.  They pin the C oracle (``ntt_oracle.c``) and are themselves
pinned by the convolution theorem / special cases in tests/test_oracle.py.

* ``forward(x, q, psi)``:  out[i] = sum_j x[j] * psi^((2*brv(i)+1)*j) mod q
  (Eq.(1), negacyclic reading C-1, bit-reversed order C-3).
* ``inverse(y, q, psi)``:  x[j] = N^-1 * sum_i y[i] * psi^(-(2*brv(i)+1)*j) mod q
  (reading C-6).
* ``negacyclic_mul(a, b, q)``: schoolbook product in Z_q[X]/(X^N+1)
  (the CKKS ring R_Q).
"""
from __future__ import annotations


def brv(i: int, logn: int) -> int:
    return int(format(i, "0%db" % logn)[::-1], 2) if logn > 0 else 0


def _logn(n: int) -> int:
    l = n.bit_length() - 1
    assert 1 << l == n, "N must be a power of two"
    return l


def forward(x, q: int, psi: int):
    n = len(x)
    lg = _logn(n)
    out = []
    for i in range(n):
        r = pow(psi, 2 * brv(i, lg) + 1, q)       # the evaluation point
        acc, p = 0, 1
        for j in range(n):
            acc += int(x[j]) * p
            p = p * r % q
        out.append(acc % q)
    return out


def inverse(y, q: int, psi: int):
    n = len(y)
    lg = _logn(n)
    psi_inv = pow(psi, q - 2, q)
    n_inv = pow(n, q - 2, q)
    out = []
    for j in range(n):
        acc = 0
        for i in range(n):
            acc += int(y[i]) * pow(psi_inv, (2 * brv(i, lg) + 1) * j, q)
        out.append(acc * n_inv % q)
    return out


def negacyclic_mul(a, b, q: int):
    n = len(a)
    c = [0] * n
    for i in range(n):
        ai = int(a[i])
        if ai == 0:
            continue
        for j in range(n):
            k = i + j
            if k < n:
                c[k] += ai * int(b[j])
            else:
                c[k - n] -= ai * int(b[j])          # X^N = -1
    return [v % q for v in c]


def is_psi(g: int, q: int, n: int) -> bool:
    """g is a primitive 2N-th root of unity iff g^N = -1 (N a power of two)."""
    return pow(g, n, q) == q - 1
