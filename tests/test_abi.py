"""C-ABI boundary checks that need no GPU: the library builds and loads, exports
every function include/wd_ntt.h declares, validates arguments before touching
CUDA, and its host-side plan math (prime test, psi) agrees with the oracle.
"""
import ctypes

import pytest

import oracle
from paper_conf_hpca_fanzzfzdtksy25_b200 import build as wdbuild
from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs

wdbuild.build()
from paper_conf_hpca_fanzzfzdtksy25_b200 import wdntt  # noqa: E402

P = inputs.bench_primes(8)


def test_exports_every_header_symbol():
    names = wdntt.header_functions()
    assert "wd_ntt_plan_create" in names and "wd_ntt_forward" in names
    lib = ctypes.CDLL(wdntt.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), n


def test_sm100a_code_present():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", wdntt.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_create_rejects_bad_arguments_without_gpu():
    E = wdntt
    for n, primes, code in [
        (4096, [P[0]], None),                       # valid: may fail later only with WD_ECUDA on CPU
        (3000, [P[0]], E.WD_EUNSUPPORTED),          # N not a power of two
        (1 << 18, [P[0]], E.WD_EUNSUPPORTED),       # N too large
        (4096, [P[0] + 2], E.WD_EPRIME),            # composite / not = 1 mod 2N
        (4096, [1073741827], E.WD_EPRIME),          # >= 2^30
        (4096, [12289], E.WD_EPRIME),               # prime but 12289 != 1 mod 8192
        (1024, [12289], None),                      # 12289 = 1 mod 2048: valid
    ]:
        arr = (ctypes.c_uint32 * len(primes))(*primes)
        h = wdntt._lib.wd_ntt_plan_create(n, arr, len(primes))
        if code is None:
            if h:
                wdntt._lib.wd_ntt_plan_destroy(h)
            else:
                assert wdntt.wd_ntt_last_error() in (E.WD_ECUDA, E.WD_ENOMEM)
        else:
            assert not h
            assert wdntt.wd_ntt_last_error() == code, (n, primes)
    assert not wdntt._lib.wd_ntt_plan_create(4096, None, 1)
    assert wdntt.wd_ntt_last_error() == E.WD_EINVAL
    arr = (ctypes.c_uint32 * 1)(P[0])
    assert not wdntt._lib.wd_ntt_plan_create(4096, arr, 0)
    assert wdntt.wd_ntt_last_error() == E.WD_EUNSUPPORTED


def test_calls_reject_null_plan():
    assert wdntt._lib.wd_ntt_forward(None, 16, 16, 1, None) == wdntt.WD_EINVAL
    assert wdntt._lib.wd_ntt_inverse(None, 16, 16, 1, None) == wdntt.WD_EINVAL
    assert wdntt._lib.wd_ntt_forward_host(None, 16, 16, 1, 16, None) == wdntt.WD_EINVAL
    assert wdntt._lib.wd_ntt_plan_autotune(None, 1, None, None) == wdntt.WD_EINVAL
    assert wdntt.wd_ntt_strerror(wdntt.WD_EPRIME).startswith("modulus")


@pytest.mark.parametrize("logn", [2, 4, 10, 12, 16, 17])
def test_plan_psi_matches_oracle(logn):
    n = 1 << logn
    for q in P[:3] + ([12289] if logn <= 10 else []) + ([17] if logn == 2 else []):
        assert wdntt.wd_ntt_root(q, n) == oracle.psi_min(q, n), (q, n)


def test_check_prime_matches_oracle():
    r = inputs.splitmix64(3, 400)
    for v in r:
        q = int(v) & ((1 << 30) - 1)
        q = (q >> 13 << 13) + 1                   # = 1 mod 8192 candidates
        if q >= (1 << 30):
            continue
        expect = oracle.is_prime(q)
        assert (wdntt.wd_ntt_check_prime(q, 4096) == 0) == expect, q


def test_binding_constants_match_header():
    """The Python binding's error and mode codes are the header's #defines (one source of truth)."""
    import os
    import re
    hdr = open(os.path.join(os.path.dirname(__file__), "..", "include", "wd_ntt.h")).read()
    defs = {m.group(1): int(m.group(2)) for m in re.finditer(r"#define\s+(WD_[A-Z0-9_]+)\s+(\d+)", hdr)}
    modes = {k: v for k, v in defs.items() if k.startswith("WD_MODE_")}
    assert len(modes) == 7 and modes["WD_MODE_FTC"] == 5 and modes["WD_MODE_TC4"] == 6
    for name, val in defs.items():
        if hasattr(wdntt, name):
            assert getattr(wdntt, name) == val, name
    for name in modes:
        assert getattr(wdntt, name) == modes[name], name
    assert sorted(wdntt.MODES.values()) == sorted(modes.values())
