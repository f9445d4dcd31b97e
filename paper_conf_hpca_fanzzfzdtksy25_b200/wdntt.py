"""Thin ctypes binding of libwdntt.so (include/wd_ntt.h).

Argument marshalling only: every step of the transform runs in the CUDA
library.  The function names are the C ABI's names.  Tensors are accepted
wherever the C side takes a device pointer (``t.data_ptr()`` is passed; use
int32/uint32 tensors holding uint32 residues); the stream defaults to torch's
current stream on the tensor's device.

There is deliberately NO fallback: if libwdntt.so is missing or fails to load,
importing this module raises.
"""
from __future__ import annotations

import ctypes
import os
import re

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libwdntt.so")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "wd_ntt.h")

WD_OK, WD_EINVAL, WD_EPRIME, WD_EUNSUPPORTED, WD_ECUDA, WD_ENOMEM = range(6)
WD_MODE_AUTO, WD_MODE_CUDA, WD_MODE_TENSOR, WD_MODE_FUSED, WD_MODE_CUDA_GEMM, WD_MODE_FTC, WD_MODE_TC4 = range(7)
MODES = {"auto": WD_MODE_AUTO, "cuda": WD_MODE_CUDA, "tensor": WD_MODE_TENSOR, "fused": WD_MODE_FUSED,
         "cuda_gemm": WD_MODE_CUDA_GEMM, "ftc": WD_MODE_FTC, "tc4": WD_MODE_TC4}


class WdNttError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        self.code = code
        super().__init__("%s: %s (code %d)" % (what, wd_ntt_strerror(code), code))


if not os.path.exists(LIB_PATH):
    raise ImportError("libwdntt.so not built: run `python -m paper_conf_hpca_fanzzfzdtksy25_b200.build` "
                      "(no CPU fallback exists by design)")
_lib = ctypes.CDLL(LIB_PATH)

_u32, _i32, _f32, _vp = ctypes.c_uint32, ctypes.c_int, ctypes.c_float, ctypes.c_void_p
_P32 = ctypes.POINTER(ctypes.c_uint32)

_SIGS = {
    "wd_ntt_plan_create": (_vp, [_u32, _P32, _u32]),
    "wd_ntt_plan_destroy": (None, [_vp]),
    "wd_ntt_forward": (_i32, [_vp, _vp, _vp, _u32, _vp]),
    "wd_ntt_inverse": (_i32, [_vp, _vp, _vp, _u32, _vp]),
    "wd_ntt_forward_host": (_i32, [_vp, _vp, _vp, _u32, _vp, _vp]),
    "wd_ntt_inverse_host": (_i32, [_vp, _vp, _vp, _u32, _vp, _vp]),
    "wd_ntt_pointwise_inverse": (_i32, [_vp, _vp, _vp, _vp, _u32, _vp]),
    "wd_rescale": (_i32, [_vp, _vp, _vp, _u32, _vp, _vp]),
    "wd_rns_conv_create": (_vp, [_vp, _vp]),
    "wd_rns_conv_create_shard": (_vp, [_vp, _vp, _P32, _u32]),
    "wd_modup_partial": (_i32, [_vp, _vp, _vp, _u32, _vp, _vp]),
    "wd_modup_finish": (_i32, [_vp, _vp, _vp, _u32, _vp]),
    "wd_rns_conv_destroy": (None, [_vp]),
    "wd_modup": (_i32, [_vp, _vp, _vp, _u32, _vp, _vp]),
    "wd_moddown": (_i32, [_vp, _vp, _vp, _u32, _vp, _vp]),
    "wd_ntt_plan_n": (_u32, [_vp]),
    "wd_ntt_plan_limbs": (_u32, [_vp]),
    "wd_ntt_plan_psi": (_u32, [_vp, _u32]),
    "wd_ntt_root": (_u32, [_u32, _u32]),
    "wd_ntt_check_prime": (_i32, [_u32, _u32]),
    "wd_ntt_plan_set_mode": (_i32, [_vp, _i32, _f32]),
    "wd_ntt_plan_autotune": (_i32, [_vp, _u32, _vp, ctypes.POINTER(ctypes.c_float)]),
    "wd_ntt_plan_get_mode": (_i32, [_vp]),
    "wd_ntt_last_launches": (_u32, []),
    "wd_ntt_last_kernel": (ctypes.c_char_p, []),
    "wd_ntt_debug_tc4_trace": (None, [_vp]),
    "wd_ntt_last_error": (_i32, []),
    "wd_ntt_strerror": (ctypes.c_char_p, [_i32]),
    "wd_ntt_version": (ctypes.c_char_p, []),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args


def header_functions() -> list[str]:
    """Names of every function declared in include/wd_ntt.h."""
    src = open(HEADER).read()
    return sorted(set(re.findall(r"\b(wd_ntt_\w+)\s*\(", src)))


def _ptr(x) -> int:
    if x is None:
        return 0
    if isinstance(x, int):
        return x
    return x.data_ptr()


def _stream(s, like=None) -> int:
    if s is None:
        import torch
        dev = like.device if like is not None and hasattr(like, "device") else None
        return torch.cuda.current_stream(dev).cuda_stream
    if isinstance(s, int):
        return s
    return s.cuda_stream


def _check(code: int, what: str) -> int:
    if code != WD_OK:
        raise WdNttError(code, what)
    return code


# ---- the ABI, same names -------------------------------------------------------
def wd_ntt_plan_create(N: int, primes, L: int | None = None) -> int:
    primes = [int(q) for q in primes]
    L = len(primes) if L is None else L
    arr = (ctypes.c_uint32 * len(primes))(*primes)
    h = _lib.wd_ntt_plan_create(N, arr, L)
    if not h:
        raise WdNttError(_lib.wd_ntt_last_error(), "wd_ntt_plan_create")
    return h


def wd_ntt_plan_destroy(plan: int) -> None:
    _lib.wd_ntt_plan_destroy(plan)


def wd_ntt_forward(plan: int, inp, out, batch: int, stream=None) -> int:
    return _check(_lib.wd_ntt_forward(plan, _ptr(inp), _ptr(out), batch, _stream(stream, inp)), "wd_ntt_forward")


def wd_ntt_inverse(plan: int, inp, out, batch: int, stream=None) -> int:
    return _check(_lib.wd_ntt_inverse(plan, _ptr(inp), _ptr(out), batch, _stream(stream, inp)), "wd_ntt_inverse")


def wd_ntt_pointwise_inverse(plan: int, a, b, out, batch: int, stream=None) -> int:
    return _check(_lib.wd_ntt_pointwise_inverse(plan, _ptr(a), _ptr(b), _ptr(out), batch, _stream(stream, a)),
                  "wd_ntt_pointwise_inverse")


def wd_rescale(plan: int, inp, out, batch: int, work, stream=None) -> int:
    return _check(_lib.wd_rescale(plan, _ptr(inp), _ptr(out), batch, _ptr(work), _stream(stream, inp)), "wd_rescale")


def wd_rns_conv_create(plan_q: int, plan_p: int) -> int:
    h = _lib.wd_rns_conv_create(plan_q, plan_p)
    if not h:
        raise WdNttError(_lib.wd_ntt_last_error(), "wd_rns_conv_create")
    return h


def wd_rns_conv_create_shard(plan_q_local: int, plan_p: int, q_all) -> int:
    q_all = [int(q) for q in q_all]
    arr = (ctypes.c_uint32 * len(q_all))(*q_all)
    h = _lib.wd_rns_conv_create_shard(plan_q_local, plan_p, arr, len(q_all))
    if not h:
        raise WdNttError(_lib.wd_ntt_last_error(), "wd_rns_conv_create_shard")
    return h


def wd_modup_partial(conv: int, inp, partial, batch: int, work, stream=None) -> int:
    return _check(_lib.wd_modup_partial(conv, _ptr(inp), _ptr(partial), batch, _ptr(work), _stream(stream, inp)),
                  "wd_modup_partial")


def wd_modup_finish(conv: int, total, out_p, batch: int, stream=None) -> int:
    return _check(_lib.wd_modup_finish(conv, _ptr(total), _ptr(out_p), batch, _stream(stream, total)),
                  "wd_modup_finish")


def wd_rns_conv_destroy(conv: int) -> None:
    _lib.wd_rns_conv_destroy(conv)


def wd_modup(conv: int, inp, out, batch: int, work, stream=None) -> int:
    return _check(_lib.wd_modup(conv, _ptr(inp), _ptr(out), batch, _ptr(work), _stream(stream, inp)), "wd_modup")


def wd_moddown(conv: int, inp, out, batch: int, work, stream=None) -> int:
    return _check(_lib.wd_moddown(conv, _ptr(inp), _ptr(out), batch, _ptr(work), _stream(stream, inp)), "wd_moddown")


def wd_ntt_forward_host(plan: int, h_in, h_out, batch: int, d_work, stream=None) -> int:
    return _check(_lib.wd_ntt_forward_host(plan, _ptr(h_in), _ptr(h_out), batch, _ptr(d_work),
                                           _stream(stream, d_work)), "wd_ntt_forward_host")


def wd_ntt_inverse_host(plan: int, h_in, h_out, batch: int, d_work, stream=None) -> int:
    return _check(_lib.wd_ntt_inverse_host(plan, _ptr(h_in), _ptr(h_out), batch, _ptr(d_work),
                                           _stream(stream, d_work)), "wd_ntt_inverse_host")


def wd_ntt_plan_n(plan: int) -> int:
    return _lib.wd_ntt_plan_n(plan)


def wd_ntt_plan_limbs(plan: int) -> int:
    return _lib.wd_ntt_plan_limbs(plan)


def wd_ntt_plan_psi(plan: int, limb: int) -> int:
    return _lib.wd_ntt_plan_psi(plan, limb)


def wd_ntt_root(q: int, N: int) -> int:
    return _lib.wd_ntt_root(q, N)


def wd_ntt_check_prime(q: int, N: int) -> int:
    return _lib.wd_ntt_check_prime(q, N)


def wd_ntt_plan_set_mode(plan: int, mode, tensor_share: float = -1.0) -> int:
    mode = MODES[mode] if isinstance(mode, str) else int(mode)
    return _check(_lib.wd_ntt_plan_set_mode(plan, mode, float(tensor_share)), "wd_ntt_plan_set_mode")


def wd_ntt_plan_get_mode(plan: int) -> int:
    return _lib.wd_ntt_plan_get_mode(plan)


def wd_ntt_last_launches() -> int:
    return _lib.wd_ntt_last_launches()


def wd_ntt_last_kernel() -> str:
    return _lib.wd_ntt_last_kernel().decode()


def wd_ntt_last_error() -> int:
    return _lib.wd_ntt_last_error()


def wd_ntt_strerror(code: int) -> str:
    return _lib.wd_ntt_strerror(code).decode()


def wd_ntt_version() -> str:
    return _lib.wd_ntt_version().decode()


# ---- small convenience wrapper (still marshalling only) ----------------------
class Plan:
    """RAII wrapper: ``Plan(N, primes)``; ``forward(x, out=None)`` on [B][L][N] int32/uint32 tensors."""

    def __init__(self, N: int, primes, mode: str | int | None = None, tensor_share: float = -1.0):
        self.N, self.primes, self.L = int(N), [int(q) for q in primes], len(primes)
        self.handle = wd_ntt_plan_create(self.N, self.primes)
        if mode is not None:
            self.set_mode(mode, tensor_share)

    def set_mode(self, mode, tensor_share: float = -1.0):
        wd_ntt_plan_set_mode(self.handle, mode, tensor_share)

    def autotune(self, batch: int, stream=None):
        """Time every execution path on ``batch`` scratch polynomials and keep the fastest
        (wd_ntt_plan_autotune).  Returns (mode, ms per forward + inverse)."""
        import torch
        ms = ctypes.c_float(0.0)
        st = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        _check(_lib.wd_ntt_plan_autotune(self.handle, int(batch), st, ctypes.byref(ms)), "wd_ntt_plan_autotune")
        return _lib.wd_ntt_plan_get_mode(self.handle), ms.value

    def psi(self, limb: int) -> int:
        return wd_ntt_plan_psi(self.handle, limb)

    def _batch(self, x) -> int:
        n = x.numel()
        assert n % (self.L * self.N) == 0 and x.is_contiguous(), "expect contiguous [B][L][N]"
        return n // (self.L * self.N)

    def forward(self, x, out=None, stream=None):
        out = x if out is None else out
        wd_ntt_forward(self.handle, x, out, self._batch(x), stream)
        return out

    def inverse(self, y, out=None, stream=None):
        out = y if out is None else out
        wd_ntt_inverse(self.handle, y, out, self._batch(y), stream)
        return out

    def pointwise_inverse(self, a, b, out=None, stream=None):
        out = a if out is None else out
        wd_ntt_pointwise_inverse(self.handle, a, b, out, self._batch(a), stream)
        return out

    def rescale(self, x, out=None, work=None, stream=None):
        """[B][L][N] NTT-domain -> [B][L-1][N] NTT-domain, round(x / primes[-1]) (wd_rescale)."""
        import torch
        b = self._batch(x)
        if out is None:
            out = torch.empty((b, self.L - 1, self.N), dtype=x.dtype, device=x.device)
        if work is None:
            work = torch.empty((b, self.N), dtype=x.dtype, device=x.device)
        wd_rescale(self.handle, x, out, b, work, stream)
        return out

    def close(self):
        if getattr(self, "handle", None):
            wd_ntt_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass


class RnsConv:
    """RAII wrapper of wd_rns_conv: ModUp / ModDown between ``plan_q`` (a limbs) and ``plan_p`` (k limbs)."""

    def __init__(self, plan_q: "Plan", plan_p: "Plan", q_all=None):
        self.pq, self.pp = plan_q, plan_p              # keep the plans alive
        if q_all is None:
            self.handle = wd_rns_conv_create(plan_q.handle, plan_p.handle)
        else:                                          # plan_q is one limb shard of q_all
            self.handle = wd_rns_conv_create_shard(plan_q.handle, plan_p.handle, q_all)

    def modup_partial(self, x, partial=None, work=None, stream=None):
        """This shard's 64-bit share of BConv_{Q->P}: [B][k][N] int64 (sum over shards, then finish)."""
        import torch
        a, k, n = self.pq.L, self.pp.L, self.pq.N
        b = x.numel() // (a * n)
        partial = torch.empty((b, k, n), dtype=torch.int64, device=x.device) if partial is None else partial
        work = torch.empty((b, a, n), dtype=x.dtype, device=x.device) if work is None else work
        wd_modup_partial(self.handle, x, partial, b, work, stream)
        return partial

    def modup_finish(self, total, out=None, stream=None):
        """Summed partials -> the P limbs of ModUp, NTT domain [B][k][N]."""
        import torch
        k, n = self.pp.L, self.pp.N
        b = total.numel() // (k * n)
        out = torch.empty((b, k, n), dtype=torch.int32, device=total.device) if out is None else out
        wd_modup_finish(self.handle, total, out, b, stream)
        return out

    def modup(self, x, out=None, work=None, stream=None):
        import torch
        a, k, n = self.pq.L, self.pp.L, self.pq.N
        b = x.numel() // (a * n)
        out = torch.empty((b, a + k, n), dtype=x.dtype, device=x.device) if out is None else out
        work = torch.empty((b, a, n), dtype=x.dtype, device=x.device) if work is None else work
        wd_modup(self.handle, x, out, b, work, stream)
        return out

    def moddown(self, x, out=None, work=None, stream=None):
        import torch
        a, k, n = self.pq.L, self.pp.L, self.pq.N
        b = x.numel() // ((a + k) * n)
        out = torch.empty((b, a, n), dtype=x.dtype, device=x.device) if out is None else out
        work = torch.empty((b, a + k, n), dtype=x.dtype, device=x.device) if work is None else work
        wd_moddown(self.handle, x, out, b, work, stream)
        return out

    def close(self):
        if getattr(self, "handle", None):
            wd_rns_conv_destroy(self.handle)
            self.handle = None

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass
