"""Python binding of libbulkgcd (include/bulkgcd.h) -- argument marshalling only.

Every step of the GCD path runs in the CUDA kernels of libbulkgcd.so (sm_100a);
this module only converts numpy arrays / torch tensors to pointers and sizes.
There is no CPU fallback: if the shared library is missing, importing the
binding's functions raises.

Names follow the C ABI: bulkgcd_pairs, bulkgcd_pairs_ex, bulkgcd_all_pairs,
bulkgcd_interleave, bulkgcd_layout_blocked, bulkgcd_cohort_count,
bulkgcd_blocked_words, bulkgcd_pairs_device, bulkgcd_all_pairs_band,
bulkgcd_cofactors, bulkgcd_cofactors_device.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

from ._build import SO, build  # noqa: F401

MODE_EXACT = 0
MODE_RSA = 1
FLAG_STATS = 1
FLAG_SMEM = 2
FLAG_ALGO_FAST_BINARY = 1 << 8
FLAG_ALGO_BINARY = 2 << 8

EINVAL, ENOMEM, ECUDA, ENODEV = -1, -2, -3, -4

_lib = None

SYMBOLS = (
    "bulkgcd_pairs", "bulkgcd_pairs_ex", "bulkgcd_all_pairs", "bulkgcd_hits_free", "bulkgcd_strerror",
    "bulkgcd_last_error", "bulkgcd_device_check", "bulkgcd_interleave", "bulkgcd_layout_blocked",
    "bulkgcd_blocked_words", "bulkgcd_cohort_count", "bulkgcd_pairs_device", "bulkgcd_all_pairs_band",
    "bulkgcd_cofactors", "bulkgcd_cofactors_device",
)


def check_moduli(N: np.ndarray, bits: int) -> None:
    """The host API's RSA-mode input rule (include/bulkgcd.h B2; PAPER.md L41 assumes odd
    inputs): every modulus odd and > 1, shape [n, bits/32].  bulkgcd_all_pairs_band
    does not check it on the device, so the band drivers (dist.py, resume.py) do:
    a zero modulus would be reported against every other one, an even one would lose
    its factors of 2."""
    W = bits // 32
    if N.ndim != 2 or N.shape[1] != W:
        raise ValueError(f"moduli must be uint32[n, {W}] for {bits} bits, got shape {N.shape}")
    if N.shape[0] == 0:
        return
    odd = (N[:, 0] & 1) == 1
    gt1 = (N[:, 0] > 1) | np.any(N[:, 1:] != 0, axis=1)
    bad = np.nonzero(~(odd & gt1))[0]
    if bad.size:
        raise ValueError(f"modulus {int(bad[0])} is even or <= 1 (RSA mode needs odd moduli > 1)")


class BulkGcdError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"libbulkgcd error {code}: {msg}")
        self.code = code


class _Hits(ctypes.Structure):
    _fields_ = [("count", ctypes.c_size_t), ("ij", ctypes.POINTER(ctypes.c_uint32)),
                ("gcd", ctypes.POINTER(ctypes.c_uint32)), ("bits", ctypes.c_uint32)]


def lib() -> ctypes.CDLL:
    """Load libbulkgcd.so (in-tree).  Raises if it has not been built."""
    global _lib
    if _lib is None:
        path = os.environ.get("BULKGCD_SO", SO)  # alternative builds of the same sources (tuning runs)
        if not os.path.exists(path):
            raise ImportError(f"libbulkgcd.so not built ({path}); run __graft_entry__.build() -- there is no fallback")
        L = ctypes.CDLL(path)
        vp, sz, u32, u64, i32 = ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
        sig = {
            "bulkgcd_pairs": ([vp, vp, sz, u32, vp], i32),
            "bulkgcd_pairs_ex": ([vp, vp, sz, u32, i32, vp, vp], i32),
            "bulkgcd_all_pairs": ([vp, sz, u32, ctypes.POINTER(_Hits)], i32),
            "bulkgcd_hits_free": ([ctypes.POINTER(_Hits)], None),
            "bulkgcd_strerror": ([i32], ctypes.c_char_p),
            "bulkgcd_last_error": ([], ctypes.c_char_p),
            "bulkgcd_device_check": ([], i32),
            "bulkgcd_interleave": ([vp, vp, sz, sz, u32, i32, vp], i32),
            "bulkgcd_layout_blocked": ([vp, vp, sz, u32, vp], i32),
            "bulkgcd_blocked_words": ([sz, u32], sz),
            "bulkgcd_cohort_count": ([sz], u64),
            "bulkgcd_pairs_device": ([vp, vp, vp, sz, sz, u32, i32, vp, vp, ctypes.c_uint, vp], i32),
            "bulkgcd_all_pairs_band": ([vp, vp, sz, u32, u64, u64, vp, u64, vp, ctypes.c_uint, vp], i32),
            "bulkgcd_cofactors": ([vp, sz, u32, ctypes.POINTER(_Hits), vp], i32),
            "bulkgcd_cofactors_device": ([vp, sz, u32, vp, u64, vp, vp, vp], i32),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


def _check(rc: int) -> None:
    if rc != 0:
        L = lib()
        raise BulkGcdError(rc, f"{L.bulkgcd_strerror(rc).decode()}: {L.bulkgcd_last_error().decode()}")


def _words(bits: int) -> int:
    return bits // 32


def _host(a, W: int) -> np.ndarray:
    a = np.ascontiguousarray(a, dtype=np.uint32)
    if a.ndim != 2 or a.shape[1] != W:
        raise ValueError(f"expected uint32[m, {W}] row-major limbs, got {a.shape}")
    return a


def _ptr(x) -> int | None:
    """Device pointer of a torch tensor (or an int / None)."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    return x.data_ptr()


def _stream(stream) -> int | None:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


# ------------------------------------------------------------- host entry points
def bulkgcd_pairs(A, B, bits: int, out: np.ndarray | None = None) -> np.ndarray:
    """G[i] = gcd(A[i], B[i]) (exact mode).  A, B: uint32[m, bits/32].  `out`: an
    optional caller-owned result array of the same shape (e.g. pinned host memory)."""
    G, _ = bulkgcd_pairs_ex(A, B, bits, MODE_EXACT, want_iters=False, out=out)
    return G


def bulkgcd_pairs_ex(A, B, bits: int, mode: int = MODE_EXACT, want_iters: bool = False,
                     out: np.ndarray | None = None):
    W = _words(bits)
    A, B = _host(A, W), _host(B, W)
    if A.shape != B.shape:
        raise ValueError("A and B must have the same shape")
    m = A.shape[0]
    if out is None:
        G = np.zeros_like(A)
    else:
        G = out
        if G.dtype != np.uint32 or G.shape != A.shape or not G.flags.c_contiguous:
            raise ValueError(f"out must be a C-contiguous uint32{list(A.shape)} array")
    it = np.zeros(m, np.uint32) if want_iters else None
    _check(lib().bulkgcd_pairs_ex(A.ctypes.data, B.ctypes.data, m, bits, mode, G.ctypes.data,
                                  it.ctypes.data if it is not None else None))
    return G, it


@dataclass
class Hits:
    ij: np.ndarray   # uint32[count, 2], sorted by (i, j)
    gcd: np.ndarray  # uint32[count, W]
    bits: int

    def as_list(self):
        return [(int(i), int(j), int.from_bytes(g.astype("<u4").tobytes(), "little"))
                for (i, j), g in zip(self.ij, self.gcd)]


def bulkgcd_all_pairs(N, bits: int) -> Hits:
    """All-pairs RSA-mode search: every (i < j) with bitlen(gcd) >= bits/2."""
    W = _words(bits)
    N = _host(N, W)
    h = _Hits()
    L = lib()
    _check(L.bulkgcd_all_pairs(N.ctypes.data, N.shape[0], bits, ctypes.byref(h)))
    try:
        c = h.count
        ij = np.ctypeslib.as_array(h.ij, shape=(c * 2,)).reshape(c, 2).copy() if c else np.zeros((0, 2), np.uint32)
        g = np.ctypeslib.as_array(h.gcd, shape=(c * W,)).reshape(c, W).copy() if c else np.zeros((0, W), np.uint32)
    finally:
        L.bulkgcd_hits_free(ctypes.byref(h))
    return Hits(ij, g, bits)


def bulkgcd_cofactors(N, bits: int, hits: Hits) -> np.ndarray:
    """Factor output: F[h, 0] = N[i] / g, F[h, 1] = N[j] / g for
    every hit (i, j, g), as uint32[count, 2, W] (exact division on the GPU)."""
    W = _words(bits)
    N = _host(N, W)
    c = len(hits.ij)
    ij = np.ascontiguousarray(hits.ij, dtype=np.uint32).reshape(c, 2)
    g = np.ascontiguousarray(hits.gcd, dtype=np.uint32).reshape(c, W)
    h = _Hits(c, ij.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)) if c else None,
              g.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)) if c else None, hits.bits)
    F = np.zeros((c, 2, W), np.uint32)
    _check(lib().bulkgcd_cofactors(N.ctypes.data, N.shape[0], bits, ctypes.byref(h), F.ctypes.data))
    return F


def bulkgcd_device_check() -> None:
    _check(lib().bulkgcd_device_check())


# ----------------------------------------------------------- device entry points
def bulkgcd_interleave(d_in, d_out, m: int, m_pad: int, bits: int, to_interleaved: bool, stream=None) -> None:
    _check(lib().bulkgcd_interleave(_ptr(d_in), _ptr(d_out), m, m_pad, bits, int(bool(to_interleaved)),
                                    _stream(stream)))


def bulkgcd_layout_blocked(d_N, d_N_blk, n: int, bits: int, stream=None) -> None:
    _check(lib().bulkgcd_layout_blocked(_ptr(d_N), _ptr(d_N_blk), n, bits, _stream(stream)))


def bulkgcd_blocked_words(n: int, bits: int) -> int:
    return int(lib().bulkgcd_blocked_words(n, bits))


def bulkgcd_cohort_count(n: int) -> int:
    return int(lib().bulkgcd_cohort_count(n))


def bulkgcd_pairs_device(d_A, d_B, d_G, m: int, m_pad: int, bits: int, mode: int, d_iters, d_scratch,
                         flags: int = 0, stream=None) -> None:
    _check(lib().bulkgcd_pairs_device(_ptr(d_A), _ptr(d_B), _ptr(d_G), m, m_pad, bits, mode, _ptr(d_iters),
                                      _ptr(d_scratch), flags, _stream(stream)))


def bulkgcd_all_pairs_band(d_N, d_N_blk, n: int, bits: int, cohort_begin: int, cohort_end: int, d_hits,
                           hit_cap: int, d_counters, flags: int = 0, stream=None) -> None:
    _check(lib().bulkgcd_all_pairs_band(_ptr(d_N), _ptr(d_N_blk), n, bits, cohort_begin, cohort_end,
                                        _ptr(d_hits), hit_cap, _ptr(d_counters), flags, _stream(stream)))


def bulkgcd_cofactors_device(d_N, n: int, bits: int, d_hits, count: int, d_F, d_bad, stream=None) -> None:
    _check(lib().bulkgcd_cofactors_device(_ptr(d_N), n, bits, _ptr(d_hits), count, _ptr(d_F), _ptr(d_bad),
                                          _stream(stream)))
