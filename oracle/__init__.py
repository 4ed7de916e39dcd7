"""CPU oracle for libbulkgcd -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(paper_conf_ipps_fujitani15_b200, include/bulkgcd.h) never imports it and the
two share no code; only the seeded input generators in ``synth`` serve both.

* :mod:`oracle.gcd_oracle` (C, ``gcd_oracle.c``): the definition -- the
  Original Euclidean algorithm (§II) over schoolbook bignums with
  Knuth Algorithm D division (paper ref. [15]).  Exact gcd of any operands.
* :mod:`oracle.approx_model` (Python ints): the paper's Approximate Euclidean
  algorithm step by step (L107, L127, L255), d-generic, with counters; used to
  pin the worked examples (Table III, the approx examples) and Table IV, and
  for per-pair iteration-count parity with the GPU.
* :mod:`oracle.approx_euclid` (C, ``approx_euclid.c``): the same paper algorithm
  as approx_model, d = 32, in plain C on word arrays -- the CPU (E) column of
  Table V for bench.py's cpu_baseline; pinned per pair against
  approx_model (tests/test_model.py).
* :func:`rsa_hit` -- the RSA-mode result mapping.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from . import approx_model  # noqa: F401  (re-exported)

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gcd_oracle.c")
_SRC2 = os.path.join(_HERE, "approx_euclid.c")
_SO = os.path.join(_HERE, "libgcd_oracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the C oracle and the C (E) baseline (gcc -O2) -> oracle/libgcd_oracle.so."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(os.path.getmtime(_SRC),
                                                                       os.path.getmtime(_SRC2)):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-o", tmp, _SRC, _SRC2, "-lpthread"])
        os.replace(tmp, _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        vp, u32, sz = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_size_t
        lib.oracle_gcd.argtypes = [vp, vp, u32, vp]
        lib.oracle_gcd.restype = ctypes.c_long
        lib.oracle_gcd_trace.argtypes = [vp, vp, u32, vp, vp, ctypes.c_long]
        lib.oracle_gcd_trace.restype = ctypes.c_long
        lib.oracle_divmod.argtypes = [vp, vp, u32, vp, vp]
        lib.oracle_divmod.restype = ctypes.c_int
        lib.oracle_gcd_batch.argtypes = [vp, vp, sz, u32, vp, ctypes.c_int]
        lib.oracle_gcd_batch.restype = ctypes.c_int
        lib.oracle_gcd_index_pairs.argtypes = [vp, vp, vp, sz, u32, vp, ctypes.c_int]
        lib.oracle_gcd_index_pairs.restype = ctypes.c_int
        lib.oracle_approx_gcd.argtypes = [vp, vp, u32, ctypes.c_int, vp, vp]
        lib.oracle_approx_gcd.restype = ctypes.c_long
        lib.oracle_approx_index_pairs.argtypes = [vp, vp, vp, sz, u32, ctypes.c_int, vp, vp, vp, ctypes.c_int]
        lib.oracle_approx_index_pairs.restype = ctypes.c_int
        _lib = lib
    return _lib


def _limbs(x: int, n: int) -> np.ndarray:
    return np.frombuffer(int(x).to_bytes(4 * n, "little"), dtype="<u4").astype(np.uint32)


def _int(a: np.ndarray) -> int:
    return int.from_bytes(np.ascontiguousarray(a, dtype="<u4").tobytes(), "little")


def _nlimbs(*xs: int) -> int:
    return max(1, max((x.bit_length() + 31) // 32 for x in xs))


def gcd(a: int, b: int) -> int:
    """Exact gcd of two non-negative Python ints through the C oracle."""
    n = _nlimbs(a, b)
    A, B, G = _limbs(a, n), _limbs(b, n), np.zeros(n, np.uint32)
    if _load().oracle_gcd(A.ctypes.data, B.ctypes.data, n, G.ctypes.data) < 0:
        raise ValueError("operand too large for the oracle")
    return _int(G)


def gcd_trace(a: int, b: int, qmax: int = 4096) -> tuple[int, int, list[int]]:
    """(gcd, iterations, quotients) of the Original Euclidean algorithm (L55)."""
    n = _nlimbs(a, b)
    A, B, G = _limbs(a, n), _limbs(b, n), np.zeros(n, np.uint32)
    Q = np.zeros(qmax, np.uint64)
    it = _load().oracle_gcd_trace(A.ctypes.data, B.ctypes.data, n, G.ctypes.data, Q.ctypes.data, qmax)
    if it < 0:
        raise ValueError("operand too large for the oracle")
    return _int(G), int(it), [int(q) for q in Q[:min(it, qmax)]]


def divmod_(x: int, y: int) -> tuple[int, int]:
    """(x div y, x mod y) via Knuth Algorithm D (the oracle's division)."""
    n = _nlimbs(x, y)
    X, Y = _limbs(x, n), _limbs(y, n)
    Q, R = np.zeros(n, np.uint32), np.zeros(n, np.uint32)
    if _load().oracle_divmod(X.ctypes.data, Y.ctypes.data, n, Q.ctypes.data, R.ctypes.data) != 0:
        raise ZeroDivisionError
    return _int(Q), _int(R)


def gcd_batch(A: np.ndarray, B: np.ndarray, nthreads: int | None = None) -> np.ndarray:
    """G[k] = gcd(A[k], B[k]) for uint32[m, W] row-major limb arrays."""
    A = np.ascontiguousarray(A, dtype=np.uint32)
    B = np.ascontiguousarray(B, dtype=np.uint32)
    assert A.shape == B.shape and A.ndim == 2
    G = np.zeros_like(A)
    nt = nthreads or os.cpu_count() or 1
    if A.shape[0] and _load().oracle_gcd_batch(A.ctypes.data, B.ctypes.data, A.shape[0], A.shape[1],
                                               G.ctypes.data, nt) != 0:
        raise RuntimeError("oracle_gcd_batch failed")
    return G


def gcd_index_pairs(N: np.ndarray, ii, jj, nthreads: int | None = None) -> np.ndarray:
    """G[k] = gcd(N[ii[k]], N[jj[k]])."""
    N = np.ascontiguousarray(N, dtype=np.uint32)
    ii = np.ascontiguousarray(ii, dtype=np.uint64)
    jj = np.ascontiguousarray(jj, dtype=np.uint64)
    G = np.zeros((ii.size, N.shape[1]), np.uint32)
    nt = nthreads or os.cpu_count() or 1
    if ii.size and _load().oracle_gcd_index_pairs(N.ctypes.data, ii.ctypes.data, jj.ctypes.data, ii.size,
                                                  N.shape[1], G.ctypes.data, nt) != 0:
        raise RuntimeError("oracle_gcd_index_pairs failed")
    return G


def approx_gcd(a: int, b: int, bits: int, early: bool) -> tuple[int, int]:
    """(result, iterations) of the C Approximate Euclid (approx_euclid.c) on one pair of
    `bits`-bit operands: early=True is RSA mode on odd inputs (g or 1), early=False the
    exact gcd of any inputs (L41)."""
    n = bits // 32
    A, B, G = _limbs(a, n), _limbs(b, n), np.zeros(n, np.uint32)
    it = _load().oracle_approx_gcd(A.ctypes.data, B.ctypes.data, n, bits if early else 0, G.ctypes.data, None)
    if it < 0:
        raise ValueError("operand too large")
    return _int(G), int(it)


def approx_index_pairs(N: np.ndarray, ii, jj, bits: int, early: bool = True, nthreads: int = 1):
    """The C (E) baseline over index pairs: (G uint32[k, W], iterations uint32[k],
    [sum iterations, sum limb-steps, beta>0 iterations])."""
    N = np.ascontiguousarray(N, dtype=np.uint32)
    ii = np.ascontiguousarray(ii, dtype=np.uint64)
    jj = np.ascontiguousarray(jj, dtype=np.uint64)
    G = np.zeros((ii.size, N.shape[1]), np.uint32)
    it = np.zeros(ii.size, np.uint32)
    ctr = np.zeros(3, np.uint64)
    if ii.size and _load().oracle_approx_index_pairs(N.ctypes.data, ii.ctypes.data, jj.ctypes.data, ii.size,
                                                     N.shape[1], bits if early else 0, G.ctypes.data, it.ctypes.data,
                                                     ctr.ctypes.data, nthreads) != 0:
        raise RuntimeError("oracle_approx_index_pairs failed")
    return G, it, [int(x) for x in ctr]


def bitlen_rows(G: np.ndarray) -> np.ndarray:
    """Bit length of each row of a uint32[m, W] limb array."""
    G = np.asarray(G, dtype=np.uint32)
    nz = G != 0
    top = np.where(nz.any(axis=1), G.shape[1] - 1 - np.argmax(nz[:, ::-1], axis=1), -1)
    word = G[np.arange(G.shape[0]), np.maximum(top, 0)].astype(np.uint64)
    wbits = np.zeros(G.shape[0], np.int64)
    w = word.copy()
    while np.any(w):
        wbits += (w != 0)
        w >>= np.uint64(1)
    return np.where(top >= 0, top * 32 + wbits, 0)


def rsa_hit(g_bitlen, bits: int):
    """RSA-mode mapping: the early-terminated
    algorithm reports g iff g has at least s/2 bits, otherwise "coprime" (1)."""
    return np.asarray(g_bitlen) >= bits // 2


def all_pairs_hits(N: np.ndarray, bits: int, ii=None, jj=None, nthreads: int | None = None):
    """RSA-mode hit set over the given (i<j) pairs (default: every pair).

    Returns a sorted list of (i, j, g_int) with bitlen(g) >= bits/2.
    """
    n = N.shape[0]
    if ii is None:
        ii, jj = np.triu_indices(n, k=1)
    G = gcd_index_pairs(N, ii, jj, nthreads)
    hit = rsa_hit(bitlen_rows(G), bits)
    out = [(int(ii[k]), int(jj[k]), _int(G[k])) for k in np.nonzero(hit)[0]]
    out.sort()
    return out


def cofactors(N: np.ndarray, hits) -> list[tuple[int, int]]:
    """Factor output (n1 = p * (n1 / p)): for each hit (i, j, g),
    (N[i] div g, N[j] div g) by the oracle's Knuth-D division; raises if g does
    not divide a modulus (remainder != 0)."""
    out = []
    for i, j, g in hits:
        qi, ri = divmod_(_int(np.asarray(N[i])), g)
        qj, rj = divmod_(_int(np.asarray(N[j])), g)
        if ri or rj:
            raise ValueError(f"gcd does not divide N[{i}] or N[{j}]")
        out.append((qi, qj))
    return out
