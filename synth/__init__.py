"""Seeded synthetic inputs for libbulkgcd's tests and bench (input generation only).

This module is shared by the CUDA path's tests/bench and by the oracle's tests,
so it deliberately contains none of the GCD method's arithmetic (no Euclid, no
division, no gcd): it draws probable primes through OpenSSL (synth.c), multiplies
pairs of them into RSA moduli n = p*q, plants shared primes, and records the
construction ground truth.

Recipe (PAPER.md L239, L451 --
the paper's moduli come from the OpenSSL toolkit, i.e. s/2-bit primes with the
top two bits set, so every n has exactly s bits):

* config k uses seed 2015 + k;
* modulus i is P[2i] * P[2i+1], P[t] = prime #t of the seed's stream;
* a planted group G = (g0, g1, ...) replaces the first prime of every member
  after g0 with P[2*g0], so each pair inside G has gcd = P[2*g0] (the other
  primes are distinct: primes_distinct(), asserted by tests for every config);
* a duplicate (a, b) sets n_b = n_a, so gcd = n_a.

Limbs are little-endian uint32, limb 0 least significant (include/bulkgcd.h).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "synth.c")
_SO = os.path.join(_HERE, "libsynth.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile synth.c -> synth/libsynth.so (gcc + OpenSSL libcrypto)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-o", tmp, _SRC,
                               "-lcrypto", "-lpthread"])
        os.replace(tmp, _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.synth_primes.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint64,
                                     ctypes.c_size_t, ctypes.c_void_p, ctypes.c_int]
        lib.synth_primes.restype = ctypes.c_int
        lib.synth_mul.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t,
                                  ctypes.c_uint32, ctypes.c_void_p]
        lib.synth_mul.restype = ctypes.c_int
        _lib = lib
    return _lib


CACHE_DIR = os.environ.get("BULKGCD_SYNTH_CACHE", os.path.join("/tmp", "bulkgcd_synth_cache"))


def primes(pbits: int, seed: int, first: int, count: int, nthreads: int | None = None) -> np.ndarray:
    """Primes #first..#first+count-1 of stream `seed`, as uint32[count, pbits/32].

    Large requests are memoised on disk (CACHE_DIR) purely to save generation
    time; the content is a deterministic function of the arguments and is
    regenerated identically when the cache is absent.  Set
    BULKGCD_SYNTH_CACHE="" to disable."""
    path = None
    if CACHE_DIR and count >= 4096:
        path = os.path.join(CACHE_DIR, f"primes_{pbits}_{seed}_{first}_{count}.npy")
        if os.path.exists(path):
            try:
                arr = np.load(path)
                if arr.shape == (count, pbits // 32) and arr.dtype == np.uint32:
                    return arr
            except (OSError, ValueError):
                pass
    out = np.zeros((count, pbits // 32), dtype=np.uint32)
    nt = nthreads or os.cpu_count() or 1
    if _load().synth_primes(pbits, seed, first, count, out.ctypes.data, nt) != 0:
        raise RuntimeError("synth_primes failed")
    if path is not None:
        try:
            os.makedirs(CACHE_DIR, exist_ok=True)
            tmp = path + f".{os.getpid()}.npy"
            np.save(tmp, out)
            os.replace(tmp, path)
        except OSError:
            pass
    return out


def multiply(p: np.ndarray, q: np.ndarray) -> np.ndarray:
    p = np.ascontiguousarray(p, dtype=np.uint32)
    q = np.ascontiguousarray(q, dtype=np.uint32)
    assert p.shape == q.shape
    out = np.zeros((p.shape[0], 2 * p.shape[1]), dtype=np.uint32)
    _load().synth_mul(p.ctypes.data, q.ctypes.data, p.shape[0], p.shape[1], out.ctypes.data)
    return out


# ---------------------------------------------------------------- conversions
def to_int(limbs) -> int:
    """uint32 little-endian limbs -> Python int."""
    return int.from_bytes(np.asarray(limbs, dtype="<u4").tobytes(), "little")


def from_int(x: int, nlimbs: int) -> np.ndarray:
    return np.frombuffer(int(x).to_bytes(4 * nlimbs, "little"), dtype="<u4").astype(np.uint32)


def ints(arr: np.ndarray) -> list[int]:
    return [to_int(r) for r in np.asarray(arr)]


def from_ints(xs, nlimbs: int) -> np.ndarray:
    out = np.zeros((len(xs), nlimbs), dtype=np.uint32)
    for i, x in enumerate(xs):
        out[i] = from_int(x, nlimbs)
    return out


# ---------------------------------------------------------------- moduli sets
@dataclass
class ModuliSet:
    bits: int
    N: np.ndarray                     # uint32[m, bits/32]
    P: np.ndarray                     # uint32[2m, bits/64] the primes (P[2i], P[2i+1] | N[i])
    groups: list = field(default_factory=list)      # planted shared-prime groups
    duplicates: list = field(default_factory=list)  # (a, b) with N[b] == N[a]
    truth: list = field(default_factory=list)       # sorted [(i, j, g_int)] construction ground truth

    @property
    def m(self) -> int:
        return self.N.shape[0]


def moduli(m: int, bits: int, seed: int, n_planted_pairs: int = 0, cliques=(), n_duplicates: int = 0,
           nthreads: int | None = None) -> ModuliSet:
    """m synthetic `bits`-bit RSA moduli with planted shared primes.

    n_planted_pairs groups of 2 moduli, then one group per entry of `cliques`
    (its size), then n_duplicates duplicated moduli; members are drawn from a
    seeded permutation so they are spread over the index range (and over tiles).
    """
    assert bits % 64 == 0 and m >= 0
    P = primes(bits // 2, seed, 0, 2 * m, nthreads)
    p = P[0::2].copy()
    q = P[1::2].copy()
    rng = np.random.Generator(np.random.Philox(key=seed))
    perm = [int(x) for x in rng.permutation(m)]
    sizes = [2] * n_planted_pairs + list(cliques)
    need = sum(sizes) + 2 * n_duplicates
    if need > m:
        raise ValueError("not enough moduli for the requested planting")
    groups, pos = [], 0
    for s in sizes:
        g = sorted(perm[pos:pos + s])
        pos += s
        groups.append(tuple(g))
        for b in g[1:]:
            p[b] = p[g[0]]
    N = multiply(p, q)
    dups = []
    for _ in range(n_duplicates):
        a, b = sorted(perm[pos:pos + 2])
        pos += 2
        N[b] = N[a]
        dups.append((a, b))
    truth = []
    for g in groups:
        shared = to_int(p[g[0]])
        for x in range(len(g)):
            for y in range(x + 1, len(g)):
                truth.append((g[x], g[y], shared))
    for a, b in dups:
        truth.append((a, b, to_int(N[a])))
    truth.sort()
    return ModuliSet(bits, N, P, groups, dups, truth)


def primes_distinct(ms: ModuliSet) -> bool:
    """True iff every drawn prime of the set is distinct (sorting the rows of P).
    With distinct primes the planted groups and duplicates are the only pairs that
    share a factor, so ms.truth is the COMPLETE hit set."""
    P = np.ascontiguousarray(ms.P)
    return np.unique(P, axis=0).shape[0] == P.shape[0]


# BASELINE.json configs[0..4].  Seed of config k is 2015 + k.
CONFIGS = {
    1: dict(m=64, bits=1024, n_planted_pairs=3),
    3: dict(m=16384, bits=1024, n_planted_pairs=8),
    4: dict(m=16384, bits=2048, n_planted_pairs=8),
    5: dict(m=65536, bits=1024, n_planted_pairs=33),
    # the paper's other Table V widths (not BASELINE.json configs)
    6: dict(m=16384, bits=512, n_planted_pairs=8),
    7: dict(m=512, bits=4096, n_planted_pairs=4),
}
CFG2_POOL = 1449          # 1449*1448/2 = 1,049,076 >= 2^20 pairs
CFG2_PAIRS = 1 << 20


def config_moduli(k: int, nthreads: int | None = None) -> ModuliSet:
    if k == 8:
        return moduli_cofactors(seed=2015 + k, **CONFIG8)
    return moduli(seed=2015 + k, nthreads=nthreads, **CONFIGS[k])


def random_cofactors(count: int, pbits: int, seed: int) -> np.ndarray:
    """count seeded random ODD pbits-bit integers with the top two bits set (the size
    profile of OpenSSL primes, without the primality test), uint32[count, pbits/32]."""
    rng = np.random.Generator(np.random.Philox(key=seed))
    P = rng.integers(0, 1 << 32, size=(count, pbits // 32), dtype=np.uint64).astype(np.uint32)
    P[:, 0] |= 1
    P[:, -1] |= 0xC0000000
    return P


def moduli_cofactors(m: int, bits: int, seed: int, n_planted_pairs: int = 0) -> ModuliSet:
    """The paper's 4096-bit Table V workload size (all pairs of 16,384
    moduli) with fast inputs: n_i = p_i * q_i from random odd bits/2-bit cofactors (top two
    bits set) instead of primes -- 32,768 2048-bit primes take ~40 min to draw on 16 cores.
    The Euclid statistics depend only on the operand sizes (same s, same top-bit profile).
    Planted pairs (a, b) share p_a, so p_a divides gcd(n_a, n_b); a non-planted pair would
    need a common factor of >= bits/2 bits between random products (negligible).  `truth`
    lists the planted (a, b, None): the gcd value is checked by divisibility, not stored."""
    P = random_cofactors(2 * m, bits // 2, seed)
    p, q = P[0::2].copy(), P[1::2].copy()
    rng = np.random.Generator(np.random.Philox(key=seed + 1))
    perm = [int(x) for x in rng.permutation(m)]
    groups = []
    for g in range(n_planted_pairs):
        a, b = sorted(perm[2 * g:2 * g + 2])
        p[b] = p[a]
        groups.append((a, b))
    N = multiply(p, q)
    return ModuliSet(bits, N, np.stack([p, q], axis=1).reshape(2 * m, -1), groups, [],
                     sorted((a, b, None) for a, b in groups))


# cfg8: 16,384 x 4096-bit moduli, all 134,209,536 pairs (the paper's Table V 4096-bit size; N1)
CONFIG8 = dict(m=16384, bits=4096, n_planted_pairs=8)


def pair_indices(n: int, count: int) -> tuple[np.ndarray, np.ndarray]:
    """The first `count` pairs (i < j) of n items in row-major order."""
    ii, jj = np.triu_indices(n, k=1)
    assert count <= ii.size
    return ii[:count].astype(np.int64), jj[:count].astype(np.int64)


def config2(count: int = CFG2_PAIRS, nthreads: int | None = None):
    """cfg2: `count` independent 1024-bit pairs = the first pairs (i<j) of a seeded pool."""
    ms = moduli(CFG2_POOL, 1024, 2015 + 2, n_planted_pairs=2, nthreads=nthreads)
    i, j = pair_indices(CFG2_POOL, count)
    return ms.N[i], ms.N[j], ms


# ----------------------------------------------------- rare-path test inputs
def _rand_int(rng: np.random.Generator, nbits: int) -> int:
    if nbits <= 0:
        return 0
    nw = (nbits + 31) // 32
    words = rng.integers(0, 1 << 32, size=nw, dtype=np.uint64)
    x = to_int(words.astype(np.uint32))
    return x & ((1 << nbits) - 1)


def mixed_pairs(count: int, bits: int, seed: int) -> tuple[list[int], list[int]]:
    """Seeded exact-mode operands (bulkgcd_pairs) covering every rare path.

    Categories cycle over: random full-size; random with random bit lengths
    (unequal lengths -> beta>0 updates, Cases 1-3); even values and zeros;
    X = a*Y + odd*2^k with k >= 32 (rshift by >= one word); one-word Y (Case 2);
    two-word Y (Case 3); near-equal X ~ Y (Case 4-C); duplicates; small common
    factors (3^a 5^b 2^c ...); a shared large factor.
    """
    rng = np.random.Generator(np.random.Philox(key=seed))
    A, B = [], []
    top = (1 << bits) - 1
    for t in range(count):
        c = t % 11
        if c == 0:
            a, b = _rand_int(rng, bits), _rand_int(rng, bits)
        elif c == 1:
            a = _rand_int(rng, int(rng.integers(1, bits + 1)))
            b = _rand_int(rng, int(rng.integers(1, bits + 1)))
        elif c == 2:
            kind = int(rng.integers(0, 5))
            a = _rand_int(rng, bits) << int(rng.integers(0, 70))
            b = _rand_int(rng, bits) << int(rng.integers(0, 70))
            if kind == 0:
                a = 0
            elif kind == 1:
                b = 0
            elif kind == 2:
                a = b = 0
        elif c == 3:
            y = _rand_int(rng, bits // 2) | 1
            k = int(rng.integers(32, 100))
            odd = _rand_int(rng, int(rng.integers(1, 64))) | 1
            alpha = _rand_int(rng, int(rng.integers(1, 40)))
            a, b = alpha * y + (odd << k), y
        elif c == 4:
            a, b = _rand_int(rng, bits), _rand_int(rng, int(rng.integers(1, 33)))
        elif c == 5:
            a, b = _rand_int(rng, bits), _rand_int(rng, int(rng.integers(33, 65)))
        elif c == 6:
            x = _rand_int(rng, bits) | (1 << (bits - 1))
            a, b = x, x - 2 * int(rng.integers(1, 1000))
        elif c == 7:
            a = _rand_int(rng, bits)
            b = a
        elif c == 8:
            f = (3 ** int(rng.integers(0, 20))) * (5 ** int(rng.integers(0, 10))) << int(rng.integers(0, 8))
            a = (f * _rand_int(rng, bits // 2)) & top
            b = (f * _rand_int(rng, bits // 2)) & top
        elif c == 9:
            g = _rand_int(rng, bits // 2) | 1
            a = g * _rand_int(rng, bits // 2 - 1)
            b = g * _rand_int(rng, bits // 2 - 1)
        else:
            a, b = 1, _rand_int(rng, bits)
        A.append(a & top)
        B.append(b & top)
    return A, B
