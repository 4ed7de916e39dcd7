"""Pins for the C oracle (oracle/gcd_oracle.c): the Original Euclidean algorithm
over schoolbook bignums (Knuth Algorithm D, ref. [15]).

Every check compares against something other than the oracle itself:
brute-force trial division, Python's math.gcd / divmod (library routines),
number-theoretic invariants, the paper's Table II, and construction ground truth.
"""
import math

import numpy as np
import pytest

import oracle
import synth
from conftest import read_golden


def _brute_gcd_grid(a, b):
    """Largest d dividing both, by trial division over every candidate d."""
    a = np.asarray(a, dtype=np.int64)
    b = np.asarray(b, dtype=np.int64)
    g = np.zeros_like(a)
    top = int(max(a.max(), b.max()))
    for d in range(1, top + 1):
        both = (a % d == 0) & (b % d == 0)
        g = np.where(both, d, g)
    # gcd(x, 0) = x, gcd(0, 0) = 0: every d divides 0, so the largest "divisor" of 0 is unbounded;
    # by definition gcd(x, 0) = x.
    g = np.where(a == 0, b, np.where(b == 0, a, g))
    return g


def test_brute_force_tiny_exhaustive():
    vals = np.arange(0, 130)
    a, b = np.meshgrid(vals, vals)
    a, b = a.ravel(), b.ravel()
    A = a.astype(np.uint32).reshape(-1, 1)
    B = b.astype(np.uint32).reshape(-1, 1)
    G = oracle.gcd_batch(A, B)[:, 0]
    assert np.array_equal(G.astype(np.int64), _brute_gcd_grid(a, b))


def test_brute_force_odd_14bit_sample():
    rng = np.random.default_rng(1)
    a = rng.integers(1, 1 << 14, size=3000) | 1
    b = rng.integers(1, 1 << 14, size=3000) | 1
    G = oracle.gcd_batch(a.astype(np.uint32).reshape(-1, 1), b.astype(np.uint32).reshape(-1, 1))[:, 0]
    assert np.array_equal(G.astype(np.int64), _brute_gcd_grid(a, b))


def test_lcm_identity_brute_force():
    """g * lcm(a, b) = a * b with lcm found by brute force (smallest common multiple)."""
    rng = np.random.default_rng(2)
    for _ in range(300):
        a, b = int(rng.integers(1, 400)), int(rng.integers(1, 400))
        lcm = next(k for k in range(a, a * b + 1, a) if k % b == 0)
        assert oracle.gcd(a, b) * lcm == a * b


@pytest.mark.parametrize("bits", [32, 64, 96, 512, 1024, 2048, 4096])
def test_against_math_gcd(bits):
    """math.gcd (CPython's Lehmer gcd) is a library routine the definition reduces to."""
    A, B = synth.mixed_pairs(330, bits, seed=bits)
    W = max(1, bits // 32)
    G = oracle.gcd_batch(synth.from_ints(A, W), synth.from_ints(B, W))
    for k, (a, b) in enumerate(zip(A, B)):
        assert synth.to_int(G[k]) == math.gcd(a, b), (k, a, b)


def test_invariants_random():
    rng = np.random.default_rng(3)
    for _ in range(200):
        nb = int(rng.integers(8, 700))
        g0 = int.from_bytes(rng.bytes(16), "little") | 1
        a = g0 * int.from_bytes(rng.bytes(nb // 8 + 1), "little")
        b = g0 * int.from_bytes(rng.bytes(nb // 8 + 1), "little")
        g = oracle.gcd(a, b)
        if a == 0 or b == 0:
            assert g == a | b
            continue
        assert a % g == 0 and b % g == 0
        assert oracle.gcd(a // g, b // g) == 1
        assert g % g0 == 0
        assert oracle.gcd(a, b) == oracle.gcd(b, a)
        assert oracle.gcd(a, a) == a and oracle.gcd(a, 0) == a and oracle.gcd(0, a) == a
    assert oracle.gcd(0, 0) == 0


def test_table2_original_euclid():
    rows = {r[0]: r[1:] for r in read_golden("table2_original_euclid.txt")}
    g, it, qs = oracle.gcd_trace(int(rows["X"][0]), int(rows["Y"][0]))
    assert g == int(rows["gcd"][0])
    assert it == int(rows["original_iterations"][0])
    assert qs == [int(q) for q in rows["original_quotients"]]


def test_knuth_d_divmod():
    """Algorithm D against Python's divmod, including the rare add-back step (D6)
    and the qhat-refinement loop (D3), which structured divisors provoke."""
    rng = np.random.default_rng(4)
    cases = []
    for _ in range(400):
        nx, ny = int(rng.integers(1, 40)), int(rng.integers(1, 20))
        cases.append((int.from_bytes(rng.bytes(4 * nx), "little"), int.from_bytes(rng.bytes(4 * ny), "little") | 1))
    B = 1 << 32
    # D6 add-back / D3 refinement provocations (Knuth 4.3.1 exercises; Hacker's Delight divmnu tests)
    cases += [
        (0x7FFF800000000000 * B**2, 0x800000000001 * B),
        (0x8000000000000000 * B**2 + 3, 0x800000000001 * B + 0xFFFFFFFF),
        ((B**3 - 1) * B, (B**2 - 1) * B + 1),
        (B**4 - 1, B**2 - 1),
        (0x0000800000000000 * B**2 + 0xFFFE, 0x8000FFFF * B + 0xFFFF),
        ((1 << 200) - 1, (1 << 100) + 1),
    ]
    for _ in range(300):  # near-multiples with near-max top limbs
        ny = int(rng.integers(2, 9))
        y = (B - 1 - int(rng.integers(0, 3))) * B ** (ny - 1) + int.from_bytes(rng.bytes(4 * (ny - 1)), "little")
        q = int.from_bytes(rng.bytes(4 * int(rng.integers(1, 4))), "little")
        cases.append((y * q + int(rng.integers(0, 2)) * (y - 1), y))
    for x, y in cases:
        if y == 0:
            continue
        assert oracle.divmod_(x, y) == divmod(x, y), (x, y)


def test_planted_primes_recovered(cfg1):
    """Construction ground truth: cfg1 (3 planted shared primes) over all 2016 pairs."""
    hits = oracle.all_pairs_hits(cfg1.N, cfg1.bits)
    assert hits == cfg1.truth
    assert len(hits) == 3


def test_rsa_mode_mapping():
    """O3: RSA-mode output is g iff bitlen(g) >= bits/2."""
    G = synth.from_ints([0, 1, (1 << 511) - 1, 1 << 511, (1 << 1024) - 1], 32)
    assert list(oracle.rsa_hit(oracle.bitlen_rows(G), 1024)) == [False, False, False, True, True]
    assert list(oracle.bitlen_rows(G)) == [0, 1, 511, 512, 1024]


def test_cofactors_construction_truth():
    """N3 factor output (n1 = p * (n1/p)): for every planted hit the
    oracle's cofactors are the construction's other primes; duplicates give (1, 1)."""
    ms = synth.moduli(40, 1024, seed=77, n_planted_pairs=2, cliques=(3,), n_duplicates=1)
    got = oracle.cofactors(ms.N, ms.truth)
    dup = set(ms.duplicates)
    for (i, j, g), (ci, cj) in zip(ms.truth, got):
        if (i, j) in dup:
            assert (ci, cj) == (1, 1) and g == synth.to_int(ms.N[i])
        else:
            assert ci == synth.to_int(ms.P[2 * i + 1]) and cj == synth.to_int(ms.P[2 * j + 1])
            assert g * ci == synth.to_int(ms.N[i]) and g * cj == synth.to_int(ms.N[j])
    with pytest.raises(ValueError):
        oracle.cofactors(ms.N, [(0, 1, 3)])
