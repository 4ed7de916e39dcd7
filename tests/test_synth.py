"""The seeded input generator: determinism, exact sizes, distinct primes, planting."""
import math

import numpy as np

import synth


def test_deterministic_and_sized():
    a = synth.moduli(40, 1024, seed=11, n_planted_pairs=2, cliques=(3,), n_duplicates=1)
    b = synth.moduli(40, 1024, seed=11, n_planted_pairs=2, cliques=(3,), n_duplicates=1)
    assert np.array_equal(a.N, b.N)
    for n in synth.ints(a.N):
        assert n.bit_length() == 1024 and n & 1
    for p in synth.ints(a.P):
        assert p.bit_length() == 512 and (p >> 510) == 3


def test_primes_distinct_and_probable_primes():
    P = synth.ints(synth.primes(256, 99, 0, 200))
    assert len(set(P)) == len(P)
    for p in P[:50]:  # Fermat + small-prime trial division as an independent sanity check
        assert pow(2, p - 1, p) == 1 and pow(3, p - 1, p) == 1
        assert all(p % s for s in (3, 5, 7, 11, 13, 17, 19, 23, 29, 31))


def test_truth_matches_gcds():
    ms = synth.moduli(40, 1024, seed=12, n_planted_pairs=2, cliques=(3,), n_duplicates=1)
    N = synth.ints(ms.N)
    found = []
    for i in range(len(N)):
        for j in range(i + 1, len(N)):
            g = math.gcd(N[i], N[j])
            if g.bit_length() >= 512:
                found.append((i, j, g))
    assert found == ms.truth
    assert len(ms.truth) == 2 + 3 + 1


def test_config1_shape(cfg1):
    assert cfg1.N.shape == (64, 32)
    assert len(cfg1.truth) == 3
    assert len(set(synth.ints(cfg1.P))) == 128  # all drawn primes distinct (planting reuses 3 of them)


def test_config2_pairs():
    i, j = synth.pair_indices(synth.CFG2_POOL, synth.CFG2_PAIRS)
    assert i.size == 1 << 20 and np.all(i < j)
    assert (int(i[0]), int(j[0])) == (0, 1)


def test_config_primes_distinct_small():
    """Every drawn prime of configs[0] and of the cfg2 pool is distinct, so their
    construction truth is complete; cfg3/4/5 are asserted
    by the GPU full-size tests, which generate those sets anyway."""
    assert synth.primes_distinct(synth.config_moduli(1))
    _, _, pool = synth.config2(16)
    assert pool.P.shape == (2 * synth.CFG2_POOL, 16) and synth.primes_distinct(pool)
    bad = synth.ModuliSet(1024, pool.N[:2], np.concatenate([pool.P[:3], pool.P[:1]]))
    assert not synth.primes_distinct(bad)
