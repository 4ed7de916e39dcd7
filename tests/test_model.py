"""Pins for the CPU model of the paper's Approximate Euclidean algorithm
(oracle/approx_model.py): the worked examples (Table III, the approx()
examples, Table II's Fast Euclid column), Table IV's mean iteration counts, the
quotient bound alpha*D^beta <= X div Y (L123), and agreement with math.gcd."""
import math

import numpy as np
import pytest

import oracle
import synth
from conftest import read_golden
from oracle import approx_model as am


def test_approx_examples():
    for X, Y, a, b, case, _cite in read_golden("approx_examples.txt"):
        assert am.approx(int(X), int(Y), 4) == (int(a), int(b), case)


def test_table3_trace():
    rows = read_golden("table3_approx_euclid.txt")
    head = {r[0]: r[1] for r in rows[:4]}
    t = am.approximate_euclid(int(head["X"], 16), int(head["Y"], 16), d=int(head["d"]), record=True, check=True)
    steps = rows[4:]
    assert t.iterations == len(steps) == 9
    assert t.gcd == int(head["gcd"])
    for got, (_n, case, a, b, x, y) in zip(t.steps, steps):
        assert got == (case, int(a), int(b), int(x, 16), int(y, 16))
    assert t.bound_violations == 0


def test_table2_fast_euclid():
    rows = {r[0]: r[1:] for r in read_golden("table2_original_euclid.txt")}
    g, it, qs = am.fast_euclid(int(rows["X"][0]), int(rows["Y"][0]))
    assert g == int(rows["gcd"][0])
    assert it == int(rows["fast_iterations"][0])
    assert qs == [int(q) for q in rows["fast_quotients"]]


def test_fast_binary_special_case():
    """L111: with (alpha, beta) = (1, 0) always, the algorithm is Fast Binary Euclid;
    Table I (L47) says Fast Binary takes 16 iterations on the Table I inputs."""
    X, Y = 1043915, 768955
    it = 0
    while Y:
        X = am.rshift(X - Y)
        if X < Y:
            X, Y = Y, X
        it += 1
    assert (X, it) == (5, 16)


@pytest.mark.parametrize("bits", [64, 96, 128, 256, 1024])
def test_exact_mode_matches_math_gcd(bits):
    A, B = synth.mixed_pairs(440, bits, seed=100 + bits)
    for a, b in zip(A, B):
        t = am.gcd_exact(a, b)
        assert t.gcd == math.gcd(a, b), (a, b)


def test_bound_and_iteration_invariants():
    """alpha*D^beta <= X div Y (L123), alpha < D outside Case 1 (L133, O4.14),
    <= 2s iterations (L49, L61) on every rare-path category."""
    bits = 256
    A, B = synth.mixed_pairs(660, bits, seed=7)
    for a, b in zip(A, B):
        if a == 0 or b == 0:
            continue
        X, Y = am.rshift(a), am.rshift(b)
        t = am.approximate_euclid(X, Y, 32, check=True)
        assert t.bound_violations == 0
        assert t.iterations <= 2 * bits
    # Cases 2-4 return alpha < D (sampled directly)
    rng = np.random.default_rng(8)
    for _ in range(3000):
        X = int.from_bytes(rng.bytes(int(rng.integers(9, 40))), "little") | 1
        Y = int.from_bytes(rng.bytes(int(rng.integers(1, 40))), "little") | 1
        if X < Y:
            X, Y = Y, X
        a, b, case = am.approx(X, Y, 32)
        assert a * (1 << (32 * b)) <= X // Y
        assert a >= 1
        if case != "1":
            assert a < (1 << 32)


def test_rare_paths_exercised():
    """The mixed generator really reaches beta > 0, rshift >= d and every case."""
    A, B = synth.mixed_pairs(1100, 1024, seed=9)
    cases, beta, rge = {}, 0, 0
    for a, b in zip(A, B):
        if a == 0 or b == 0:
            continue
        t = am.gcd_exact(a, b)
        beta += t.beta_pos
        rge += t.r_ge_d
        for k, v in t.cases.items():
            cases[k] = cases.get(k, 0) + v
    assert beta > 0 and rge > 0
    assert set(cases) >= {"1", "2-A", "2-B", "3-A", "3-B", "4-A", "4-B", "4-C"}


def test_rsa_mode_semantics(cfg1):
    """Early termination returns g iff bitlen(g) >= s/2 (O3), matching the oracle's
    exact gcd under the same mapping, and finds exactly the planted hits."""
    N = synth.ints(cfg1.N)
    hits = []
    for i in range(len(N)):
        for j in range(i + 1, len(N)):
            t = am.gcd_rsa(N[i], N[j], 1024)
            if t.gcd != 1:
                hits.append((i, j, t.gcd))
    assert hits == cfg1.truth


def _table4():
    return {(r[0], int(r[1])): [float(x) for x in r[2:]] for r in read_golden("table4_iterations.txt")}


@pytest.mark.parametrize("bits,npairs", [(512, 3000), (1024, 3000), (2048, 400)])
def test_table4_means(bits, npairs):
    """Table IV column (E) (and (A) via the oracle) within 3 combined standard
    errors of the paper's 10,000-pair means.  Inputs: synthetic OpenSSL-style moduli."""
    tab = _table4()
    ms = synth.moduli(npairs + 1, bits, seed=4000 + bits)
    N = synth.ints(ms.N)
    early = np.array([am.gcd_rsa(N[k], N[k + 1], bits).iterations for k in range(npairs)], float)
    non = np.array([am.approximate_euclid(N[k], N[k + 1], 32).iterations for k in range(min(npairs, 1000))],
                   float)
    for name, arr, paper in (("early", early, tab[("early", bits)][4]), ("nonterm", non, tab[("nonterm", bits)][4])):
        se = math.sqrt(arr.var() / arr.size + arr.var() / 10000)
        assert abs(arr.mean() - paper) <= 3 * se + 0.05, (name, bits, arr.mean(), paper, se)
    # column (A): the Original Euclidean algorithm's iteration count, from the C oracle
    orig = np.array([oracle.gcd_trace(N[k], N[k + 1], qmax=1)[1] for k in range(min(npairs, 1000))], float)
    paper_a = tab[("nonterm", bits)][0]
    se = math.sqrt(orig.var() / orig.size + orig.var() / 10000)
    assert abs(orig.mean() - paper_a) <= 3 * se + 0.05, (bits, orig.mean(), paper_a)


def test_table1_binary_and_fast_binary():
    """Table I (L47, L69-L81): on X = 1043915, Y = 768955 the Binary Euclidean
    algorithm takes 24 iterations and Fast Binary 16; both return 5."""
    for fn, it in ((am.binary_euclid, 24), (am.fast_binary_euclid, 16)):
        t = fn(1043915, 768955)
        assert (t.gcd, t.iterations) == (5, it)
        assert fn(768955, 1043915).iterations == it  # X < Y on entry: swap first


@pytest.mark.parametrize("bits,npairs", [(512, 1500), (1024, 800)])
def test_table4_binary_columns(bits, npairs):
    """Table IV columns (C) Binary and (D) Fast Binary, both modes, within 3 combined
    standard errors of the paper's 10,000-pair means (comparison algorithms, N2)."""
    tab = _table4()
    ms = synth.moduli(npairs + 1, bits, seed=4000 + bits)
    N = synth.ints(ms.N)
    for col, fn in ((2, am.binary_euclid), (3, am.fast_binary_euclid)):
        for mode, early in (("early", bits), ("nonterm", None)):
            # (C) early-terminate has no listing in the paper (only (E)'s, L255).  Its printed means
            # (L303/L305) fit a threshold of s/2 - 1 bits, not (E)'s s/2 (reading 20: with
            # s/2 our mean sits 1.5 iterations = 11 standard errors low at 512 bits).  The model is
            # pinned here under that reading; the GPU kernels keep (E)'s s/2 for every algorithm.
            kw = {"early_offset": 1} if (col, mode) == (2, "early") else {}
            arr = np.array([fn(N[k], N[k + 1], early, **kw).iterations for k in range(npairs)], float)
            paper = tab[(mode, bits)][col]
            se = math.sqrt(arr.var() / arr.size + arr.var() / 10000)
            assert abs(arr.mean() - paper) <= 3 * se + 0.05, (col, mode, bits, arr.mean(), paper, se)
    g = [am.binary_euclid(N[k], N[k + 1]).gcd for k in range(50)]
    assert g == [math.gcd(N[k], N[k + 1]) for k in range(50)]


@pytest.mark.parametrize("bits", [512, 1024, 2048, 4096])
def test_c_approx_euclid_matches_model(bits):
    """oracle/approx_euclid.c (the CPU (E) column of Table V) is the
    paper's algorithm: per pair, the same result and the same iteration count as the
    model, in RSA mode on synthetic moduli and in exact mode on the rare-path operands
    (Cases 1-3, beta > 0, rshift >= 32, even and zero inputs)."""
    ms = synth.moduli(24, bits, seed=900 + bits, n_planted_pairs=2)
    N = synth.ints(ms.N)
    for i in range(len(N)):
        for j in range(i + 1, min(len(N), i + 6)):
            t = am.gcd_rsa(N[i], N[j], bits)
            assert oracle.approx_gcd(N[i], N[j], bits, True) == (t.gcd, t.iterations), (bits, i, j)
    A, B = synth.mixed_pairs(220, bits, seed=77 + bits)
    for a, b in zip(A, B):
        t = am.gcd_exact(a, b)
        assert oracle.approx_gcd(a, b, bits, False) == (t.gcd, t.iterations), (bits, a, b)
        assert t.gcd == math.gcd(a, b)


def test_c_approx_euclid_batch_and_counters(cfg1):
    """The batch entry (threads) equals the single-pair calls; its counters equal the
    model's iterations, limb-steps and beta > 0 counts (M2's units)."""
    ii, jj = np.triu_indices(cfg1.m, k=1)
    G, it, ctr = oracle.approx_index_pairs(cfg1.N, ii, jj, 1024, True, nthreads=4)
    N = synth.ints(cfg1.N)
    tr = [am.gcd_rsa(N[i], N[j], 1024) for i, j in zip(ii, jj)]
    assert [int(x) for x in it] == [t.iterations for t in tr]
    assert ctr == [sum(t.iterations for t in tr), sum(t.limb_steps for t in tr), sum(t.beta_pos for t in tr)]
    hits = sorted((int(i), int(j), synth.to_int(G[k])) for k, (i, j) in enumerate(zip(ii, jj)) if synth.to_int(G[k]) != 1)
    assert hits == cfg1.truth
