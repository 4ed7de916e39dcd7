"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bit-exact on every gcd value and on the exact hit set; per-pair iteration
counts against the paper-algorithm model (the kernels implement the same
exact-floor approx(), so the counts must agree pair by pair).
"""
import math

import numpy as np
import pytest

import oracle
import synth
from oracle import approx_model as am

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def bg():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_fujitani15_b200 as bg
    bg.bulkgcd_device_check()
    return bg


# ------------------------------------------------------------------ pairs
@pytest.mark.parametrize("bits,count", [(512, 3000), (1024, 5000), (2048, 1500)])
def test_pairs_exact_mixed(bg, bits, count):
    """Exact mode on every rare-path category (even, zero, beta > 0, r >= 32,
    Cases 1-4, duplicates, common factors), a ragged count (not a multiple of 32)."""
    W = bits // 32
    A, B = synth.mixed_pairs(count, bits, seed=bits + 1)
    Ah, Bh = synth.from_ints(A, W), synth.from_ints(B, W)
    G = bg.bulkgcd_pairs(Ah, Bh, bits)
    want = oracle.gcd_batch(Ah, Bh)
    bad = np.nonzero(~np.all(G == want, axis=1))[0]
    assert bad.size == 0, [(int(k), A[k], B[k]) for k in bad[:3]]


def test_pairs_exact_iteration_parity(bg):
    bits, W = 1024, 32
    A, B = synth.mixed_pairs(1100, bits, seed=77)
    ms = synth.moduli(400, bits, seed=78)
    N = synth.ints(ms.N)
    A += N[:200]
    B += N[200:]
    Ah, Bh = synth.from_ints(A, W), synth.from_ints(B, W)
    G, it = bg.bulkgcd_pairs_ex(Ah, Bh, bits, bg.MODE_EXACT, want_iters=True)
    for k, (a, b) in enumerate(zip(A, B)):
        t = am.gcd_exact(a, b)
        assert synth.to_int(G[k]) == t.gcd == math.gcd(a, b)
        assert int(it[k]) == t.iterations, (k, a, b, int(it[k]), t.iterations)


@pytest.mark.parametrize("bits", [512, 1024, 2048])
def test_pairs_rsa_mode(bg, bits):
    W = bits // 32
    ms = synth.moduli(801, bits, seed=900 + bits, n_planted_pairs=20, n_duplicates=3)
    N = synth.ints(ms.N)
    rng = np.random.default_rng(bits)
    ii = list(range(800)) + [a for a, b, _ in ms.truth]
    jj = [int(x) for x in rng.integers(0, 801, size=800)] + [b for a, b, _ in ms.truth]
    A = [N[i] for i in ii]
    B = [N[j] for j in jj]
    Ah, Bh = synth.from_ints(A, W), synth.from_ints(B, W)
    G, it = bg.bulkgcd_pairs_ex(Ah, Bh, bits, bg.MODE_RSA, want_iters=True)
    Gx = oracle.gcd_batch(Ah, Bh)
    hit = oracle.rsa_hit(oracle.bitlen_rows(Gx), bits)
    for k in range(len(A)):
        want = synth.to_int(Gx[k]) if hit[k] else 1
        assert synth.to_int(G[k]) == want, k
        t = am.gcd_rsa(A[k], B[k], bits)
        assert t.gcd == want
        assert int(it[k]) == t.iterations, (k, int(it[k]), t.iterations)


def test_pairs_edge_cases(bg):
    W = 32
    assert bg.bulkgcd_pairs(np.zeros((0, W), np.uint32), np.zeros((0, W), np.uint32), 1024).shape == (0, W)
    top = (1 << 1024) - 1
    A = [0, 0, 5, top, top, top - 2, 1 << 1023, 1, 3 ** 600, (1 << 1023) + 1]
    B = [0, 7, 0, top, top - 2, top, 1 << 1000, top, 3 ** 500, (1 << 1023) + 1]
    Ah, Bh = synth.from_ints(A, W), synth.from_ints(B, W)
    G = bg.bulkgcd_pairs(Ah, Bh, 1024)
    assert [synth.to_int(g) for g in G] == [math.gcd(a, b) for a, b in zip(A, B)]


def test_pairs_errors(bg):
    W = 32
    Z = np.zeros((1, W), np.uint32)
    with pytest.raises(bg.BulkGcdError) as e:
        bg.bulkgcd_pairs_ex(Z, Z, 1024, bg.MODE_RSA)  # RSA mode needs odd moduli > 1
    assert e.value.code == bg.EINVAL
    with pytest.raises(bg.BulkGcdError) as e:
        bg.bulkgcd_pairs(np.zeros((1, 3), np.uint32), np.zeros((1, 3), np.uint32), 96)
    assert e.value.code == bg.EINVAL


# -------------------------------------------------------------- all pairs
def test_all_pairs_config1(bg, cfg1):
    hits = bg.bulkgcd_all_pairs(cfg1.N, 1024).as_list()
    assert hits == oracle.all_pairs_hits(cfg1.N, 1024) == cfg1.truth


@pytest.mark.parametrize("n,bits", [(2, 1024), (33, 1024), (95, 512), (70, 2048), (161, 1024)])
def test_all_pairs_exhaustive_small(bg, n, bits):
    """Every pair checked by the oracle; ragged n; cliques and duplicates."""
    ms = synth.moduli(n, bits, seed=n * 7 + bits, n_planted_pairs=min(3, n // 2),
                      cliques=(4,) if n >= 33 else (), n_duplicates=2 if n >= 33 else 0)
    hits = bg.bulkgcd_all_pairs(ms.N, bits).as_list()
    assert hits == oracle.all_pairs_hits(ms.N, bits) == ms.truth


def test_all_pairs_errors(bg, cfg1):
    N = cfg1.N.copy()
    N[5, 0] &= ~np.uint32(1)
    with pytest.raises(bg.BulkGcdError) as e:
        bg.bulkgcd_all_pairs(N, 1024)
    assert e.value.code == bg.EINVAL
    one = cfg1.N[:3].copy()
    one[1] = 0
    one[1, 0] = 1
    with pytest.raises(bg.BulkGcdError):
        bg.bulkgcd_all_pairs(one, 1024)
    assert bg.bulkgcd_all_pairs(cfg1.N[:1], 1024).ij.shape == (0, 2)


@pytest.mark.parametrize("n,bits", [(40, 1024), (37, 512), (36, 2048)])
def test_cofactors_factor_output(bg, n, bits):
    """N3: exact division of both moduli of every hit by g (GPU) == the oracle's
    Knuth-D quotients == the construction's other primes."""
    ms = synth.moduli(n, bits, seed=n + bits, n_planted_pairs=2, cliques=(3,), n_duplicates=1)
    hits = bg.bulkgcd_all_pairs(ms.N, bits)
    assert hits.as_list() == ms.truth
    F = bg.bulkgcd_cofactors(ms.N, bits, hits)
    got = [(synth.to_int(F[h, 0]), synth.to_int(F[h, 1])) for h in range(F.shape[0])]
    assert got == oracle.cofactors(ms.N, ms.truth)


def test_cofactors_errors(bg, cfg1):
    hits = bg.bulkgcd_all_pairs(cfg1.N, 1024)
    assert bg.bulkgcd_cofactors(cfg1.N, 1024, bg.Hits(hits.ij[:0], hits.gcd[:0], 1024)).shape == (0, 2, 32)
    bad = bg.Hits(hits.ij.copy(), hits.gcd.copy(), 1024)
    bad.gcd[0, 0] += 2  # odd, but no longer a divisor
    with pytest.raises(bg.BulkGcdError) as e:
        bg.bulkgcd_cofactors(cfg1.N, 1024, bad)
    assert e.value.code == bg.EINVAL
    bad = bg.Hits(hits.ij.copy(), hits.gcd.copy(), 1024)
    bad.ij[0, 1] = cfg1.m
    with pytest.raises(bg.BulkGcdError):
        bg.bulkgcd_cofactors(cfg1.N, 1024, bad)
    with pytest.raises(bg.BulkGcdError):
        bg.bulkgcd_cofactors(cfg1.N, 1024, bg.Hits(hits.ij, hits.gcd, 2048))


def _band_run(bg, ms, bits, c0, c1, cap):
    W = bits // 32
    dev = torch.device("cuda")
    dN = torch.from_numpy(ms.N.view(np.int32)).to(dev)
    dB = torch.empty(bg.bulkgcd_blocked_words(ms.m, bits), dtype=torch.int32, device=dev)
    bg.bulkgcd_layout_blocked(dN, dB, ms.m, bits)
    dH = torch.zeros(max(cap, 1) * (2 + W), dtype=torch.int32, device=dev)
    dC = torch.zeros(8, dtype=torch.int64, device=dev)
    bg.bulkgcd_all_pairs_band(dN, dB, ms.m, bits, c0, c1, dH, cap, dC, bg.FLAG_STATS)
    torch.cuda.synchronize()
    count = int(dC[0].item())
    rec = dH.cpu().numpy().view(np.uint32).reshape(-1, 2 + W)[:min(count, cap)]
    out = sorted((int(r[0]), int(r[1]), synth.to_int(r[2:])) for r in rec)
    return count, out, dC.cpu().numpy()


def test_band_partition_and_overflow(bg):
    ms = synth.moduli(300, 1024, seed=31, n_planted_pairs=6, cliques=(3,))
    total = bg.bulkgcd_cohort_count(ms.m)
    full = []
    for parts in (1, 2, 3, 8):
        cuts = [total * p // parts for p in range(parts + 1)]
        got = []
        for p in range(parts):
            c, out, _ = _band_run(bg, ms, 1024, cuts[p], cuts[p + 1], 64)
            assert c == len(out)
            got += out
        got.sort()
        if parts == 1:
            full = got
        assert got == full == ms.truth
    # fault injection: a hit buffer too small for the band is counted, not overrun
    c, out, _ = _band_run(bg, ms, 1024, 0, total, 2)
    assert c == len(ms.truth) and len(out) == 2 and set(out) <= set(ms.truth)


def test_all_pairs_stats_counters(bg, cfg1):
    total = bg.bulkgcd_cohort_count(cfg1.m)
    _, _, ctr = _band_run(bg, cfg1, 1024, 0, total, 16)
    N = synth.ints(cfg1.N)
    tr = [am.gcd_rsa(N[i], N[j], 1024) for i in range(64) for j in range(i + 1, 64)]
    assert int(ctr[2]) == sum(t.iterations for t in tr)      # iterations (Table IV's unit)
    assert int(ctr[4]) == sum(t.limb_steps for t in tr)      # limb-steps (the roofline's unit, M2)


@pytest.mark.parametrize("bits,n", [(512, 72), (2048, 40)])
def test_all_pairs_stats_counters_widths(bg, bits, n):
    """Per-width iteration and limb-step totals of the all-pairs kernels (W = 16: 4-limb mix2 pass;
    W = 64: complement form, approx() hoisted, swap on resume) equal the paper's algorithm as the
    model runs it (L107/L127, RSA mode), with planted hits and a clique among the moduli."""
    ms = synth.moduli(n, bits, seed=7000 + bits, n_planted_pairs=3, cliques=(3,))
    total = bg.bulkgcd_cohort_count(ms.m)
    count, out, ctr = _band_run(bg, ms, bits, 0, total, 64)
    assert out == ms.truth and count == len(ms.truth)
    N = synth.ints(ms.N)
    tr = [am.gcd_rsa(N[i], N[j], bits) for i in range(n) for j in range(i + 1, n)]
    assert int(ctr[2]) == sum(t.iterations for t in tr)
    assert int(ctr[4]) == sum(t.limb_steps for t in tr)


def _golden_hits(name):
    """(sha256 of N, sorted [(i, j, g)]) from a tools/oracle_sweep.py golden file."""
    import os
    from conftest import GOLDEN
    sha, hits = None, []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            if line.startswith("#"):
                if "sha256(N) = " in line:
                    sha = line.split("sha256(N) = ")[1].split()[0]
                continue
            i, j, g = line.split()
            hits.append((int(i), int(j), int(g, 16)))
    return sha, hits


def test_all_pairs_config3_full(bg):
    """BASELINE configs[2] at full size, in the launch configuration bench.py times:
    the GPU hit set equals, gcd by gcd, the full CPU-oracle sweep of all 134,209,536
    pairs (tests/golden/cfg3_hits.txt, written by tools/oracle_sweep.py from oracle/
    only), and equals the construction ground truth, which is complete because every
    drawn prime is distinct."""
    import hashlib
    ms = synth.config_moduli(3)
    assert synth.primes_distinct(ms)
    sha, golden = _golden_hits("cfg3_hits.txt")
    assert sha == hashlib.sha256(np.ascontiguousarray(ms.N).tobytes()).hexdigest()
    hits = bg.bulkgcd_all_pairs(ms.N, 1024).as_list()
    assert hits == golden == ms.truth


def test_all_pairs_config4_full(bg):
    """BASELINE configs[3] (2048-bit, 16,384 moduli) at full size: exact hit set
    against construction ground truth, plus a seeded sample through the oracle."""
    ms = synth.config_moduli(4)
    assert ms.bits == 2048
    assert synth.primes_distinct(ms)  # construction truth is the complete hit set (O5(f))
    hits = bg.bulkgcd_all_pairs(ms.N, 2048).as_list()
    assert hits == ms.truth
    rng = np.random.default_rng(4)
    ii = rng.integers(0, ms.m, size=60_000)
    jj = rng.integers(0, ms.m, size=60_000)
    keep = ii < jj
    ii, jj = ii[keep], jj[keep]
    hit = oracle.rsa_hit(oracle.bitlen_rows(oracle.gcd_index_pairs(ms.N, ii, jj)), 2048)
    truth = {(a, b) for a, b, _ in ms.truth}
    assert [bool(h) for h in hit] == [(int(a), int(b)) in truth for a, b in zip(ii, jj)]


def test_all_pairs_config5_full(bg):
    """BASELINE configs[4] (65,536 moduli, 2,147,450,880 pairs) on one GPU: the
    exact hit set (33 planted pairs) against construction ground truth."""
    ms = synth.config_moduli(5)
    assert synth.primes_distinct(ms)  # construction truth is the complete hit set (O5(f))
    hits = bg.bulkgcd_all_pairs(ms.N, 1024).as_list()
    assert len(ms.truth) == 33 and hits == ms.truth


def test_pairs_config2_full_bit_exact(bg):
    """BASELINE configs[1] at full size (2^20 exact-mode pairs, the bench's launch):
    every gcd bit-exact against the oracle's classical Euclid."""
    A, B, _ = synth.config2()
    G = bg.bulkgcd_pairs(A, B, 1024)
    want = oracle.gcd_batch(A, B)
    assert G.shape == want.shape and np.array_equal(G, want)
    assert int((oracle.bitlen_rows(G) > 1).sum()) >= 2  # the planted pairs are among them


def test_pairs_config2_full_rsa_mode(bg):
    """The RSA (early-terminate, L243-L255) pairs kernel on the full 2^20 pairs of
    configs[1], the launch the one-entry resume of euclid_loop runs in: every result
    equals the oracle's exact gcd when it has >= bits/2 bits, else 1 (reading 18)."""
    A, B, ms = synth.config2()
    G, _ = bg.bulkgcd_pairs_ex(A, B, 1024, bg.MODE_RSA)
    Gx = oracle.gcd_batch(A, B)
    hit = oracle.rsa_hit(oracle.bitlen_rows(Gx), 1024)
    want = np.zeros_like(Gx)
    want[:, 0] = 1
    want[hit] = Gx[hit]
    assert G.shape == want.shape and np.array_equal(G, want)
    assert int(hit.sum()) >= 2  # the planted pairs are among them


def test_pairs_chunked_host_path(bg):
    """Host batches above 2^17 pairs run in overlapped chunks on three streams:
    gcds and per-pair iteration counts equal single-chunk calls on the same
    pairs (ragged last chunk, both modes), and the gcds equal the oracle on a
    sample."""
    A, B, _ = synth.config2(3 * (1 << 18) + 777)
    for mode in (bg.MODE_EXACT, bg.MODE_RSA):
        G, it = bg.bulkgcd_pairs_ex(A, B, 1024, mode, want_iters=True)
        for lo in (0, 1 << 18, 3 * (1 << 18)):
            hi = min(lo + 100_000, A.shape[0])
            g1, it1 = bg.bulkgcd_pairs_ex(A[lo:hi], B[lo:hi], 1024, mode, want_iters=True)
            assert np.array_equal(G[lo:hi], g1) and np.array_equal(it[lo:hi], it1)
    idx = np.random.default_rng(5).integers(0, A.shape[0], 4000)
    G = bg.bulkgcd_pairs(A, B, 1024)
    assert np.array_equal(G[idx], oracle.gcd_batch(A[idx], B[idx]))


def _dist_worker(rank, world, port, out):
    import os
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)  # one GPU on the test box: every rank shares it
    from paper_conf_ipps_fujitani15_b200.dist import all_pairs_distributed
    ms = synth.moduli(200, 1024, seed=77, n_planted_pairs=5, cliques=(3,))
    hits = all_pairs_distributed(ms.N, 1024).as_list()
    out[rank] = (hits == ms.truth, len(hits))
    dist.destroy_process_group()


def test_distributed_band_driver_on_one_gpu(bg):
    """dist.all_pairs_distributed with 3 ranks (gloo exchange) sharing cuda:0:
    bands + hit gather + merge reproduce the exact hit set on every rank."""
    import socket
    import torch.multiprocessing as mp
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    out = mp.Manager().dict()
    mp.spawn(_dist_worker, args=(3, port, out), nprocs=3, join=True)
    assert all(out[r][0] for r in range(3)), dict(out)


def _nccl_worker(rank, world, port, out):
    import os
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)
    from paper_conf_ipps_fujitani15_b200 import dist as bgd
    ms = synth.moduli(200, 1024, seed=78, n_planted_pairs=5, cliques=(3,))
    N = torch.from_numpy(ms.N.view(np.int32)).to(dev)
    dist.broadcast(N, src=0)  # bench.py's replication of the moduli (rank 0 generates)
    st = bgd.AllPairsBand(N.cpu().numpy().view(np.uint32), 1024, rank, world)
    st.upload()
    st.layout()
    st.search()
    rec = bgd.gather_hits(st.local_hits())  # NCCL all-gather of counts + padded records
    hits = bgd.records_to_hits(rec.cpu().numpy(), 1024).as_list()
    out[rank] = (hits == ms.truth, len(hits), dist.get_backend(), rec.is_cuda)
    dist.destroy_process_group()


def test_nccl_exchange_single_rank(bg):
    """The NCCL data plane of the multi-GPU path (communicator on cuda:0, broadcast of the
    moduli, all-gather of hit counts and padded hit records on device tensors) with one rank:
    the only NCCL configuration a one-GPU box can run without ranks that wait on each other."""
    import socket
    import torch.multiprocessing as mp
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    out = mp.Manager().dict()
    mp.spawn(_nccl_worker, args=(1, port, out), nprocs=1, join=True)
    ok, n, backend, on_device = out[0]
    assert ok and backend == "nccl" and on_device, dict(out)


def test_bench_multirank_path_gloo(bg):
    """bench.py's N > 1 code path (torchrun, band split, hit exchange, max-over-ranks
    timing) on the single test GPU, with gloo standing in for NCCL."""
    import json
    import os
    import socket
    import subprocess
    import sys
    from conftest import ROOT
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    env = dict(os.environ, BULKGCD_BENCH_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--workload", "cfg1", "--steps", "3", "--warmup", "3", "--no-cpu-baseline",
           "--e2e-steps", "1"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout
    rec = json.loads(lines[0])
    assert rec["n_gpus"] == 2 and rec["config"]["hits_ok"] and rec["config"]["hits"] == 3
    assert rec["value"] > 0 and rec["e2e"]["value"] > 0


def test_concurrent_host_threads(bg, cfg1):
    """include/bulkgcd.h B5 (reentrant; the only global state is the lazily created
    per-device context): 4 host threads call bulkgcd_pairs (one of them above the
    2^17-pair chunk size, i.e. the multi-stream chunked path) and bulkgcd_all_pairs at
    the same time, three rounds each.  ctypes drops the GIL around the C calls, so the
    calls overlap; every result must equal the oracle's."""
    import threading
    jobs = []
    for t in range(4):
        if t == 0:
            A, B, _ = synth.config2(300_000)
        else:
            a, b = synth.mixed_pairs(2000 + 500 * t, 1024, seed=700 + t)
            A, B = synth.from_ints(a, 32), synth.from_ints(b, 32)
        ms = synth.moduli(96 + 32 * t, 1024, seed=800 + t, n_planted_pairs=2, cliques=(3,))
        jobs.append((A, B, ms))
    out = [[] for _ in jobs]
    errs = []

    def work(t):
        try:
            A, B, ms = jobs[t]
            for _ in range(3):
                out[t].append((bg.bulkgcd_pairs(A, B, 1024), bg.bulkgcd_all_pairs(ms.N, 1024).as_list()))
        except Exception as e:  # noqa: BLE001 -- reported below
            errs.append((t, repr(e)))

    th = [threading.Thread(target=work, args=(t,)) for t in range(len(jobs))]
    for x in th:
        x.start()
    for x in th:
        x.join()
    assert not errs, errs
    for (A, B, ms), res in zip(jobs, out):
        want_g = oracle.gcd_batch(A, B)
        want_h = oracle.all_pairs_hits(ms.N, 1024)
        assert want_h == ms.truth
        assert len(res) == 3
        for G, hits in res:
            assert np.array_equal(G, want_g)
            assert hits == want_h
