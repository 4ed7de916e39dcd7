"""Full oracle sweep of an all-pairs config -> tests/golden/cfg<k>_hits.txt (test infrastructure).

Calls ONLY the CPU oracle (oracle.gcd_index_pairs: classical Euclid with Knuth-D
division) and the seeded input generator (synth).  Every pair
i < j of configs[k] (all m(m-1)/2 pairs) is computed
exactly; a pair is a hit iff bitlen(gcd) >= bits/2 (RSA-mode mapping,
SURVEY.md §8(c) O3 / DESIGN.md reading 18).  The GPU full-size test compares
its hit set with this file gcd by gcd.

    python tools/oracle_sweep.py 3            # ~13 min on 8 cores (1.34e8 pairs)
"""
from __future__ import annotations

import argparse
import hashlib
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import synth  # noqa: E402


def sweep(N: np.ndarray, bits: int, chunk: int = 1 << 20, log=None):
    """All pairs i < j of N in row-major order, `chunk` pairs per oracle call."""
    n = N.shape[0]
    hits = []
    total = n * (n - 1) // 2
    done = 0
    t0 = time.time()
    i = 0
    while i < n - 1:
        # rows i..i2-1 hold about `chunk` pairs
        rows, cnt = [], 0
        i2 = i
        while i2 < n - 1 and (cnt == 0 or cnt + (n - 1 - i2) <= chunk):
            cnt += n - 1 - i2
            i2 += 1
        ii = np.concatenate([np.full(n - 1 - r, r, np.uint64) for r in range(i, i2)])
        jj = np.concatenate([np.arange(r + 1, n, dtype=np.uint64) for r in range(i, i2)])
        hits += oracle.all_pairs_hits(N, bits, ii, jj)
        done += cnt
        i = i2
        if log:
            el = time.time() - t0
            log(f"  {done}/{total} pairs ({100 * done / total:.1f}%), {len(hits)} hits, {el:.0f} s, "
                f"{done / max(el, 1e-9) / 1e3:.1f} k GCD/s")
    hits.sort()
    return hits, done


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", type=int)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    ms = synth.config_moduli(a.config)
    out = a.out or os.path.join(ROOT, "tests", "golden", f"cfg{a.config}_hits.txt")
    t0 = time.time()
    hits, pairs = sweep(ms.N, ms.bits, log=lambda s: print(s, flush=True))
    el = time.time() - t0
    sha = hashlib.sha256(np.ascontiguousarray(ms.N).tobytes()).hexdigest()
    with open(out + ".tmp", "w") as f:
        f.write(f"# Full CPU-oracle sweep of BASELINE.json configs[{a.config - 1}] (cfg{a.config}): every pair i<j of "
                f"{ms.m} synthetic {ms.bits}-bit moduli\n")
        f.write("# (PAPER.md L451/L453: all m(m-1)/2 pairs; hit iff bitlen(gcd) >= bits/2, SURVEY.md §8(c) O3).\n")
        f.write("# Written by tools/oracle_sweep.py, which calls only oracle/ (classical Euclid + Knuth D, L45/L55)\n")
        f.write(f"# and synth/ (seed {2015 + a.config}).  sha256(N) = {sha}\n")
        f.write(f"# pairs {pairs}  hits {len(hits)}  oracle time {el:.0f} s on {os.cpu_count()} cores\n")
        f.write("# i j gcd_hex\n")
        for i, j, g in hits:
            f.write(f"{i} {j} {g:x}\n")
    os.replace(out + ".tmp", out)
    print(f"wrote {out}: {len(hits)} hits over {pairs} pairs in {el:.0f} s")


if __name__ == "__main__":
    main()
