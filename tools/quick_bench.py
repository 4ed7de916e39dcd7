"""Quick device-resident timing of the two kernels (tuning aid, not the bench contract).

python tools/quick_bench.py [--cfg 3] [--pairs 262144] [--reps 3]
Uses BULKGCD_SO to pick an alternative build of the same sources.
"""
import argparse
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_fujitani15_b200 as bg  # noqa: E402
import synth  # noqa: E402


def time_allpairs(ms, bits, reps, stats=False, flags=0):
    dev = torch.device("cuda")
    W = bits // 32
    dN = torch.from_numpy(ms.N.view(np.int32)).to(dev)
    dB = torch.empty(bg.bulkgcd_blocked_words(ms.m, bits), dtype=torch.int32, device=dev)
    bg.bulkgcd_layout_blocked(dN, dB, ms.m, bits)
    total = bg.bulkgcd_cohort_count(ms.m)
    cap = 4096
    dH = torch.zeros(cap * (2 + W), dtype=torch.int32, device=dev)
    dC = torch.zeros(8, dtype=torch.int64, device=dev)
    # stats run
    bg.bulkgcd_all_pairs_band(dN, dB, ms.m, bits, 0, total, dH, cap, dC, bg.FLAG_STATS | flags)
    torch.cuda.synchronize()
    ctr = dC.cpu().numpy()
    pairs = ms.m * (ms.m - 1) // 2
    print(f"  hits={ctr[0]} truth={len(ms.truth)} iters/pair={ctr[2] / pairs:.2f} slow/pair={ctr[3] / pairs:.4f} "
          f"limbs/pair={ctr[4] / pairs:.1f} simt_eff={ctr[2] / max(ctr[5], 1):.4f} "
          f"word_eff={ctr[4] / max(ctr[6], 1):.4f} warp_iters/pair={ctr[5] / 32 / pairs:.3f}")
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        bg.bulkgcd_all_pairs_band(dN, dB, ms.m, bits, 0, total, dH, cap, dC, flags)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    t = min(ts)
    print(f"  all-pairs n={ms.m} bits={bits}: {t * 1e3:.1f} ms  {pairs / t / 1e9:.3f} G GCD/s  "
          f"{t / pairs * 1e9:.3f} ns/GCD  (runs: {[round(x * 1e3, 1) for x in ts]})")
    return t


def time_pairs(m, bits, reps, mode):
    dev = torch.device("cuda")
    W = bits // 32
    if bits == 1024:
        A, B, _ = synth.config2(m)
    else:  # the first m pairs (i < j) of a seeded pool at this width
        pool = int((1 + (1 + 8 * m) ** 0.5) / 2) + 1
        ms = synth.moduli(pool, bits, 4242, n_planted_pairs=2)
        i, j = synth.pair_indices(pool, m)
        A, B = ms.N[i], ms.N[j]
    m_pad = (m + 31) // 32 * 32
    dA = torch.from_numpy(A.view(np.int32)).to(dev)
    dB = torch.from_numpy(B.view(np.int32)).to(dev)
    dAc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
    dBc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
    dGc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
    dS = torch.zeros(8, dtype=torch.int64, device=dev)
    bg.bulkgcd_interleave(dA, dAc, m, m_pad, bits, True)
    bg.bulkgcd_interleave(dB, dBc, m, m_pad, bits, True)
    bg.bulkgcd_pairs_device(dAc, dBc, dGc, m, m_pad, bits, mode, None, dS, bg.FLAG_STATS)
    torch.cuda.synchronize()
    s = dS.cpu().numpy()
    print(f"  iters/pair={s[2] / m:.2f} slow/pair={s[3] / m:.4f}")
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        bg.bulkgcd_pairs_device(dAc, dBc, dGc, m, m_pad, bits, mode, None, dS, 0)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    t = min(ts)
    print(f"  pairs m={m} mode={mode}: {t * 1e3:.2f} ms  {m / t / 1e9:.3f} G GCD/s")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cfg", type=int, default=3)
    ap.add_argument("--pairs", type=int, default=1 << 18)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--flags", default="", help="comma list: smem, fastbin, binary")
    ap.add_argument("--pair-bits", type=int, default=1024)
    a = ap.parse_args()
    print("lib:", os.environ.get("BULKGCD_SO", bg.SO))
    t0 = time.time()
    ms = synth.config_moduli(a.cfg)
    print(f"  generated cfg{a.cfg} in {time.time() - t0:.1f}s")
    fl = {"smem": bg.FLAG_SMEM, "fastbin": bg.FLAG_ALGO_FAST_BINARY, "binary": bg.FLAG_ALGO_BINARY}
    flags = 0
    for f in filter(None, a.flags.split(",")):
        flags |= fl[f]
    time_allpairs(ms, ms.bits, a.reps, flags=flags)
    if a.pairs:
        time_pairs(a.pairs, a.pair_bits, a.reps, bg.MODE_EXACT)
        time_pairs(a.pairs, a.pair_bits, a.reps, bg.MODE_RSA)


if __name__ == "__main__":
    main()
