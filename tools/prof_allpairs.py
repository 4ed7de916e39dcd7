"""Run the all-pairs band kernel a few times on n synthetic moduli (for ncu)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_fujitani15_b200 as bg  # noqa: E402
import synth  # noqa: E402

# python tools/prof_allpairs.py N BITS [REPS]  (random moduli)  |  python tools/prof_allpairs.py cfgK [REPS]
if len(sys.argv) > 1 and sys.argv[1].startswith("cfg"):
    ms = synth.config_moduli(int(sys.argv[1][3:]))
    n, bits = ms.m, ms.bits
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
else:
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 2048
    bits = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
    reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
    ms = synth.moduli(n, bits, seed=5, n_planted_pairs=2)
W = bits // 32
dev = torch.device("cuda")
dN = torch.from_numpy(ms.N.view(np.int32)).to(dev)
dB = torch.empty(bg.bulkgcd_blocked_words(n, bits), dtype=torch.int32, device=dev)
bg.bulkgcd_layout_blocked(dN, dB, n, bits)
total = bg.bulkgcd_cohort_count(n)
dH = torch.zeros(1024 * (2 + W), dtype=torch.int32, device=dev)
dC = torch.zeros(8, dtype=torch.int64, device=dev)
for _ in range(reps):
    bg.bulkgcd_all_pairs_band(dN, dB, n, bits, 0, total, dH, 1024, dC, 0)
torch.cuda.synchronize()
print("hits", int(dC[0]))
