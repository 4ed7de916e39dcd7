"""Small all-pairs + pairs workload for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_fujitani15_b200 as bg  # noqa: E402
import synth  # noqa: E402

for bits, n in ((1024, 150), (512, 97), (2048, 70), (4096, 40)):
    ms = synth.moduli(n, bits, seed=bits + n, n_planted_pairs=3, cliques=(3,))
    assert bg.bulkgcd_all_pairs(ms.N, bits).as_list() == ms.truth, bits
A, B = synth.mixed_pairs(700, 1024, seed=3)
G = bg.bulkgcd_pairs(synth.from_ints(A, 32), synth.from_ints(B, 32), 1024)
import math  # noqa: E402
assert [synth.to_int(g) for g in G] == [math.gcd(a, b) for a, b in zip(A, B)]
# the chunked host path (> 2^18 pairs: two streams, overlapped copies), RSA mode
A2, B2, _ = synth.config2((1 << 18) + 100)
G2, it2 = bg.bulkgcd_pairs_ex(A2, B2, 1024, bg.MODE_RSA, want_iters=True)
g1, i1 = bg.bulkgcd_pairs_ex(A2[-300:], B2[-300:], 1024, bg.MODE_RSA, want_iters=True)
assert np.array_equal(G2[-300:], g1) and np.array_equal(it2[-300:], i1)
print("sanitize workload ok")
