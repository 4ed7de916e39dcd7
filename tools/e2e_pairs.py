"""Host-timed bulkgcd_pairs on cfg2-shaped pinned host buffers (the bench's e2e leg), best of N."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_fujitani15_b200 as bg  # noqa: E402
import synth  # noqa: E402

m = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 20
A, B, _ = synth.config2(m)
pin = lambda a: torch.from_numpy(a.view(np.int32)).pin_memory().numpy().view(np.uint32)
A, B = pin(A), pin(B)
G = torch.empty(A.shape, dtype=torch.int32).pin_memory().numpy().view(np.uint32)
bg.bulkgcd_pairs(A, B, 1024, out=G)
ts = []
for _ in range(7):
    t0 = time.perf_counter()
    bg.bulkgcd_pairs(A, B, 1024, out=G)
    ts.append(time.perf_counter() - t0)
t = min(ts)
print(f"  e2e pairs m={m}: {t * 1e3:.2f} ms  {m / t / 1e6:.1f} M GCD/s  (runs {[round(x * 1e3, 2) for x in ts]})")
