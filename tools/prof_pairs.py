"""Run the bulk pairs kernel once on cfg2-shaped pairs (for ncu): python tools/prof_pairs.py [m] [mode]."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_fujitani15_b200 as bg  # noqa: E402
import synth  # noqa: E402

m = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 18
mode = int(sys.argv[2]) if len(sys.argv) > 2 else bg.MODE_EXACT
W = 32
A, B, _ = synth.config2(m)
m_pad = (m + 31) // 32 * 32
dev = torch.device("cuda")
dA = torch.from_numpy(A.view(np.int32)).to(dev)
dB = torch.from_numpy(B.view(np.int32)).to(dev)
dAc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
dBc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
dGc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
dS = torch.zeros(8, dtype=torch.int64, device=dev)
bg.bulkgcd_interleave(dA, dAc, m, m_pad, 1024, True)
bg.bulkgcd_interleave(dB, dBc, m, m_pad, 1024, True)
bg.bulkgcd_pairs_device(dAc, dBc, dGc, m, m_pad, 1024, mode, None, dS, 0)
torch.cuda.synchronize()
print("ok")
