"""beta > 0 rate of approx() at 4096 bits on the GPU.

The paper: 1191 of 201,277,617,364 approx() calls return beta != 0 on 4096-bit moduli
(non-terminate runs, reading 19).  Here: `chunks` x 2^20 pairs of seeded random
odd 4096-bit operands with the top two bits set (the size profile of the moduli), exact
mode (= non-terminate) through bulkgcd_pairs_device with FLAG_STATS; counter 7 of the
shared-memory pairs kernel counts the iterations with beta > 0 (tests/test_gpu_smem.py pins
it to the C implementation of the paper's algorithm event for event).

    python tools/beta_rate.py [chunks] [out.json]
"""
import json
import math
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_fujitani15_b200 as bg  # noqa: E402


def main():
    chunks = int(sys.argv[1]) if len(sys.argv) > 1 else 4
    out = sys.argv[2] if len(sys.argv) > 2 else None
    m, W, bits = 1 << 20, 128, 4096
    dev = torch.device("cuda")
    m_pad = m
    dAc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
    dBc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
    dGc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
    dR = torch.empty(m * W, dtype=torch.int32, device=dev)
    calls = beta = 0
    t0 = time.time()
    for c in range(chunks):
        g = torch.Generator(device=dev)
        g.manual_seed(253_000 + c)
        for dst in (dAc, dBc):  # random odd operands, top two bits set, row-major then interleaved
            dR.copy_(torch.randint(-(1 << 31), 1 << 31, (m * W,), dtype=torch.int64, device=dev, generator=g)
                     .to(torch.int32))
            v = dR.view(m, W)
            v[:, 0] |= 1
            v[:, W - 1] |= -0x40000000  # 0xC0000000
            bg.bulkgcd_interleave(dR, dst, m, m_pad, bits, True)
        dS = torch.zeros(8, dtype=torch.int64, device=dev)
        bg.bulkgcd_pairs_device(dAc, dBc, dGc, m, m_pad, bits, bg.MODE_EXACT, None, dS, bg.FLAG_STATS)
        torch.cuda.synchronize()
        s = dS.cpu().numpy()
        calls += int(s[2])
        beta += int(s[7])
    rate = beta / calls
    paper = 1191 / 201_277_617_364
    res = {"pairs": chunks * m, "bits": bits, "mode": "exact (non-terminate)", "approx_calls": calls,
           "calls_per_gcd": calls / (chunks * m), "beta_pos": beta, "rate": rate,
           "rate_95ci": [max(0.0, (beta - 1.96 * math.sqrt(beta)) / calls), (beta + 1.96 * math.sqrt(beta)) / calls],
           "paper": {"beta_pos": 1191, "approx_calls": 201_277_617_364, "rate": paper, "cite": "PAPER.md L253"},
           "ratio_to_paper": rate / paper,
           "inputs": "seeded random odd 4096-bit integers with the top two bits set (torch.Generator seeds 253000+c)",
           "seconds": time.time() - t0}
    print(json.dumps(res))
    if out:
        with open(out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
