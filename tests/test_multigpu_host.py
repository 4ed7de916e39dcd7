"""Multi-GPU plumbing without GPUs: the band partition is a pure host function,
and the hit-list exchange (counts + padded all-gather + merge) runs here over
gloo with world_size 2 on CPU tensors."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_fujitani15_b200.dist import band, band_pairs, gather_hits, pairs_before, records_to_hits


def test_band_covers_exactly_once_and_balances():
    for total in (0, 1, 7, 1000, 4_194_304, 67_108_864):
        for world in (1, 2, 3, 4, 8):
            cuts = [band(total, world, r) for r in range(world)]
            assert cuts[0][0] == 0 and cuts[-1][1] == total
            for (a0, a1), (b0, b1) in zip(cuts, cuts[1:]):
                assert a1 == b0
            sizes = [b - a for a, b in cuts]
            assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        band(10, 2, 2)


def _cohort_pairs_brute(n):
    """Pairs per cohort id by direct enumeration of include/bulkgcd.h's cohort order."""
    out = []
    for b in range((n + 31) // 32):
        for j in range(32 * b + 1, n):
            out.append(sum(1 for t in range(32) if 32 * b + t < j))
    return np.array(out, dtype=np.int64)


def test_pairs_before_matches_enumeration():
    for n in (2, 3, 31, 32, 33, 64, 65, 100, 257):
        cp = _cohort_pairs_brute(n)
        assert cp.sum() == n * (n - 1) // 2
        pre = np.concatenate([[0], np.cumsum(cp)])
        for c in range(len(cp) + 1):
            assert pairs_before(c, n) == pre[c], (n, c)


@pytest.mark.parametrize("n", [64, 257, 16384, 65536])
def test_band_pairs_balance(n):
    """SURVEY.md §8(e) G1 at the configs' sizes (cfg3: 16,384 moduli; cfg5: 65,536 for the
    8-GPU run): the bands of N = 2/4/8 ranks tile the cohort range and each holds its
    share of the n(n-1)/2 pairs to within one cohort (< 32 pairs)."""
    from paper_conf_ipps_fujitani15_b200 import bulkgcd_cohort_count  # host helper of the C ABI
    total_c = (n + 31) // 32 * (n - 1) - 16 * ((n + 31) // 32) * ((n + 31) // 32 - 1)
    total_p = n * (n - 1) // 2
    assert bulkgcd_cohort_count(n) == total_c  # the C ABI's host helper (no GPU needed)
    for world in (1, 2, 3, 4, 8):
        cuts = [band_pairs(n, world, r) for r in range(world)]
        assert cuts[0][0] == 0 and cuts[-1][1] == total_c
        for (a0, a1), (b0, b1) in zip(cuts, cuts[1:]):
            assert a1 == b0 and a0 <= a1
        for r, (c0, c1) in enumerate(cuts):
            got = pairs_before(c1, n) - pairs_before(c0, n)
            assert abs(got - total_p / world) < 32 + 1e-9, (n, world, r, got, total_p / world)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, W, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    # rank r holds r+1 synthetic records {i, j, g...} (rank 1 holds two, rank 0 one); rank 2 none
    n_local = [1, 2, 0][rank]
    rec = torch.zeros((n_local, 2 + W), dtype=torch.int32)
    for k in range(n_local):
        rec[k, 0] = 100 - 10 * rank - k
        rec[k, 1] = 200 + rank
        rec[k, 2] = 7 + rank * 10 + k
    allrec = gather_hits(rec)
    hits = records_to_hits(allrec.numpy(), 32 * W)
    out[rank] = [tuple(map(int, r)) for r in hits.ij]
    dist.destroy_process_group()


def test_gather_hits_gloo_world3():
    W = 4
    port = _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(3, port, W, out), nprocs=3, join=True)
    want = sorted([(100, 200), (90, 201), (89, 201)])
    for r in range(3):
        assert out[r] == want
