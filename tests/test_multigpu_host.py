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

from paper_conf_ipps_fujitani15_b200.dist import band, gather_hits, records_to_hits


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
