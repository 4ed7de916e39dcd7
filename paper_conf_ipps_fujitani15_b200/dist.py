"""Multi-GPU all-pairs search: balanced row bands of the pair triangle, one
process per GPU, and one exchange step -- the hit lists are all-gathered over
NCCL (north_star: "the pair triangle is partitioned across
the GPUs by balanced row bands; only the small hit lists are combined").

The partition works on cohort ids (include/bulkgcd.h: a cohort is 32
consecutive rows x one column; ids are ordered row block by row block, so a
contiguous id range is a row band).  Every cohort holds up to 32 pairs of equal
cost, so equal-length id ranges are balanced to within one cohort.

torch is used only for device memory, streams and the process group; all GCD
work runs in libbulkgcd's kernels.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import (FLAG_STATS, Hits, bulkgcd_all_pairs_band, bulkgcd_blocked_words, bulkgcd_cohort_count,
               bulkgcd_layout_blocked, check_moduli)


def band(total: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous cohort range of `rank` out of `world` equal shares of [0, total)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    return total * rank // world, total * (rank + 1) // world


class AllPairsBand:
    """Device-resident state for one GPU's band of the all-pairs search."""

    def __init__(self, N: np.ndarray, bits: int, rank: int = 0, world: int = 1, device=None, hit_cap: int = 1024):
        self.bits, self.W = bits, bits // 32
        self.n = int(N.shape[0])
        self.device = torch.device(device if device is not None else "cuda")
        N = np.ascontiguousarray(N, dtype=np.uint32)
        check_moduli(N, bits)
        self.h_N = torch.from_numpy(N.view(np.int32)).pin_memory() if self.device.type == "cuda" else \
            torch.from_numpy(N.view(np.int32))
        self.d_N = torch.empty(self.h_N.shape, dtype=torch.int32, device=self.device)
        self.d_blk = torch.empty(bulkgcd_blocked_words(self.n, bits), dtype=torch.int32, device=self.device)
        self.total = bulkgcd_cohort_count(self.n)
        self.c0, self.c1 = band(self.total, world, rank)
        self.cap = hit_cap
        self.d_hits = torch.empty(self.cap * (2 + self.W), dtype=torch.int32, device=self.device)
        self.d_ctr = torch.zeros(8, dtype=torch.int64, device=self.device)

    def upload(self, non_blocking: bool = True) -> None:
        """H2D copy of the moduli (host pinned -> device)."""
        self.d_N.copy_(self.h_N, non_blocking=non_blocking)

    def layout(self) -> None:
        bulkgcd_layout_blocked(self.d_N, self.d_blk, self.n, self.bits)

    def search(self, flags: int = 0) -> None:
        """The band kernel (asynchronous on the current stream)."""
        bulkgcd_all_pairs_band(self.d_N, self.d_blk, self.n, self.bits, self.c0, self.c1, self.d_hits, self.cap,
                               self.d_ctr, flags)

    def local_hits(self) -> torch.Tensor:
        """Synchronises; retries with a larger buffer on overflow.  Returns int32[count, 2+W] on device."""
        count = int(self.d_ctr[0].item())
        if count > self.cap:
            self.cap = count
            self.d_hits = torch.empty(self.cap * (2 + self.W), dtype=torch.int32, device=self.device)
            self.search()
            count = int(self.d_ctr[0].item())
        return self.d_hits[: count * (2 + self.W)].view(count, 2 + self.W)

    def stats(self) -> tuple[int, int]:
        self.search(FLAG_STATS)
        c = self.d_ctr.cpu().numpy()
        return int(c[2]), int(c[3])


def gather_hits(local: torch.Tensor, group=None) -> torch.Tensor:
    """All-gather variable-length hit lists: counts first, then records padded to
    the largest count (the only cross-GPU traffic).  Returns every rank's
    records concatenated (unsorted), on local's device."""
    width = local.shape[1]
    dev = local.device
    if dist.get_backend(group) == "gloo" and local.is_cuda:  # gloo collectives run on host tensors
        local = local.cpu()
    cnt = torch.tensor([local.shape[0]], dtype=torch.int64, device=local.device)
    world = dist.get_world_size(group)
    counts = [torch.zeros_like(cnt) for _ in range(world)]
    dist.all_gather(counts, cnt, group=group)
    counts = [int(c.item()) for c in counts]
    m = max(counts)
    if m == 0:
        return local.new_zeros((0, width)).to(dev)
    pad = local.new_zeros((m, width))
    pad[: local.shape[0]] = local
    parts = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(parts, pad, group=group)
    return torch.cat([p[:c] for p, c in zip(parts, counts)]).to(dev)


def records_to_hits(rec: np.ndarray, bits: int) -> Hits:
    """Sort records {i, j, g[W]} by (i, j) into a Hits object."""
    W = bits // 32
    rec = np.asarray(rec).view(np.uint32).reshape(-1, 2 + W)
    order = np.lexsort((rec[:, 1], rec[:, 0]))
    rec = rec[order]
    return Hits(rec[:, :2].copy(), rec[:, 2:].copy(), bits)


def all_pairs_distributed(N: np.ndarray, bits: int, group=None) -> Hits:
    """Public multi-GPU entry: every rank passes the same host moduli; each
    searches its band on its current CUDA device and all ranks return the
    complete, sorted hit set."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    st = AllPairsBand(N, bits, rank, world)
    st.upload()
    st.layout()
    st.search()
    local = st.local_hits()
    allrec = gather_hits(local, group) if world > 1 else local
    return records_to_hits(allrec.cpu().numpy(), bits)
