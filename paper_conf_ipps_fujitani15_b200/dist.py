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


def _pairs_in_first(o):
    """Pairs in the first o cohorts of a row block: cohort d (1-based) holds min(32, d) pairs
    (lanes 32b + t < j with j = 32b + d), so sum_{d <= o} min(32, d)."""
    o = np.asarray(o, dtype=np.int64)
    return np.where(o <= 32, o * (o + 1) // 2, 528 + 32 * (o - 32))


def _row_block_prefix(n: int):
    """(cohort prefix P[b], pair prefix Q[b]) over row blocks b = 0..nb (cohorts of row block b
    are j = 32b+1 .. n-1, ordered as in include/bulkgcd.h's cohort ids)."""
    nb = (n + 31) // 32
    b = np.arange(nb, dtype=np.int64)
    cnt = np.maximum(n - 1 - 32 * b, 0)
    P = np.concatenate([[0], np.cumsum(cnt)])
    Q = np.concatenate([[0], np.cumsum(_pairs_in_first(cnt))])
    return P, Q


def pairs_before(c: int, n: int) -> int:
    """Number of pairs i < j in the cohorts [0, c) of an n-moduli all-pairs search."""
    P, Q = _row_block_prefix(n)
    c = min(max(int(c), 0), int(P[-1]))
    b = int(np.searchsorted(P, c, side="right")) - 1
    b = min(b, len(P) - 2) if len(P) > 1 else 0
    return int(Q[b] + _pairs_in_first(c - P[b])) if len(P) > 1 else 0


def band_pairs(n: int, world: int, rank: int) -> tuple[int, int]:
    """Row band of `rank` balanced by PAIRS (= work): the cohort range
    [c_r, c_{r+1}) with c_r the first cohort at which the pair count reaches
    r * n(n-1)/2 / world.  Bands tile [0, cohort_total) and each holds its share of the
    pairs to within one cohort (< 32 pairs), whereas equal cohort counts (band()) give
    up to ~0.1% more pairs to the first bands (their rows have fewer partial cohorts)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    P, Q = _row_block_prefix(n)
    total_pairs = n * (n - 1) // 2

    def cut(r):
        if r == 0:
            return 0
        if r == world:
            return int(P[-1])
        t = -(-r * total_pairs // world)  # ceil(r * total / world)
        b = int(np.searchsorted(Q, t, side="left")) - 1  # Q[b] < t <= Q[b+1]
        need = t - int(Q[b])
        o = int(np.ceil((np.sqrt(8 * need + 1) - 1) / 2)) if need <= 528 else 32 + -(-(need - 528) // 32)
        while o > 0 and _pairs_in_first(o - 1) >= need:
            o -= 1
        while _pairs_in_first(o) < need:
            o += 1
        return int(P[b]) + o

    return cut(rank), cut(rank + 1)


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
        self.c0, self.c1 = band_pairs(self.n, world, rank)
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
