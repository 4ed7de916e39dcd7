"""Resumable all-pairs search: a cohort-range cursor with
an atomic on-disk checkpoint, so a long search over a large key corpus
(the point of the method is breaking weak keys in collections of
real RSA moduli, ref. [14]: millions of keys) survives interruptions and can
be split across boxes.

The unit of work is the cohort of include/bulkgcd.h (32 consecutive rows x one
column; ids ordered row block by row block).  A search over [c_begin, c_end)
runs in chunks of `chunk` cohorts through bulkgcd_all_pairs_band; after every
chunk the cursor and the hit records found so far are written to the
checkpoint (temporary file + os.replace: a crash leaves either the previous or
the new checkpoint, never a torn one).  Re-running with the same checkpoint
path continues at the cursor.  A checkpoint is bound to its input: n, bits,
the SHA-256 of the moduli and the cohort range; a mismatch raises instead of
mixing results from different corpora.

Multi-box: give each box its own (part, parts) -- the same balanced row bands
as dist.band -- and its own checkpoint; merge_checkpoints() combines the
finished parts.  Moduli stay resident in HBM for the whole search (65,536
1024-bit moduli are 8 MiB; 10^8 would be 12.8 GB, still far below 180 GB), so
"out of core" here is about time, not memory.

Host orchestration only: every GCD runs in libbulkgcd's kernels.
"""
from __future__ import annotations

import hashlib
import json
import os
from dataclasses import dataclass

import numpy as np

from . import Hits, bulkgcd_cohort_count, check_moduli

FORMAT = "bulkgcd-resume-v1"


def digest(N: np.ndarray) -> str:
    return hashlib.sha256(np.ascontiguousarray(N, dtype=np.uint32).tobytes()).hexdigest()


def part_range(total: int, parts: int, part: int) -> tuple[int, int]:
    """Cohort range of `part` out of `parts` equal contiguous shares (row bands)."""
    if parts < 1 or not 0 <= part < parts:
        raise ValueError("bad part/parts")
    return total * part // parts, total * (part + 1) // parts


@dataclass
class State:
    n: int
    bits: int
    sha256: str
    c_begin: int
    c_end: int
    cursor: int
    records: np.ndarray  # uint32[count, 2 + W]: {i, j, g[W]} in discovery order

    @property
    def done(self) -> bool:
        return self.cursor >= self.c_end

    def meta(self) -> dict:
        return {"format": FORMAT, "n": self.n, "bits": self.bits, "sha256": self.sha256,
                "c_begin": self.c_begin, "c_end": self.c_end, "cursor": self.cursor}

    def hits(self) -> Hits:
        W = self.bits // 32
        rec = self.records.reshape(-1, 2 + W)
        order = np.lexsort((rec[:, 1], rec[:, 0]))
        rec = rec[order]
        return Hits(rec[:, :2].copy(), rec[:, 2:].copy(), self.bits)


def save(path: str, st: State) -> None:
    """Atomic write: temporary file in the same directory, fsync, rename."""
    tmp = f"{path}.tmp{os.getpid()}"
    with open(tmp, "wb") as f:
        np.savez(f, meta=np.frombuffer(json.dumps(st.meta()).encode(), dtype=np.uint8), records=st.records)
        f.flush()
        os.fsync(f.fileno())
    os.replace(tmp, path)


def load(path: str) -> State:
    with np.load(path) as z:
        meta = json.loads(bytes(z["meta"]).decode())
        rec = np.array(z["records"], dtype=np.uint32)
    if meta.get("format") != FORMAT:
        raise ValueError(f"{path}: not a {FORMAT} checkpoint")
    return State(meta["n"], meta["bits"], meta["sha256"], meta["c_begin"], meta["c_end"], meta["cursor"], rec)


class DeviceRunner:
    """Runs cohort ranges on the current CUDA device (moduli resident in HBM)."""

    def __init__(self, N: np.ndarray, bits: int, hit_cap: int = 1024):
        from .dist import AllPairsBand
        self.st = AllPairsBand(N, bits, hit_cap=hit_cap)
        self.st.upload(non_blocking=False)
        self.st.layout()

    def __call__(self, c0: int, c1: int) -> np.ndarray:
        self.st.c0, self.st.c1 = c0, c1
        self.st.search()
        return self.st.local_hits().cpu().numpy().view(np.uint32)


def all_pairs_resumable(N: np.ndarray, bits: int, checkpoint: str, *, chunk: int = 1 << 20, part: int = 0,
                        parts: int = 1, max_chunks: int | None = None, runner=None) -> State:
    """Search the cohort range of `part` of `parts` in chunks of `chunk` cohorts,
    checkpointing after each; resumes from `checkpoint` if it exists.

    Returns the state: `.done` tells whether the range is finished, `.hits()`
    the sorted hits found in it so far.  `max_chunks` stops after that many
    chunks (a bounded slice of a long search, and the interruption tests).
    `runner(c0, c1) -> uint32[k, 2+W]` defaults to DeviceRunner (libbulkgcd)."""
    if chunk < 1:
        raise ValueError("chunk must be >= 1")
    N = np.ascontiguousarray(N, dtype=np.uint32)
    W = bits // 32
    check_moduli(N, bits)
    n = int(N.shape[0])
    c_begin, c_end = part_range(bulkgcd_cohort_count(n), parts, part)
    want = State(n, bits, digest(N), c_begin, c_end, c_begin, np.zeros((0, 2 + W), np.uint32))
    if os.path.exists(checkpoint):
        st = load(checkpoint)
        if st.meta() | {"cursor": 0} != want.meta() | {"cursor": 0}:
            raise ValueError(f"{checkpoint} belongs to another search: {st.meta()} vs {want.meta()}")
        if not c_begin <= st.cursor <= c_end:
            raise ValueError(f"{checkpoint}: cursor {st.cursor} outside [{c_begin}, {c_end}]")
    else:
        st = want
        save(checkpoint, st)
    if st.done:
        return st
    run = runner if runner is not None else DeviceRunner(N, bits)
    k = 0
    while not st.done and (max_chunks is None or k < max_chunks):
        c1 = min(st.cursor + chunk, c_end)
        rec = np.asarray(run(st.cursor, c1), dtype=np.uint32).reshape(-1, 2 + W)
        st = State(n, bits, st.sha256, c_begin, c_end, c1, np.concatenate([st.records, rec]))
        save(checkpoint, st)
        k += 1
    return st


def merge_checkpoints(paths) -> Hits:
    """Combine the finished parts of one search (same corpus, disjoint ranges
    covering every cohort) into one sorted hit set."""
    states = [load(p) for p in paths]
    if not states:
        raise ValueError("no checkpoints")
    s0 = states[0]
    for s in states:
        if (s.n, s.bits, s.sha256) != (s0.n, s0.bits, s0.sha256):
            raise ValueError("checkpoints of different searches")
        if not s.done:
            raise ValueError(f"part [{s.c_begin}, {s.c_end}) unfinished (cursor {s.cursor})")
    spans = sorted((s.c_begin, s.c_end) for s in states)
    pos = 0
    for a, b in spans:
        if a != pos:
            raise ValueError(f"cohorts [{pos}, {a}) missing or overlapping")
        pos = b
    if pos != bulkgcd_cohort_count(s0.n):
        raise ValueError("cohort ranges do not cover the search")
    rec = np.concatenate([s.records for s in states])
    return State(s0.n, s0.bits, s0.sha256, 0, pos, pos, rec).hits()
