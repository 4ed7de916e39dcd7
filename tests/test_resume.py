"""Resumable all-pairs search: cursor, atomic checkpoint,
resume, input binding, multi-part merge.

Host logic runs here on CPU with a cohort runner built from the ORACLE (the
pairs of each cohort of include/bulkgcd.h, classical Euclid), so the
orchestration is checked against ground truth without a GPU; the gpu test runs
the same driver on libbulkgcd's band kernel."""
import os

import numpy as np
import pytest

import oracle
import synth
from paper_conf_ipps_fujitani15_b200 import bulkgcd_all_pairs, bulkgcd_cohort_count
from paper_conf_ipps_fujitani15_b200.resume import (all_pairs_resumable, load, merge_checkpoints, part_range,
                                                    save)

BITS = 1024
W = BITS // 32


def cohorts(n):
    """Cohort id -> (row block b, column j), in id order (include/bulkgcd.h)."""
    return [(b, j) for b in range((n + 31) // 32) for j in range(32 * b + 1, n)]


class OracleRunner:
    """runner(c0, c1): hit records {i, j, g[W]} of cohorts [c0, c1), by the oracle."""

    def __init__(self, N):
        self.N, self.ids, self.calls = N, cohorts(N.shape[0]), []

    def __call__(self, c0, c1):
        self.calls.append((c0, c1))
        ii, jj = [], []
        for b, j in self.ids[c0:c1]:
            for t in range(32):
                if 32 * b + t < j:
                    ii.append(32 * b + t)
                    jj.append(j)
        if not ii:
            return np.zeros((0, 2 + W), np.uint32)
        hits = oracle.all_pairs_hits(self.N, BITS, np.array(ii), np.array(jj))
        rec = np.zeros((len(hits), 2 + W), np.uint32)
        for r, (i, j, g) in enumerate(hits):
            rec[r, 0], rec[r, 1] = i, j
            rec[r, 2:] = synth.from_int(g, W)
        return rec[::-1].copy()  # discovery order is arbitrary: the driver must sort


@pytest.fixture(scope="module")
def ms():
    return synth.moduli(77, BITS, seed=91, n_planted_pairs=3, cliques=(3,), n_duplicates=1)


def test_cohort_enumeration_matches_library_count(ms):
    assert len(cohorts(ms.m)) == bulkgcd_cohort_count(ms.m)


def test_interrupted_search_resumes_to_the_exact_hit_set(ms, tmp_path):
    ck = str(tmp_path / "search.ckpt")
    truth = oracle.all_pairs_hits(ms.N, BITS)
    total = bulkgcd_cohort_count(ms.m)
    run = OracleRunner(ms.N)
    st = all_pairs_resumable(ms.N, BITS, ck, chunk=13, max_chunks=3, runner=run)
    assert not st.done and st.cursor == 39 and run.calls == [(0, 13), (13, 26), (26, 39)]
    assert load(ck).cursor == 39
    # "crash": a stale temporary file next to the checkpoint is ignored
    with open(ck + ".tmp999", "wb") as f:
        f.write(b"torn")
    run2 = OracleRunner(ms.N)
    st = all_pairs_resumable(ms.N, BITS, ck, chunk=13, max_chunks=2, runner=run2)
    assert run2.calls == [(39, 52), (52, 65)]
    run3 = OracleRunner(ms.N)
    st = all_pairs_resumable(ms.N, BITS, ck, chunk=1000, runner=run3)
    assert st.done and st.cursor == total and run3.calls == [(65, total)]
    assert st.hits().as_list() == truth
    # a finished checkpoint does no work
    run4 = OracleRunner(ms.N)
    assert all_pairs_resumable(ms.N, BITS, ck, runner=run4).hits().as_list() == truth and not run4.calls


def test_checkpoint_is_bound_to_its_input(ms, tmp_path):
    ck = str(tmp_path / "a.ckpt")
    all_pairs_resumable(ms.N, BITS, ck, chunk=5, max_chunks=1, runner=OracleRunner(ms.N))
    other = ms.N.copy()
    other[5, 0] ^= 2
    with pytest.raises(ValueError, match="another search"):
        all_pairs_resumable(other, BITS, ck, runner=OracleRunner(other))
    with pytest.raises(ValueError, match="another search"):
        all_pairs_resumable(ms.N, BITS, ck, parts=2, runner=OracleRunner(ms.N))
    st = load(ck)
    st.cursor = st.c_end + 1
    save(ck, st)
    with pytest.raises(ValueError, match="outside"):
        all_pairs_resumable(ms.N, BITS, ck, runner=OracleRunner(ms.N))


def test_parts_merge_to_the_full_search(ms, tmp_path):
    truth = oracle.all_pairs_hits(ms.N, BITS)
    total = bulkgcd_cohort_count(ms.m)
    paths = [str(tmp_path / f"p{k}.ckpt") for k in range(3)]
    assert [part_range(total, 3, k) for k in range(3)][-1][1] == total
    for k, p in enumerate(paths[:2]):
        assert all_pairs_resumable(ms.N, BITS, p, chunk=17, part=k, parts=3, runner=OracleRunner(ms.N)).done
    with pytest.raises(ValueError, match="cover"):
        merge_checkpoints(paths[:2])
    all_pairs_resumable(ms.N, BITS, paths[2], chunk=17, part=2, parts=3, max_chunks=1, runner=OracleRunner(ms.N))
    with pytest.raises(ValueError, match="unfinished"):
        merge_checkpoints(paths)
    all_pairs_resumable(ms.N, BITS, paths[2], chunk=17, part=2, parts=3, runner=OracleRunner(ms.N))
    assert merge_checkpoints(paths).as_list() == truth
    with pytest.raises(ValueError, match="missing or overlapping"):
        merge_checkpoints([paths[0], paths[2]] + [paths[2]])


def test_bad_arguments(ms, tmp_path):
    with pytest.raises(ValueError):
        all_pairs_resumable(ms.N, BITS, str(tmp_path / "x"), chunk=0, runner=OracleRunner(ms.N))
    with pytest.raises(ValueError):
        all_pairs_resumable(ms.N[:, :8], BITS, str(tmp_path / "y"), runner=OracleRunner(ms.N))
    with pytest.raises(ValueError):
        part_range(10, 2, 2)
    assert not os.path.exists(str(tmp_path / "x"))


@pytest.mark.gpu
def test_resumable_search_on_the_gpu(tmp_path):
    """The driver on libbulkgcd's band kernel: interrupted + resumed in odd-sized
    chunks = the one-shot bulkgcd_all_pairs = the construction ground truth."""
    m = synth.moduli(300, BITS, seed=92, n_planted_pairs=4, cliques=(3,), n_duplicates=1)
    ck = str(tmp_path / "gpu.ckpt")
    st = all_pairs_resumable(m.N, BITS, ck, chunk=97, max_chunks=5)
    assert not st.done and st.cursor == 5 * 97
    st = all_pairs_resumable(m.N, BITS, ck, chunk=1111)
    assert st.done
    want = bulkgcd_all_pairs(m.N, BITS).as_list()
    assert st.hits().as_list() == want == oracle.all_pairs_hits(m.N, BITS)
