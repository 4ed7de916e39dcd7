"""CPU-side checks of the C ABI: the library builds for sm_100a, loads, exports
every function include/bulkgcd.h declares, and its host-only logic (argument
validation, cohort enumeration) behaves -- no GPU compute calls here."""
import os
import re

import numpy as np
import pytest

from conftest import ROOT


@pytest.fixture(scope="module")
def bg():
    import paper_conf_ipps_fujitani15_b200 as bg
    bg.build()
    return bg


def _declared():
    src = open(os.path.join(ROOT, "include", "bulkgcd.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(bulkgcd_\w+)\s*\(", src)))


def test_exports_every_declared_symbol(bg):
    L = bg.lib()
    names = _declared()
    assert len(names) >= 13
    for n in names:
        assert hasattr(L, n), n
    assert set(names) == set(bg.SYMBOLS)


def test_sass_is_sm100a(bg):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", bg.SO], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def test_strerror_and_device_check(bg):
    L = bg.lib()
    assert L.bulkgcd_strerror(0) == b"ok"
    assert L.bulkgcd_strerror(bg.EINVAL) == b"invalid argument"
    rc = L.bulkgcd_device_check()
    assert rc in (0, bg.ENODEV)


def test_host_validation_no_gpu_needed(bg):
    W = 32
    Z = np.zeros((2, W), np.uint32)
    with pytest.raises(bg.BulkGcdError) as e:
        bg.bulkgcd_pairs(np.zeros((2, 3), np.uint32), np.zeros((2, 3), np.uint32), 96)
    assert e.value.code == bg.EINVAL
    with pytest.raises(bg.BulkGcdError) as e:
        bg.bulkgcd_all_pairs(Z, 1024)  # even moduli rejected before any device work
    assert e.value.code == bg.EINVAL
    # m = 0 / n < 2 are no-ops
    assert bg.bulkgcd_pairs(np.zeros((0, W), np.uint32), np.zeros((0, W), np.uint32), 1024).shape == (0, W)
    # a caller-owned result buffer must match the operands
    for bad in (np.zeros((3, W), np.uint32), np.zeros((2, W), np.int64), np.zeros((W, 2), np.uint32).T):
        with pytest.raises(ValueError):
            bg.bulkgcd_pairs(Z, Z, 1024, out=bad)
    out = np.zeros((0, W), np.uint32)
    assert bg.bulkgcd_pairs(Z[:0], Z[:0], 1024, out=out) is out
    one = np.zeros((1, W), np.uint32)
    one[0, 0] = 3
    assert bg.bulkgcd_all_pairs(one, 1024).ij.shape == (0, 2)
    # cofactors: bits mismatch / index out of range are rejected on the host; no hits is a no-op
    h = bg.Hits(np.array([[0, 1]], np.uint32), np.ones((1, W), np.uint32), 2048)
    with pytest.raises(bg.BulkGcdError) as e:
        bg.bulkgcd_cofactors(Z, 1024, h)
    assert e.value.code == bg.EINVAL
    h = bg.Hits(np.array([[0, 2]], np.uint32), np.ones((1, W), np.uint32), 1024)
    with pytest.raises(bg.BulkGcdError) as e:
        bg.bulkgcd_cofactors(Z, 1024, h)
    assert e.value.code == bg.EINVAL
    assert bg.bulkgcd_cofactors(Z, 1024, bg.Hits(h.ij[:0], h.gcd[:0], 1024)).shape == (0, 2, W)


def test_cohort_enumeration(bg):
    """Cohort count = number of (row block, column j > 32 b) units; every pair
    i < j lies in exactly one cohort."""
    for n in (0, 1, 2, 31, 32, 33, 64, 100, 1000, 16384, 65536):
        nb = (n + 31) // 32
        want = sum(max(0, n - 32 * b - 1) for b in range(nb))
        assert bg.bulkgcd_cohort_count(n) == want
        assert bg.bulkgcd_blocked_words(n, 1024) == nb * 32 * 32
    n = 77
    pairs = set()
    for b in range((n + 31) // 32):
        for j in range(32 * b + 1, n):
            for t in range(32):
                i = 32 * b + t
                if i < j:
                    assert (i, j) not in pairs
                    pairs.add((i, j))
    assert len(pairs) == n * (n - 1) // 2


def test_generated_pass_is_committed(tmp_path):
    """csrc/duff_pass.cuh is what gen_duff.py emits with the default settings (no tuning
    variable in the environment changes the production kernels)."""
    import os
    import subprocess
    import sys
    here = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                        "paper_conf_ipps_fujitani15_b200", "csrc")
    env = {k: v for k, v in os.environ.items() if not k.startswith("BULKGCD_")}
    env["BULKGCD_DUFF_OUT"] = str(tmp_path / "duff_pass.cuh")
    subprocess.check_call([sys.executable, os.path.join(here, "gen_duff.py")], env=env)
    with open(os.path.join(here, "duff_pass.cuh")) as f, open(tmp_path / "duff_pass.cuh") as g:
        assert f.read() == g.read()
