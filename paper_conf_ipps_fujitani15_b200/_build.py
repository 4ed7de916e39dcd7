"""Build libbulkgcd.so in-tree with nvcc for sm_100a (no JIT, no torch extension).

The library is a plain C-ABI shared object (include/bulkgcd.h); CUDA runtime is
linked statically, so the .so only needs the driver at run time.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
SO = os.path.join(PKG, "libbulkgcd.so")
SOURCES = ["api.cu"]
HEADERS = ["kernels.cuh", "euclid.cuh", "smem_euclid.cuh", "hybrid_euclid.cuh", "duff_pass.cuh", "factor.cuh", "gen_duff.py"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

NVCC_FLAGS = [
    "-O3", "-std=c++17",
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-lineinfo", "-Xptxas", "-v",
    "-shared", "-Xcompiler", "-fPIC",
    "-cudart", "static",
]


def _stale() -> bool:
    if not os.path.exists(SO):
        return True
    t = os.path.getmtime(SO)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "bulkgcd.h")]
    return any(os.path.getmtime(d) > t for d in deps if os.path.exists(d))


def build(force: bool = False, verbose: bool = False, extra_flags=(), out: str | None = None) -> str:
    """Regenerate duff_pass.cuh and compile libbulkgcd.so (sm_100a).

    `out`/`extra_flags` build a variant of the same sources elsewhere (tuning)."""
    so = out or SO
    if out is None and not (force or _stale()):
        return SO
    subprocess.check_call([sys.executable, os.path.join(CSRC, "gen_duff.py")])
    tmp = so + f".tmp{os.getpid()}"
    cmd = [NVCC, *NVCC_FLAGS, *extra_flags, "-I", os.path.join(ROOT, "include"), "-o", tmp,
           *[os.path.join(CSRC, s) for s in SOURCES]]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        raise RuntimeError(f"nvcc failed ({res.returncode}):\n{res.stderr[-8000:]}")
    with open(so + ".ptxas.log", "w") as f:
        f.write(res.stderr)
    if verbose:
        print(res.stderr)
    os.replace(tmp, so)
    return so


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
