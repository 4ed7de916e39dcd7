"""Build variants of libbulkgcd.so with extra nvcc flags (tuning aid).

python tools/variants.py NAME='-DFOO=1 -DBAR=2' NAME2='...'
writes build/variants/libbulkgcd_NAME.so and prints their register/spill lines.
Time them on the GPU with BULKGCD_SO=build/variants/libbulkgcd_NAME.so python tools/quick_bench.py
"""
import os
import re
import shlex
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_fujitani15_b200 import _build  # noqa: E402

OUT = os.path.join(_build.ROOT, "build", "variants")


def main():
    os.makedirs(OUT, exist_ok=True)
    for arg in sys.argv[1:]:
        name, _, flags = arg.partition("=")
        so = os.path.join(OUT, f"libbulkgcd_{name}.so")
        toks = shlex.split(flags)
        env = dict(t[4:].split("=", 1) for t in toks if t.startswith("env:"))  # env:KEY=VAL -> gen_duff settings
        extra = [t for t in toks if not t.startswith("env:")]
        if env:  # the variant's own generated pass (parallel variant builds do not race on csrc/duff_pass.cuh)
            hdr = os.path.join(OUT, f"duff_pass_{name}.cuh")
            env["BULKGCD_DUFF_OUT"] = hdr
            extra.append(f'-DBULKGCD_DUFF_HEADER="{hdr}"')
        saved = {k: os.environ.get(k) for k in env}
        os.environ.update(env)
        try:
            _build.build(out=so, extra_flags=extra)
        finally:
            for k, v in saved.items():
                if v is None:
                    os.environ.pop(k, None)
                else:
                    os.environ[k] = v
        log = open(so + ".ptxas.log").read()
        for m in re.finditer(r"Compiling entry function '_ZN7bulkgcd15allpairs_kernelILi(\d+)ELb0[^']*'[^\n]*\n"
                             r"[^\n]*\n([^\n]*)\n([^\n]*)\n", log):
            print(f"{name:>12} W={m.group(1)}: {m.group(2).strip()} | {m.group(3).strip()}")


if __name__ == "__main__":
    main()
