"""Per-opcode executed warp-instructions of one kernel from an ncu source-page CSV
(`ncu -i X.ncu-rep --page source --csv --print-source sass`), split into the fused
update pass (from each BRXU to the closing `SHF.R.W.U32 ..., RZ`) and the rest.

    python tools/ncu_opmix.py SRC.csv [WARP_ITERATIONS]
"""
import csv
import re
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ia, isrc, iex = hdr.index("Address"), hdr.index("Source"), hdr.index("Instructions Executed")
isamp = hdr.index("Warp Stall Sampling (All Samples)")
per = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
mix = {"pass": Counter(), "rest": Counter()}
samp = {"pass": 0, "rest": 0}
in_pass = False
for r in rows[2:]:
    if len(r) <= iex:
        continue
    src = r[isrc].strip()
    m = re.match(r"(@!?U?P\w+\s+)?([A-Z0-9_.]+)", src)
    if not m:
        continue
    op = m.group(2)
    n = float(r[iex] or 0)
    reg = "pass" if in_pass else "rest"
    if op.startswith("BRX"):
        in_pass = True
    elif in_pass and op.startswith("SHF.R.W") and src.rstrip(" ;").endswith("RZ"):
        in_pass = False
    key = op + (" (pred)" if m.group(1) else "")
    mix[reg][key] += n
    samp[reg] += float(r[isamp] or 0)
for reg in ("pass", "rest"):
    tot = sum(mix[reg].values())
    print(f"== {reg}: {tot / per:.1f} warp-instr per unit, stall samples {samp[reg]}")
    for op, n in mix[reg].most_common(40):
        if n / per >= 0.2:
            print(f"   {op:32s} {n / per:8.2f}")
