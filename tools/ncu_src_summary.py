"""Summarise an ncu source-page CSV (--page source --csv --print-source sass):
executed warp-instructions and stall samples by opcode, and the hottest
straight-line regions.  python tools/ncu_src_summary.py src.csv [n_regions]"""
import csv
import re
import sys
from collections import Counter, defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
recs = []
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    src = r[ix["Source"]].strip()
    m = re.match(r"(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]+)", src)
    op = m.group(1) if m else src.split()[0] if src else "?"
    recs.append((int(r[ix["Address"]], 16), src, op, int(r[ix["Instructions Executed"]] or 0),
                 int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)))
tot_i = sum(x[3] for x in recs)
tot_s = sum(x[4] for x in recs)
print(f"total warp-inst {tot_i:.4g}  samples {tot_s}")
byop = defaultdict(lambda: [0, 0])
for _, _, op, n, s in recs:
    byop[op][0] += n
    byop[op][1] += s
print(f"{'opcode':24s} {'inst%':>7s} {'samp%':>7s}")
for op, (n, s) in sorted(byop.items(), key=lambda kv: -kv[1][0])[:40]:
    print(f"{op:24s} {100 * n / tot_i:7.2f} {100 * s / max(tot_s, 1):7.2f}")
# regions: consecutive instructions with the same execution count
reg = []
cur = None
for a, src, op, n, s in recs:
    if cur and cur["n"] == n:
        cur["k"] += 1
        cur["s"] += s
        cur["ops"][op] += 1
    else:
        cur = {"a": a, "n": n, "k": 1, "s": s, "ops": Counter([op])}
        reg.append(cur)
reg.sort(key=lambda r: -r["n"] * r["k"])
nshow = int(sys.argv[2]) if len(sys.argv) > 2 else 25
print("\nhottest regions (same execution count): start, count, #inst, inst%, samp%, ops")
for r in reg[:nshow]:
    print(f"{r['a'] & 0xfffff:6x} {r['n']:>10d} {r['k']:4d} {100 * r['n'] * r['k'] / tot_i:6.2f} "
          f"{100 * r['s'] / max(tot_s, 1):6.2f}  {dict(r['ops'].most_common(6))}")
