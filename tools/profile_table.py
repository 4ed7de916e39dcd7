"""Markdown table of the committed bench lines (README / DESIGN numbers): python tools/profile_table.py [DIR]"""
import json
import os
import sys

d = sys.argv[1] if len(sys.argv) > 1 else os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                                         "profiles")
rows = [("cfg3", "r2_bench_cfg3.json"), ("cfg4", "r2_bench_cfg4.json"), ("cfg5", "r2_bench_cfg5.json"),
        ("cfg2", "r2_bench_cfg2.json"), ("cfg1", "r2_bench_cfg1.json"), ("cfg6", "r2_bench_cfg6.json"),
        ("cfg7", "r2_bench_cfg7.json"), ("cfg8", "r2_bench_cfg8.json"),
        ("cfg3 (C)", "r2_bench_cfg3_algoC.json"), ("cfg3 (D)", "r2_bench_cfg3_algoD.json"),
        ("reference arm", "r2_bench_reference_arm.json")]
print("| workload | ms/step | GCD/s | ns/GCD | e2e GCD/s | roofline frac (P_int) | ALU-pipe frac | lane / pass-word eff. |")
print("|---|---|---|---|---|---|---|---|")
for name, f in rows:
    p = os.path.join(d, f)
    if not os.path.exists(p):
        continue
    j = json.loads(open(p).read())
    r = j.get("roofline") or {}
    ap = r.get("alu_pipe") or {}
    e2e = (j.get("e2e") or {}).get("value")
    ns = 1e9 / j["value"] if j.get("value") else None
    fmt = lambda x, k=3: ("%.*f" % (k, x)) if isinstance(x, (int, float)) else "-"
    eff = (f"{fmt(r.get('lane_efficiency'))} / {fmt(r.get('pass_word_efficiency'))}"
           if r.get("lane_efficiency") is not None else "-")
    print(f"| {name} | {fmt(j.get('ms_per_step'), 2)} | {j.get('value', 0):.4g} | {fmt(ns)} | "
          f"{e2e and format(e2e, '.4g') or '-'} | {fmt(r.get('frac'))} | {fmt(ap.get('frac'))} | {eff} |")
