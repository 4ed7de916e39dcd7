"""Per-workload DRAM traffic of the hot kernel (one `ncu --set full` capture each, on the
GPU box) -> profiles/r2_ncu_traffic.json, which bench.py reads for roofline.traffic.

    python tools/ncu_traffic.py OUTDIR   (writes OUTDIR/<workload>.ncu-rep, OUTDIR/r2_ncu_traffic.json)
"""
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import ncu_summary  # noqa: E402

JOBS = {  # workload -> (kernel regex, driver command)
    "cfg3": ("regex:allpairs_kernel", ["python", "tools/prof_allpairs.py", "cfg3", "1"]),
    "cfg4": ("regex:allpairs_kernel", ["python", "tools/prof_allpairs.py", "cfg4", "1"]),
    "cfg6": ("regex:allpairs_kernel", ["python", "tools/prof_allpairs.py", "cfg6", "1"]),
    "cfg8": ("regex:allpairs_hybrid", ["python", "tools/prof_allpairs.py", "cfg8", "1"]),
    # the 4096-bit hybrid kernel at cfg7 size (ncu fails to replay the 5.5 s cfg8 launch)
    "cfg7": ("regex:allpairs_hybrid", ["python", "tools/prof_allpairs.py", "cfg7", "1"]),
    "cfg2": ("regex:pairs_kernel", ["python", "tools/prof_pairs.py", "1048576", "0"]),
}


def summarize(r, rep_name):
    """Summary of one capture from its raw page ({metric: (value, unit)})."""
    s = {}
    for k, name in ncu_summary.KEYS.items():
        if k in r:
            s[name] = ncu_summary.num(r[k][0])
            s[name + "_unit"] = r[k][1]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    dr = s.get("dram_read_bytes", 0.0) * scale.get(s.get("dram_read_bytes_unit", "byte"), 1)
    dw = s.get("dram_write_bytes", 0.0) * scale.get(s.get("dram_write_bytes_unit", "byte"), 1)
    stalls = {k.split("issue_stalled_")[1]: ncu_summary.num(v[0]) for k, v in r.items()
              if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")}
    tot = sum(v for v in stalls.values() if isinstance(v, float)) or 1.0
    s["stall_sample_share"] = {k: round(v / tot, 4) for k, v in sorted(stalls.items(), key=lambda kv: -kv[1])
                               if isinstance(v, float) and v / tot > 0.01}
    s["kernel"] = r.get("Kernel Name", ("?", ""))[0]
    s["dram_bytes_per_launch"] = dr + dw
    s["report"] = rep_name
    return s


def raw_csv(path):
    rows = list(csv.reader(open(path)))
    h, units, v = rows[0], rows[1], rows[2]
    return {k: (x, u) for k, u, x in zip(h, units, v)}


def main():
    out = sys.argv[1]
    only = sys.argv[2:] or list(JOBS)
    os.makedirs(out, exist_ok=True)
    path = os.path.join(out, "r2_ncu_traffic.json")
    res = json.load(open(path)) if os.path.exists(path) else {}
    for w in only:
        regex, cmd = JOBS[w]
        rep = os.path.join(out, f"r2_{w}")
        subprocess.run(["ncu", "--set", "full", "--import-source", "on", "--clock-control", "none", "-k", regex,
                        "-c", "1", "-f", "-o", rep] + cmd, cwd=ROOT, check=False,
                       stdout=open(rep + ".log", "w"), stderr=subprocess.STDOUT)
        if not os.path.exists(rep + ".ncu-rep"):
            print(w, "capture failed (see", rep + ".log)", flush=True)
            continue
        # keep the raw page next to the report (small; the report itself may stay on the box)
        with open(os.path.join(out, f"{w}_raw.csv"), "w") as f:
            subprocess.run(["ncu", "-i", rep + ".ncu-rep", "--page", "raw", "--csv"], stdout=f, check=False)
        res[w] = summarize(raw_csv(os.path.join(out, f"{w}_raw.csv")), os.path.basename(rep) + ".ncu-rep")
        print(w, res[w]["kernel"][:60], "dram bytes/launch", res[w]["dram_bytes_per_launch"], flush=True)
        with open(path, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--from-raw":  # --from-raw OUT.json w=RAW.csv ... (rebuild offline)
        res = {}
        for a in sys.argv[3:]:
            w, _, f = a.partition("=")
            res[w] = summarize(raw_csv(f), f"r2_{w}.ncu-rep")
        json.dump(res, open(sys.argv[2], "w"), indent=1)
    else:
        main()
