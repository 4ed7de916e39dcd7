"""Fill roofline.traffic of bench lines from the ncu capture of the same run and build.

    python tools/merge_traffic.py RUNDIR DEST   (RUNDIR/r2_bench_<w>.json + RUNDIR/r2_ncu_traffic.json -> DEST/)

bench.py reads profiles/r2_ncu_traffic.json when it runs; tools/refresh_r2.sh measures the bench lines
before its ncu captures, so the lines of that run get the traffic of that run here (dram bytes read +
written per launch of the workload's hot kernel, `ncu --set full`)."""
import json
import os
import shutil
import sys

run, dest = sys.argv[1], sys.argv[2]
traffic = json.load(open(os.path.join(run, "r2_ncu_traffic.json")))
for f in sorted(os.listdir(run)):
    if not (f.startswith("r2_bench_") and f.endswith(".json")):
        continue
    line = json.loads(open(os.path.join(run, f)).read())
    w = line.get("config", {}).get("workload", "").split(":")[0]
    r = line.get("roofline")
    if r is not None and w in traffic and line.get("impl") != "reference" and "algo" not in f:
        r["traffic"] = traffic[w]["dram_bytes_per_launch"]
        r["traffic_source"] = f"profiles/r2_ncu_traffic.json ({traffic[w]['report']}, same build)"
    with open(os.path.join(dest, f), "w") as g:
        g.write(json.dumps(line) + "\n")
    print(f, w, r and r.get("traffic"))
shutil.copy(os.path.join(run, "r2_ncu_traffic.json"), os.path.join(dest, "r2_ncu_traffic.json"))
