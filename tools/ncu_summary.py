"""Summarise an ncu --set full capture of the all-pairs kernel into profiles/.

python tools/ncu_summary.py gpurun_out/prof.ncu-rep profiles/ncu_summary.json [launches.csv]

Writes the JSON bench.py reads (`allpairs_dram_bytes_per_launch` = traffic)
plus the integer-pipe evidence north_star asks for: issue utilisation, ALU /
FMA pipe utilisation, warp execution efficiency, DRAM GB/s.
"""
import csv
import io
import json
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "duration_ns",
    "dram__bytes_read.sum": "dram_read_bytes",
    "dram__bytes_write.sum": "dram_write_bytes",
    "smsp__inst_executed.sum": "warp_inst_executed",
    "smsp__thread_inst_executed.sum": "thread_inst_executed",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active": "alu_pipe_pct",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active": "fma_pipe_pct",
    "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active": "fp64_pipe_pct",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active": "xu_pipe_pct",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active": "lsu_pipe_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "sm__instruction_throughput.avg.pct_of_peak_sustained_active": "sm_inst_throughput_pct",
    "smsp__thread_inst_executed_per_inst_executed.ratio": "threads_per_inst",
    "launch__registers_per_thread": "registers_per_thread",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
    "launch__grid_size": "grid_size",
    "launch__block_size": "block_size",
    "sm__cycles_elapsed.avg.per_second": "sm_clock_hz",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_throughput_pct",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active": "alu_pipe_cycles_pct",
    "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed": "fmaheavy_pipe_cycles_pct",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active": "fma_pipe_cycles_pct",
}


def opcode_mix(rep):
    """Executed warp-instructions per SASS opcode (source page), share of the total."""
    import re
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = next((r for r in rows if "Source" in r and "Instructions Executed" in r), None)
    if hdr is None:
        return {}
    i_src, i_ex = hdr.index("Source"), hdr.index("Instructions Executed")
    i_smp = hdr.index("Warp Stall Sampling (All Samples)")
    cnt, smp = {}, {}
    for r in rows[rows.index(hdr) + 1:]:
        m = re.match(r"\s*(@!?U?P\w+\s+)?([A-Z0-9_]+(\.[A-Z0-9_.]+)?)", r[i_src])
        if not m or not r[i_ex]:
            continue
        op = m.group(2)
        cnt[op] = cnt.get(op, 0) + int(r[i_ex])
        smp[op] = smp.get(op, 0) + int(r[i_smp] or 0)
    tot, tots = sum(cnt.values()) or 1, sum(smp.values()) or 1
    top = sorted(cnt.items(), key=lambda kv: -kv[1])[:24]
    return {"total_warp_inst": tot, "per_opcode": {k: {"inst_share": round(v / tot, 4),
                                                       "stall_sample_share": round(smp[k] / tots, 4)}
                                                   for k, v in top}}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units, v = rows[0], rows[1], rows[2]
    return {k: (x, u) for k, u, x in zip(h, units, v)}


def num(x):
    try:
        return float(x.replace(",", ""))
    except ValueError:
        return x


def main():
    rep, out = sys.argv[1], sys.argv[2]
    r = raw(rep)
    s = {"report": rep, "kernel": r.get("Kernel Name", ("?", ""))[0]}
    for k, name in KEYS.items():
        if k in r:
            s[name] = num(r[k][0])
            s[name + "_unit"] = r[k][1]
    stalls = {k.split("issue_stalled_")[1]: num(v[0]) for k, v in r.items()
              if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")}
    tot = sum(v for v in stalls.values() if isinstance(v, float)) or 1.0
    s["stall_sample_share"] = {k: round(v / tot, 4) for k, v in sorted(stalls.items(), key=lambda kv: -kv[1]) if v}
    dr = s.get("dram_read_bytes", 0.0)
    dw = s.get("dram_write_bytes", 0.0)
    # units: ncu reports bytes with a unit column (byte / Kbyte / Mbyte)
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    dr *= scale.get(s.get("dram_read_bytes_unit", "byte"), 1)
    dw *= scale.get(s.get("dram_write_bytes_unit", "byte"), 1)
    s["allpairs_dram_bytes_per_launch"] = dr + dw
    if "threads_per_inst" in s:
        s["warp_execution_efficiency"] = s["threads_per_inst"] / 32.0
    if "duration_ns" in s:
        dur = s["duration_ns"] * (1e-3 if s.get("duration_ns_unit") == "us" else 1)
        if s.get("duration_ns_unit") == "ms":
            dur = s["duration_ns"] * 1e6
        s["dram_GBps"] = (dr + dw) / (dur * 1e-9) / 1e9 if dur else None
    if len(sys.argv) > 3:
        lines = [ln for ln in open(sys.argv[3]) if ln.startswith('"')]
        rd = list(csv.DictReader(io.StringIO("".join(lines))))
        tot_ns = sum(float(x["Metric Value"]) for x in rd)
        share = {}
        for x in rd:
            k = x["Kernel Name"].split("(")[0]
            share[k] = share.get(k, 0.0) + float(x["Metric Value"])
        s["launch_list_share"] = {k: round(v / tot_ns, 5) for k, v in share.items()}
    s["opcode_mix"] = opcode_mix(rep)
    with open(out, "w") as f:
        json.dump(s, f, indent=1)
    print(json.dumps(s, indent=1))


if __name__ == "__main__":
    main()
