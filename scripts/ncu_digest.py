#!/usr/bin/env python
"""Digest of one `ncu --set full` report: speed-of-light, occupancy, issue,
stall reasons (PC sampling) and the instruction counts.

    python scripts/ncu_digest.py gpurun_out/prof_r02_C2.ncu-rep [--json out.json]
"""
import csv
import io
import json
import subprocess
import sys

KEYS = ["Duration", "DRAM Throughput", "Memory Throughput", "Issue Slots Busy", "Registers Per Thread", "Block Size",
        "Grid Size", "Achieved Active Warps Per SM", "Theoretical Active Warps per SM", "Eligible Warps Per Scheduler",
        "Warp Cycles Per Issued Instruction", "Executed Ipc Active", "SM Busy", "L2 Hit Rate",
        "Dynamic Shared Memory Per Block"]
RAW = ["dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
       "smsp__sass_inst_executed_op_global_ld.sum", "smsp__sass_inst_executed_op_global_st.sum",
       "smsp__inst_executed_pipe_xu.sum", "sm__pipe_xu_cycles_active.avg.pct_of_peak_sustained_active",
       "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum"]


def rows(path, page):
    out = subprocess.run(["ncu", "-i", path, "--page", page, "--csv"], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def num(x):
    try:
        return float(str(x).replace(",", ""))
    except ValueError:
        return None


def digest(path):
    d = {"report": path, "details": {}, "raw": {}, "stalls_pct": {}}
    r = rows(path, "details")
    if r:
        h = r[0]
        for row in r[1:]:
            m = dict(zip(h, row))
            if m.get("Metric Name") in KEYS:
                d["details"][m["Metric Name"]] = f'{m["Metric Value"]} {m["Metric Unit"]}'.strip()
            d["kernel"] = m.get("Kernel Name")
    r = rows(path, "raw")
    if len(r) >= 2:
        h, v = r[0], r[-1]
        m = dict(zip(h, v))
        for k in RAW:
            if k in m:
                d["raw"][k] = m[k]
        st = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): num(x) or 0.0 for k, x in m.items()
              if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
        tot = sum(st.values()) or 1.0
        d["stalls_pct"] = {k: round(100 * x / tot, 1) for k, x in sorted(st.items(), key=lambda kv: -kv[1]) if x > 0}
    return d


if __name__ == "__main__":
    dd = digest(sys.argv[1])
    if "--json" in sys.argv:
        with open(sys.argv[sys.argv.index("--json") + 1], "w") as f:
            json.dump(dd, f, indent=1)
    print(dd.get("kernel"))
    for k, v in dd["details"].items():
        print(f"  {k:40s} {v}")
    for k, v in dd["raw"].items():
        print(f"  {k:60s} {v}")
    print("  stalls:", ", ".join(f"{k} {v}%" for k, v in list(dd["stalls_pct"].items())[:10]))
