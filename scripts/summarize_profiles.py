#!/usr/bin/env python
"""Summarise a GPU round's evidence (gpurun_out/) into profiles/<round>_*.

    python scripts/summarize_profiles.py r01

Writes profiles/<round>_summary.md (bench lines, per-launch ncu times and DRAM
bytes, one `ncu --set full` digest per config incl. stall reasons and the
executed-instruction mix) and profiles/ncu_traffic.json (DRAM bytes per launch
of each config's stitched kernel, read by bench.py's roofline.traffic).
"""

import collections
import csv
import glob
import io
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")

RAW = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
       "dram__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
       "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
       "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
       "launch__block_size", "launch__shared_mem_per_block_dynamic", "smsp__inst_executed.sum",
       "smsp__inst_executed_pipe_xu.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
       "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum", "lts__t_bytes.sum"]


def ncu_csv(args):
    r = subprocess.run(["ncu", *args], capture_output=True, text=True)
    return list(csv.reader(io.StringIO(r.stdout)))


def launches(path):
    """Per-launch rows of an `ncu --metrics ... --csv --log-file` list."""
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    if not rows:
        return []
    h = rows[0]
    iname, imet, ival, iid = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    per = collections.OrderedDict()
    for r in rows[1:]:
        per.setdefault((r[iid], r[iname]), {})[r[imet]] = float(r[ival].replace(",", ""))
    return [(k[1], v) for k, v in per.items()]


def full_digest(rep):
    rows = ncu_csv(["-i", rep, "--page", "raw", "--csv"])
    if len(rows) < 3:
        return None
    h, u, v = rows[0], rows[1], rows[2]
    d = {"kernel": v[h.index("Kernel Name")]}
    for m in RAW:
        if m in h:
            d[m] = f"{v[h.index(m)]} {u[h.index(m)]}".strip()
    src = ncu_csv(["-i", rep, "--page", "source", "--csv", "--print-source", "sass"])
    if len(src) > 2:
        hh = src[1]
        iS, iE = hh.index("Source"), hh.index("Instructions Executed")
        mix, stalls = collections.Counter(), collections.Counter()
        scols = [c for c in hh if c.startswith("stall_") and "Not Issued" not in c]
        for r in src[2:]:
            if len(r) < len(hh):
                continue
            toks = r[iS].split()
            if not toks:
                continue
            op = toks[1] if toks[0].startswith("@") and len(toks) > 1 else toks[0]
            mix[op.split(".")[0]] += int(float(r[iE] or 0))
            for c in scols:
                stalls[c] += int(float(r[hh.index(c)] or 0))
        tot = sum(mix.values()) or 1
        d["instruction_mix_top"] = {k: round(100.0 * n / tot, 1) for k, n in mix.most_common(12)}
        st = sum(stalls.values()) or 1
        d["stall_samples_top"] = {k: round(100.0 * n / st, 1) for k, n in stalls.most_common(6)}
    return d


def main():
    rnd = sys.argv[1] if len(sys.argv) > 1 else "r01"
    os.makedirs(PROF, exist_ok=True)
    lines = [f"# {rnd}: B200 measurements (gpurun)", ""]
    gpu = os.path.join(OUT, "gpu.txt")
    if os.path.exists(gpu):
        lines += ["```", open(gpu).read().strip(), "```", ""]
    lines += ["## bench.py lines (CUDA-graph replay, events on the launch stream)", "",
              "| cfg | GB/s | us/subgraph | % of 8 TB/s | frac of measured peak | % of copy kernel | e2e GB/s | sm MHz | reasons |",
              "|---|---|---|---|---|---|---|---|---|"]
    for c in ("C1", "C2", "C3", "C4", "C5", "C3v"):
        p = os.path.join(OUT, f"bench_{c}.json")
        if not os.path.exists(p):
            continue
        try:
            d = json.load(open(p))
        except Exception:
            continue
        shutil.copy(p, os.path.join(PROF, f"{rnd}_bench_{c}.json"))
        lines.append(f"| {c} | {d['value']} | {d['us_per_subgraph']} | {d['pct_of_8TBps']} | {d['roofline']['frac']} | "
                     f"{d['pct_of_copy_kernel']} | {(d.get('e2e') or {}).get('value')} | {d['clocks']['sm_mhz']} | {d['clocks']['reasons']} |")
    ref = os.path.join(OUT, "bench_ref.json")
    if os.path.exists(ref):
        shutil.copy(ref, os.path.join(PROF, f"{rnd}_bench_reference.json"))
    traffic = {}
    lines += ["", "## ncu launch lists (`--metrics gpu__time_duration.sum,dram__bytes_*`, cold-cache, serialised)", "",
              "| cfg | kernel | launches | median us | DRAM read MB/launch | DRAM write MB/launch |", "|---|---|---|---|---|---|"]
    for c in ("C1", "C2", "C3", "C4", "C5", "C3v"):
        p = os.path.join(OUT, f"launches_{c}.csv")
        if not os.path.exists(p):
            continue
        shutil.copy(p, os.path.join(PROF, f"{rnd}_launches_{c}.csv"))
        ls = [v for n, v in launches(p) if n.startswith("astitch_")]
        if not ls:
            continue
        ts = sorted(v.get("gpu__time_duration.sum", 0) for v in ls)
        rd = sorted(v.get("dram__bytes_read.sum", 0) for v in ls)
        wr = sorted(v.get("dram__bytes_write.sum", 0) for v in ls)
        med = lambda a: a[len(a) // 2]
        name = [n for n, _ in launches(p) if n.startswith("astitch_")][0]
        lines.append(f"| {c} | `{name}` | {len(ls)} | {med(ts) / 1e3:.2f} | {med(rd) / 1e6:.2f} | {med(wr) / 1e6:.2f} |")
        traffic[c] = int(med(rd) + med(wr))
    lb = os.path.join(OUT, "launches_bench_C5.csv")
    if os.path.exists(lb):
        shutil.copy(lb, os.path.join(PROF, f"{rnd}_launches_bench_C5.csv"))
        ls = launches(lb)
        tot = sum(v.get("gpu__time_duration.sum", 0) for _, v in ls) or 1
        by = collections.Counter()
        for n, v in ls:
            by[n.split("_")[0] + "_" + (n.split("_")[1] if "_" in n else "")] += v.get("gpu__time_duration.sum", 0)
        lines += ["", f"Launch list of `bench.py --steps 3 --warmup 3` under ncu ({len(ls)} launches): time share by kernel family:", ""]
        for k, v in by.most_common():
            lines.append(f"* `{k}`: {100.0 * v / tot:.1f}%")
    lines += ["", "## ncu --set full digests (one launch each)", ""]
    reps = sorted(glob.glob(os.path.join(OUT, f"prof_{rnd}_C*.ncu-rep"))) or \
        sorted(glob.glob(os.path.join(OUT, "prof_C*.ncu-rep")))
    for rep in reps:
        c = os.path.basename(rep).split(".")[0].split("_")[-1]
        d = full_digest(rep)
        if d is None:
            continue
        lines += [f"### {c}", "", "```", json.dumps(d, indent=1), "```", ""]
        try:
            rb = float(d["dram__bytes_read.sum"].split()[0]) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[d["dram__bytes_read.sum"].split()[1]]
            wb = float(d["dram__bytes_write.sum"].split()[0]) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[d["dram__bytes_write.sum"].split()[1]]
            traffic[c.split("_")[0]] = int(rb + wb)
        except Exception:
            pass
    with open(os.path.join(PROF, "ncu_traffic.json"), "w") as f:
        json.dump(traffic, f, indent=1)
    with open(os.path.join(PROF, f"{rnd}_summary.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
