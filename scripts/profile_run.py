#!/usr/bin/env python
"""Minimal launcher for ncu: plan one config and run it `--iters` times.

Inputs are drawn on the device with torch (values only matter for timing;
parity is tests/test_parity_gpu.py).  Usage under gpurun:

  ncu --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/launches.csv python scripts/profile_run.py --config C5
  ncu --set full --clock-control none --import-source on -k regex:astitch_ -s 2 -c 1 \
      -o gpurun_out/prof_C5 python scripts/profile_run.py --config C5
"""

import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--iters", type=int, default=5)
    ap.add_argument("--flags", type=int, default=0)
    ap.add_argument("--rows", type=int, default=None)
    ap.add_argument("--cols", type=int, default=None)
    ap.add_argument("--tune", default=None)
    args = ap.parse_args()

    import torch
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
    from workloads import gen, specs

    spec = specs.get(args.config, rows=args.rows, cols=args.cols)
    if spec.get("segments"):  # packed varlen: seeded segment layout + table
        spec = gen.ragged_spec(spec, gen.CONFIG_SEEDS.get(args.config, 0))
    R, C = spec["rows"], spec["cols"]
    g = torch.Generator(device="cuda").manual_seed(0)
    tdt = {"F32": torch.float32, "BF16": torch.bfloat16, "F16": torch.float16}
    ins = []
    for name, kind, dt in spec["inputs"]:
        if kind == "LENGTHS":
            L = gen.lengths_for(spec, gen.CONFIG_SEEDS.get(args.config, 0))
            ins.append(torch.from_numpy(L).cuda())
            continue
        if kind == "SEGMENTS":
            t = gen.segment_table(spec["segments"]["seg_rows"], spec["segments"]["seg_cols"])
            ins.append(torch.from_numpy(t).cuda())
            continue
        shape = {"FULL": (spec["segments"]["elems"],) if spec.get("segments") else (R, C),
                 "ROWVEC": (R,), "COLVEC": (C,)}[kind]
        ins.append(torch.randn(shape, generator=g, device="cuda", dtype=torch.float32).to(tdt[dt]))
    plan = A.Plan(A.Graph.from_spec(spec), R, C, device=0, flags=args.flags, tune=args.tune)
    outs = plan.alloc_outputs()
    ws = plan.alloc_workspace()
    for _ in range(args.iters):
        plan.run(ins, outs, ws=ws)
    torch.cuda.synchronize()
    d = plan.describe()
    print({"kernel": d["kernels"][0]["name"], "grid": d["kernels"][0]["grid"], "threads": d["mapping"]["threads"],
           "regs": d["kernels"][0]["regs"], "bytes": d["compulsory_bytes"]})


if __name__ == "__main__":
    main()
