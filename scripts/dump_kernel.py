#!/usr/bin/env python
"""Plan a config on the host (no GPU) and write its generated CUDA source and
sm_100a cubin, for `cuobjdump -sass` / `nvdisasm` inspection.

  python scripts/dump_kernel.py C3 /tmp/out [--flags N] [--rows R] [--cols C]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("outdir")
    ap.add_argument("--flags", type=int, default=0)
    ap.add_argument("--rows", type=int, default=None)
    ap.add_argument("--cols", type=int, default=None)
    ap.add_argument("--tune", default=None, help="astitch_plan_ex tuning string, e.g. bps=2,unroll=2")
    a = ap.parse_args()
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
    from workloads import specs
    s = specs.get(a.config, rows=a.rows, cols=a.cols)
    if s.get("segments"):
        from workloads import gen
        s = gen.ragged_spec(s, gen.CONFIG_SEEDS.get(a.config, 0))
    p = A.Plan(A.Graph.from_spec(s), s["rows"], s["cols"], device=-1, flags=a.flags, tune=a.tune)
    os.makedirs(a.outdir, exist_ok=True)
    base = os.path.join(a.outdir, f"{a.config}_f{a.flags}")
    with open(base + ".cu", "w") as f:
        f.write(p.source(0))
    with open(base + ".cubin", "wb") as f:
        f.write(p.cubin(0))
    print(base, p.describe()["kernels"][0])


if __name__ == "__main__":
    main()
