"""Summarise gpurun_out/ablation.jsonl (scripts/ablation.sh) as a markdown table:
us per subgraph and slowdown of each ablated plan relative to the default."""
import json
import sys

FLAG_NAMES = {0: "default", 2: "FORCE_GLOBAL", 4: "NO_PACK", 8: "NO_SPLIT", 32: "NO_TMA", 64: "NO_PREFETCH"}


def main(path):
    rows = [json.loads(l) for l in open(path) if l.strip()]
    base = {}
    for d in rows:
        if d.get("flags") == 0 and not d.get("failed"):
            base[d["config"]["workload"]] = d["us_per_subgraph"]
    print("| workload | plan | template | us / subgraph | GB/s | x default |")
    print("|---|---|---|---|---|---|")
    for d in rows:
        w = d["config"]["workload"]
        name = FLAG_NAMES.get(d["flags"], str(d["flags"]))
        if d.get("failed"):
            print(f"| {w} | {name} | - | failed | - | - |")
            continue
        us = d["us_per_subgraph"]
        rel = us / base[w] if w in base else float("nan")
        print(f"| {w} | {name} | {d['config']['template']} | {us:.2f} | {d['value']:.0f} | {rel:.2f} |")


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/ablation.jsonl")
