#!/bin/bash
# Ablation sweep mirroring the paper's Table 4 on the synthetic
# workloads: each config with the default plan and with one optimisation
# switched off (flags of include/astitch.h):
#   2 FORCE_GLOBAL  regional -> global demotion (row reductions via HBM + grid barrier)
#   4 NO_PACK       no horizontal packing (one row per warp, XLA-style mapping)
#   8 NO_SPLIT      no task splitting of long rows
#  32 NO_TMA        no bulk-copy (TMA) staging: packed tiles, tma_sweep, tma_team
#  64 NO_PREFETCH   no software prefetch of the next row
# Output: gpurun_out/ablation.jsonl (one bench.py line per run, "flags" added).
mkdir -p gpurun_out
out=gpurun_out/ablation.jsonl
: > $out
run() {  # config flags [extra bench args]
  c=$1; f=$2; shift 2
  line=$(timeout 600 python bench.py --config $c --flags $f --no-cpu-baseline --no-e2e --steps 20 --warmup 5 "$@" 2>/dev/null | tail -1)
  if [ -n "$line" ]; then
    echo "$line" | python -c "import json,sys; d=json.load(sys.stdin); d['flags']=$f; d['extra']='$*'; print(json.dumps(d))" >> $out
  else
    echo "{\"config\": {\"workload\": \"$c\"}, \"flags\": $f, \"extra\": \"$*\", \"failed\": true}" >> $out
  fi
}
for f in 0 2 4; do run C1 $f; done
for f in 0 2 4 64; do run C2 $f; done
for f in 0 2 4 32 64; do run C3 $f; done
for f in 0 2 4 32; do run C4 $f; done
for f in 0 4 32 64; do run C5 $f; done
for f in 0 4; do run fig6a $f; done
for f in 0 8; do run fig6b $f --rows 64 --cols 300000; done
python scripts/summarize_ablation.py $out
