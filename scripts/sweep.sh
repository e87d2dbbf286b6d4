#!/bin/bash
# Mapping sweep: bench.py lines for (config, flags, tuning) triples given on
# stdin as "CONFIG FLAGS TUNING [ROWS COLS]" (TUNING "-" = none); summary table at the end.
#   printf 'C5 0 -\nC5 0 sync=0\n' | bash scripts/sweep.sh gpurun_out/sweep.jsonl
out=${1:-gpurun_out/sweep.jsonl}
mkdir -p $(dirname $out)
: > $out
while read cfg flags tune rows cols; do
  [ -z "$cfg" ] && continue
  t=""; [ "$tune" != "-" ] && t="--tune $tune"
  sh=""; [ -n "$rows" ] && sh="--rows $rows --cols $cols"
  line=$(timeout 300 python bench.py --config $cfg --flags $flags $t $sh --no-cpu-baseline --no-e2e --steps 20 --warmup 5 2>>$out.err | tail -1)
  echo "{\"cfg\": \"$cfg\", \"flags\": $flags, \"tune\": \"$tune ${rows}x${cols}\", \"line\": ${line:-null}}" >> $out
done
python - "$out" <<'PY'
import json, sys
for l in open(sys.argv[1]):
    d = json.loads(l); b = d["line"]
    if not b:
        print(d["cfg"], d["flags"], d["tune"], "FAILED"); continue
    c = b["config"]
    print(f'{d["cfg"]:5s} {d["flags"]:3d} {d["tune"]:34s} {b["us_per_subgraph"]:9.2f} us {b["value"]:8.1f} GB/s '
          f'regs {c["regs"]} grid {c["grid"]} thr {c["threads"]}')
PY
