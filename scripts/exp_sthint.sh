#!/bin/bash
# store cache-hint experiment on the HBM-bound configs
for c in C3 C4 C5; do
  for h in "" ".cs"; do
    ASTITCH_ST_HINT=$h timeout 300 python bench.py --config $c --no-cpu-baseline > /tmp/o.json 2>/tmp/e.txt
    python -c "import json; d=json.load(open('/tmp/o.json')); print('$c', 'hint=$h', d['value'], d['us_per_subgraph'])" 2>/dev/null || (echo "fail $c $h"; tail -2 /tmp/e.txt)
  done
done
