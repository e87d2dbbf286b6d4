#!/bin/bash
# programmatic dependent launch on/off (flag 512 = NO_PDL)
for c in C1 C2 C3 C4; do
  for f in 0 512; do
    timeout 300 python bench.py --config $c --no-cpu-baseline --flags $f > /tmp/o.json 2>/tmp/e.txt
    python -c "import json; d=json.load(open('/tmp/o.json')); print('$c', 'flags=$f', d['value'], d['us_per_subgraph'])" 2>/dev/null || (echo "fail $c $f"; tail -2 /tmp/e.txt)
  done
done
