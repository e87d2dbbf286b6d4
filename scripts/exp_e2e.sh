#!/bin/bash
# end-to-end (pinned host buffers) vs chunk count
for c in C5 C3; do
 for k in 1 4 8 16; do
  timeout 300 python bench.py --config $c --no-cpu-baseline --e2e-chunks $k --e2e-steps 3 > /tmp/o.json 2>/tmp/e.txt
  python -c "import json; d=json.load(open('/tmp/o.json')); print('$c chunks=$k', 'e2e', d['e2e']['value'], 'GB/s', d['e2e']['ms_per_step'], 'ms; kernel', d['value'])" 2>/dev/null || (echo "fail $c $k"; tail -3 /tmp/e.txt)
 done
done
