#!/bin/bash
# C4 packed-tile pipeline experiment: stages, tile rows, threads
b() { timeout 120 python bench.py --config C4 --no-cpu-baseline "$@" > /tmp/o.json 2>/tmp/e.txt; python -c "import json; d=json.load(open('/tmp/o.json')); print('C4', '${ASTITCH_TILE}', d['value'], d['us_per_subgraph'], d['config']['template'], 'regs', d['config']['regs'], 'grid', d['config']['grid'])" 2>/dev/null || (echo "fail ${ASTITCH_TILE}"; tail -2 /tmp/e.txt); }
b
for t in "3,128,128" "6,128,128" "4,256,256" "6,64,64" "8,64,64" "4,64,64" "5,128,128" "3,256,256"; do ASTITCH_TILE=$t b; done
