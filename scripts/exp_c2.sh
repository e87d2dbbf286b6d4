#!/bin/bash
# C2 latency experiment: templates / teams / prefetch
b() { timeout 120 python bench.py --config C2 --no-cpu-baseline "$@" > /tmp/o.json 2>/tmp/e.txt; python -c "import json; d=json.load(open('/tmp/o.json')); print('C2', '$*', '${ASTITCH_FORCE_TEAM}', d['value'], d['us_per_subgraph'], d['config']['template'], 'regs', d['config']['regs'], 'grid', d['config']['grid'])" 2>/dev/null || (echo "fail $*"; tail -2 /tmp/e.txt); }
b; b --flags 32; b --flags 96
ASTITCH_FORCE_TEAM=96 b --flags 32; ASTITCH_FORCE_TEAM=96 b --flags 96
ASTITCH_FORCE_TEAM=64 b --flags 32; ASTITCH_FORCE_TEAM=64 b --flags 96
ASTITCH_FORCE_TEAM=16 b --flags 96
