#!/bin/bash
# usage: bench_brief.sh CONFIG [extra bench args]; prints one summary line
c=$1; shift
python bench.py --config $c --no-cpu-baseline "$@" 2>/dev/null | python -c "
import json,sys
d=json.load(sys.stdin)
print('$c', '$*', d['value'], 'GB/s', d['us_per_subgraph'], 'us', 'frac', d['roofline']['frac'], d['config']['template'], 'regs', d['config']['regs'], 'grid', d['config']['grid'], 'clk', d['clocks']['sm_mhz'], d['clocks']['reasons'])"
