#!/bin/bash
# split-factor experiment for few long rows (fig6b shape family)
for cols in 30000 300000; do
 for v in "2,512" "4,512" "8,512" "8,1024" "4,1024"; do
   ASTITCH_FORCE_SPLIT=$v timeout 100 python bench.py --config fig6b --cols $cols --no-cpu-baseline > /tmp/o.json 2> /tmp/e.txt
   python -c "import json; d=json.load(open('/tmp/o.json')); print('fig6b', $cols, '$v', d['value'], d['us_per_subgraph'], d['config']['template'], d['config']['grid'])" 2>/dev/null || (echo "fail $cols $v"; tail -2 /tmp/e.txt)
 done
 timeout 100 python bench.py --config fig6b --cols $cols --no-cpu-baseline --flags 8 > /tmp/o.json 2>/tmp/e.txt
 python -c "import json; d=json.load(open('/tmp/o.json')); print('fig6b', $cols, 'nosplit', d['value'], d['us_per_subgraph'], d['config']['template'], d['config']['grid'])" 2>/dev/null || (echo "fail nosplit"; tail -2 /tmp/e.txt)
done
