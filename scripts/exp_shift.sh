#!/bin/bash
# shifted fp32 precise row sums vs the fp64 tree (ASTITCH_PRECISE_F64=1)
timeout 900 python -m pytest tests/ -q -m gpu -x 2>&1 | tail -2
for c in C2 C4 C2 C4; do
  echo -n "$c shifted: "; bash scripts/bench_brief.sh $c --no-e2e
  echo -n "$c f64:     "; ASTITCH_PRECISE_F64=1 bash scripts/bench_brief.sh $c --no-e2e
done
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
