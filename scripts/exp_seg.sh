#!/bin/bash
# C3v: two-deep segment lookahead vs one-deep (ASTITCH_SEG_LOOKAHEAD1=1)
timeout 900 python -m pytest tests/ -q -m gpu -x 2>&1 | tail -2
for i in 1 2; do
  echo -n "C3v lookahead2: "; bash scripts/bench_brief.sh C3v --no-e2e
  echo -n "C3v lookahead1: "; ASTITCH_SEG_LOOKAHEAD1=1 bash scripts/bench_brief.sh C3v --no-e2e
done
for c in C1 C2 C3 C4 C5; do echo -n "$c: "; bash scripts/bench_brief.sh $c --no-e2e; done
