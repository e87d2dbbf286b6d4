#!/bin/bash
# C2 one-wave row teams vs the previous mapping
timeout 900 python -m pytest tests/ -q -m gpu -x 2>&1 | tail -2
for i in 1 2 3; do
  echo -n "C2 one-wave: "; bash scripts/bench_brief.sh C2 --no-e2e
  echo -n "C2 thr=256: "; ASTITCH_FORCE_THREADS=256 bash scripts/bench_brief.sh C2 --no-e2e
done
for r in 1184 2368 3000 4736; do echo -n "C2 rows=$r: "; bash scripts/bench_brief.sh C2 --no-e2e --rows $r; done
