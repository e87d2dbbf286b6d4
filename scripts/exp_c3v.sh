#!/bin/bash
# C3 / C3v tuning sweep: row unroll (rows per team in flight) and team size
mkdir -p gpurun_out
python -m pytest tests/test_ragged_gpu.py -q -m gpu -x 2>&1 | tail -2
for c in C3v C3; do
  for u in 1 2 4; do
    ASTITCH_FORCE_UNROLL=$u bash scripts/bench_brief.sh $c --no-e2e
  done
  for t in 8 32; do
    ASTITCH_FORCE_TEAM=$t bash scripts/bench_brief.sh $c --no-e2e
    ASTITCH_FORCE_TEAM=$t ASTITCH_FORCE_UNROLL=2 bash scripts/bench_brief.sh $c --no-e2e
  done
done
