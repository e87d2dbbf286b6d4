#!/bin/bash
# dynamic row tiles (ASTITCH_DYN_TILES=1) for persistent prefetching row teams
ASTITCH_DYN_TILES=1 timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_runtime_gpu.py -q -x 2>&1 | tail -2
for c in C3 fig6a; do
  for i in 1 2; do
  echo -n "$c static: "; bash scripts/bench_brief.sh $c --no-e2e
  echo -n "$c dyn: "; ASTITCH_DYN_TILES=1 bash scripts/bench_brief.sh $c --no-e2e
  done
done
echo -n "C2@32768 static: "; bash scripts/bench_brief.sh C2 --no-e2e --rows 32768
echo -n "C2@32768 dyn: "; ASTITCH_DYN_TILES=1 bash scripts/bench_brief.sh C2 --no-e2e --rows 32768
echo -n "C3 dyn bps4: "; ASTITCH_DYN_TILES=1 ASTITCH_FORCE_BPS=4 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "C3 dyn U2 bps2: "; ASTITCH_DYN_TILES=1 ASTITCH_FORCE_UNROLL=2 ASTITCH_FORCE_BPS=2 bash scripts/bench_brief.sh C3 --no-e2e
