#!/bin/bash
# C2 latency structure: rows per wave (trips), prefetch, PDL
for r in 592 1184 2368 4096 4736 8192; do
  echo -n "C2 rows=$r: "; bash scripts/bench_brief.sh C2 --no-e2e --rows $r
done
echo -n "C2 NO_PREFETCH: "; bash scripts/bench_brief.sh C2 --no-e2e --flags 64
echo -n "C2 NO_PDL: "; bash scripts/bench_brief.sh C2 --no-e2e --flags 512
echo -n "C2 thr=128 bps=7: "; ASTITCH_FORCE_THREADS=128 ASTITCH_FORCE_BPS=7 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C2 thr=128 bps=8: "; ASTITCH_FORCE_THREADS=128 ASTITCH_FORCE_BPS=8 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C2 thr=256 bps=3: "; ASTITCH_FORCE_BPS=3 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C2 thr=256 bps=4: "; ASTITCH_FORCE_BPS=4 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C2 hoist: "; ASTITCH_HOIST=1 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C1: "; bash scripts/bench_brief.sh C1 --no-e2e
echo -n "C1 NO_PDL: "; bash scripts/bench_brief.sh C1 --no-e2e --flags 512
