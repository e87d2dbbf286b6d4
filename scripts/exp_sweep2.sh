#!/bin/bash
# mapping sweep for the packed varlen C3v and the latency-bound C2
for t in 8 16 32; do for b in 2 3 4; do
  echo -n "C3v T=$t bps=$b: "; ASTITCH_FORCE_TEAM=$t ASTITCH_FORCE_BPS=$b bash scripts/bench_brief.sh C3v --no-e2e
done; done
echo -n "C3v T=32 thr=128 bps=6: "; ASTITCH_FORCE_TEAM=32 ASTITCH_FORCE_THREADS=128 ASTITCH_FORCE_BPS=6 bash scripts/bench_brief.sh C3v --no-e2e
echo -n "C2 default: "; bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C2 thr=128 bps=7: "; ASTITCH_FORCE_THREADS=128 ASTITCH_FORCE_BPS=7 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C2 thr=128 bps=8: "; ASTITCH_FORCE_THREADS=128 ASTITCH_FORCE_BPS=8 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C2 thr=256 bps=4: "; ASTITCH_FORCE_BPS=4 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C2 T=16 bps=2: "; ASTITCH_FORCE_TEAM=16 ASTITCH_FORCE_BPS=2 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "C2 eager: "; bash scripts/bench_brief.sh C2 --no-e2e --eager
echo -n "C1 eager: "; bash scripts/bench_brief.sh C1 --no-e2e --eager
echo -n "C3 default: "; bash scripts/bench_brief.sh C3 --no-e2e
