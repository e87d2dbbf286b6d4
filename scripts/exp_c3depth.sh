#!/bin/bash
# C3: more row loads in flight per warp (row unroll 2, ping-pong buffers)
for u in 1 2; do for b in 2 3; do
  echo -n "C3 U=$u bps=$b: "; ASTITCH_FORCE_UNROLL=$u ASTITCH_FORCE_BPS=$b bash scripts/bench_brief.sh C3 --no-e2e
done; done
echo -n "C3 pingpong: "; ASTITCH_PINGPONG=1 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "C3 pingpong bps=3: "; ASTITCH_PINGPONG=1 ASTITCH_FORCE_BPS=3 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "C3 T=8 U=1 bps=3: "; ASTITCH_FORCE_TEAM=8 ASTITCH_FORCE_BPS=3 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "C3 T=8 U=1 bps=2: "; ASTITCH_FORCE_TEAM=8 ASTITCH_FORCE_BPS=2 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "C3 T=32 bps=4: "; ASTITCH_FORCE_TEAM=32 ASTITCH_FORCE_BPS=4 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "C3 T=32 bps=6: "; ASTITCH_FORCE_TEAM=32 ASTITCH_FORCE_BPS=6 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "C3 T=32 bps=8: "; ASTITCH_FORCE_TEAM=32 ASTITCH_FORCE_BPS=8 bash scripts/bench_brief.sh C3 --no-e2e
