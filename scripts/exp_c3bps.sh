#!/bin/bash
# C3 occupancy sweep after early unpack (fixed blocks/SM targets)
for b in 2 3 4; do
  echo -n "C3 bps=$b: "; ASTITCH_FORCE_BPS=$b bash scripts/bench_brief.sh C3 --no-e2e
done
for t in 32 8; do for b in 2 3; do
  echo -n "C3 T=$t bps=$b: "; ASTITCH_FORCE_TEAM=$t ASTITCH_FORCE_BPS=$b bash scripts/bench_brief.sh C3 --no-e2e
done; done
echo -n "C3 threads=128 bps=6: "; ASTITCH_FORCE_THREADS=128 ASTITCH_FORCE_BPS=6 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "C3 threads=512 bps=1: "; ASTITCH_FORCE_THREADS=512 ASTITCH_FORCE_BPS=1 bash scripts/bench_brief.sh C3 --no-e2e
for b in 1 2 3; do
  echo -n "C3v bps=$b: "; ASTITCH_FORCE_BPS=$b bash scripts/bench_brief.sh C3v --no-e2e
done
echo -n "C3 old bps=4: "; ASTITCH_FORCE_BPS=4 ASTITCH_LATE_UNPACK=1 ASTITCH_STORE_SELECT=1 ASTITCH_GUARD_LIGHT=1 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "C3 old bps=2: "; ASTITCH_FORCE_BPS=2 ASTITCH_LATE_UNPACK=1 ASTITCH_STORE_SELECT=1 ASTITCH_GUARD_LIGHT=1 bash scripts/bench_brief.sh C3 --no-e2e
