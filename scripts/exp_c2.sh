#!/bin/bash
# C2 latency experiments: block size x occupancy target x colvec hoisting
bash scripts/bench_brief.sh C2 --no-e2e
for cfg in "128 4 0" "128 7 0" "128 8 0" "256 4 0" "128 7 1" "256 3 1"; do
  set -- $cfg
  echo -n "th=$1 bps=$2 hoist=$3  "
  ASTITCH_FORCE_THREADS=$1 ASTITCH_FORCE_BPS=$2 ASTITCH_HOIST=$3 bash scripts/bench_brief.sh C2 --no-e2e
done
echo -n "T=16 "; ASTITCH_FORCE_TEAM=16 bash scripts/bench_brief.sh C2 --no-e2e
echo -n "T=16 bps4 "; ASTITCH_FORCE_TEAM=16 ASTITCH_FORCE_BPS=4 bash scripts/bench_brief.sh C2 --no-e2e
