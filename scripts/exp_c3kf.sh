#!/bin/bash
# C3 (padded masked softmax): KF specialisation at fixed occupancy targets
bash scripts/bench_brief.sh C3 --no-e2e
for cfg in "16 3" "16 2" "8 2" "8 3" "32 2" "32 3"; do
  set -- $cfg
  echo -n "KF T=$1 bps=$2: "; ASTITCH_KF=1 ASTITCH_FORCE_TEAM=$1 ASTITCH_FORCE_BPS=$2 bash scripts/bench_brief.sh C3 --no-e2e
done
echo -n "noKF T=16 bps=2: "; ASTITCH_FORCE_TEAM=16 ASTITCH_FORCE_BPS=2 bash scripts/bench_brief.sh C3 --no-e2e
echo -n "noKF T=16 bps=4: "; ASTITCH_FORCE_TEAM=16 ASTITCH_FORCE_BPS=4 bash scripts/bench_brief.sh C3 --no-e2e
