#!/bin/bash
# C4 packed TMA tiles: stages / tile rows / threads (prefetch distance = stages - 2)
for t in "4,128,128" "5,128,128" "6,128,128" "8,64,64" "6,64,64" "4,256,256" "3,256,256" "5,96,96" "6,96,96"; do
  echo -n "C4 tile=$t: "; ASTITCH_TILE=$t bash scripts/bench_brief.sh C4 --no-e2e
done
