#!/bin/bash
# early unpack / absorbed stores / unguarded light ops: A/B on B200
# (ASTITCH_LATE_UNPACK=1, ASTITCH_STORE_SELECT=1, ASTITCH_GUARD_LIGHT=1 restore the previous code)
for c in C3 C3v C2 C5 C4 C1; do
  echo -n "$c new: "; bash scripts/bench_brief.sh $c --no-e2e
  echo -n "$c old: "; ASTITCH_LATE_UNPACK=1 ASTITCH_STORE_SELECT=1 ASTITCH_GUARD_LIGHT=1 bash scripts/bench_brief.sh $c --no-e2e
done
for v in ASTITCH_LATE_UNPACK ASTITCH_STORE_SELECT ASTITCH_GUARD_LIGHT; do
  echo -n "C3 $v=1: "; env $v=1 bash scripts/bench_brief.sh C3 --no-e2e
done
