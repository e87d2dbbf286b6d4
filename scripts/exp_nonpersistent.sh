#!/bin/bash
./scripts/micro/stream_mix 2>&1 | grep -E "dynamic|prefetch|tiled U1 t256|persistent U4 t512 x 1"
for c in C3 C3v fig6a; do
  echo -n "$c persistent: "; bash scripts/bench_brief.sh $c --no-e2e
  echo -n "$c nonpersistent: "; ASTITCH_NONPERSISTENT=1 bash scripts/bench_brief.sh $c --no-e2e
done
for b in 2 3 4; do echo -n "C3 nonpersistent bps=$b: "; ASTITCH_NONPERSISTENT=1 ASTITCH_FORCE_BPS=$b bash scripts/bench_brief.sh C3 --no-e2e; done
echo -n "C3v nonpersistent bps=3: "; ASTITCH_NONPERSISTENT=1 ASTITCH_FORCE_BPS=3 bash scripts/bench_brief.sh C3v --no-e2e
echo -n "C2 rows=32768 persistent: "; bash scripts/bench_brief.sh C2 --no-e2e --rows 32768
echo -n "C2 rows=32768 nonpersistent: "; ASTITCH_NONPERSISTENT=1 bash scripts/bench_brief.sh C2 --no-e2e --rows 32768
