#!/bin/bash
# ping-pong prefetch buffers vs early-unpack copy form, per config
for c in C3 C5 fig6a; do
  for i in 1 2; do
  echo -n "$c default: "; bash scripts/bench_brief.sh $c --no-e2e
  echo -n "$c pingpong: "; ASTITCH_PINGPONG=1 bash scripts/bench_brief.sh $c --no-e2e
  done
done
echo -n "C3 NO_PACK default: "; bash scripts/bench_brief.sh C3 --no-e2e --flags 4
echo -n "C3 NO_PACK pingpong: "; ASTITCH_PINGPONG=1 bash scripts/bench_brief.sh C3 --no-e2e --flags 4
echo -n "lmsoftmax default: "; bash scripts/bench_brief.sh lmsoftmax --no-e2e
echo -n "C2 rows=32768 default: "; bash scripts/bench_brief.sh C2 --no-e2e --rows 32768
echo -n "C2 rows=32768 pingpong: "; ASTITCH_PINGPONG=1 bash scripts/bench_brief.sh C2 --no-e2e --rows 32768
