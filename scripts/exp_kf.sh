#!/bin/bash
# KF (chunk-count) specialisation of masked rows x team size: C3 / C3v timing
for c in C3 C3v; do
  for t in 4 8 16; do
    ASTITCH_FORCE_TEAM=$t bash scripts/bench_brief.sh $c --no-e2e
    ASTITCH_FORCE_TEAM=$t ASTITCH_NO_KF=1 bash scripts/bench_brief.sh $c --no-e2e
  done
done
