#!/bin/bash
# few long rows: cluster size from one wave (default) vs the previous K=8 split and no split;
# store-stream occupancy cap: read-mostly rows keep full occupancy
timeout 1200 python -m pytest tests/ -q -m gpu 2>&1 | tail -2
echo -n "fig6b 64x300000 default: "; bash scripts/bench_brief.sh fig6b --no-e2e --rows 64 --cols 300000
echo -n "fig6b 64x300000 NO_SPLIT: "; bash scripts/bench_brief.sh fig6b --no-e2e --rows 64 --cols 300000 --flags 8
echo -n "fig6b 64x300000 split_row K=8: "; ASTITCH_NO_STREAM=1 ASTITCH_FORCE_SPLIT=8 bash scripts/bench_brief.sh fig6b --no-e2e --rows 64 --cols 300000 --flags 256
echo -n "fig6b 64x30000 default: "; bash scripts/bench_brief.sh fig6b --no-e2e
echo -n "fig6b 64x30000 FORCE_SPLIT: "; bash scripts/bench_brief.sh fig6b --no-e2e --flags 256
echo -n "C1 16x2M: "; bash scripts/bench_brief.sh C1 --no-e2e --rows 16 --cols 2000000
echo -n "fig6b 3x4M: "; bash scripts/bench_brief.sh fig6b --no-e2e --rows 3 --cols 4000000
echo -n "fig6a: "; bash scripts/bench_brief.sh fig6a --no-e2e
echo -n "C3 NO_PACK: "; bash scripts/bench_brief.sh C3 --no-e2e --flags 4
echo -n "C4 NO_PACK: "; bash scripts/bench_brief.sh C4 --no-e2e --flags 4
for c in C1 C2 C3 C3v C4 C5; do echo -n "$c: "; bash scripts/bench_brief.sh $c --no-e2e; done
