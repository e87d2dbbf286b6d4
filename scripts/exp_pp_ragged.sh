#!/bin/bash
# ping-pong buffers for packed varlen rows (opt-in ASTITCH_PINGPONG_RAGGED=1)
ASTITCH_PINGPONG_RAGGED=1 timeout 600 python -m pytest tests/test_ragged_gpu.py -q 2>&1 | tail -1
echo -n "C3v default: "; bash scripts/bench_brief.sh C3v --no-e2e
echo -n "C3v pp: "; ASTITCH_PINGPONG_RAGGED=1 bash scripts/bench_brief.sh C3v --no-e2e
echo -n "C3v pp bps2: "; ASTITCH_PINGPONG_RAGGED=1 ASTITCH_FORCE_BPS=2 bash scripts/bench_brief.sh C3v --no-e2e
echo -n "C3v pp T16 bps3: "; ASTITCH_PINGPONG_RAGGED=1 ASTITCH_FORCE_TEAM=16 ASTITCH_FORCE_BPS=3 bash scripts/bench_brief.sh C3v --no-e2e
echo -n "C3v pp T16: "; ASTITCH_PINGPONG_RAGGED=1 ASTITCH_FORCE_TEAM=16 bash scripts/bench_brief.sh C3v --no-e2e
