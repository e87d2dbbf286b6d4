#!/bin/bash
# C5: counter-ordered 128-row tiles with per-tile column partials (ASTITCH_DYN_COLRED=1)
ASTITCH_DYN_COLRED=1 timeout 1200 python -m pytest tests/test_parity_gpu.py tests/test_runtime_gpu.py -q -x 2>&1 | tail -2
for i in 1 2; do
  echo -n "C5 static: "; bash scripts/bench_brief.sh C5 --no-e2e --steps 10
  echo -n "C5 dyn128: "; ASTITCH_DYN_COLRED=1 bash scripts/bench_brief.sh C5 --no-e2e --steps 10
done
for tr in 64 256 512; do
  echo -n "C5 dyn$tr: "; ASTITCH_DYN_COLRED=1 ASTITCH_DYN_COLRED_ROWS=$tr bash scripts/bench_brief.sh C5 --no-e2e --steps 10
done
echo -n "C5 dyn128 thr256 bps2: "; ASTITCH_DYN_COLRED=1 ASTITCH_FORCE_THREADS=256 ASTITCH_FORCE_BPS=2 bash scripts/bench_brief.sh C5 --no-e2e --steps 10
