#!/bin/bash
# row_stream: inputs staged in smem (ASTITCH_STAGE=1, budget ASTITCH_STAGE_KB per CTA) vs re-read from L2/HBM
timeout 600 python -m pytest tests/test_parity_gpu.py -q -m gpu -x -k "row_stream" 2>&1 | tail -2
run() { timeout 300 python bench.py "$@" --no-cpu-baseline --no-e2e --steps 10 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$*', d['us_per_subgraph'], 'us', d['value'], 'GB/s', d['config']['template'], d['config']['grid'], d['config']['regs'])"; }
for a in "--config lmsoftmax" "--config C1 --rows 4096 --cols 100000" "--config C4 --rows 4096 --cols 60000"; do
  run $a
  ASTITCH_STAGE=1 run $a
  ASTITCH_STAGE=1 ASTITCH_STAGE_KB=40 run $a
done
