#!/bin/bash
# e2e (pinned host buffers through astitch_run_host_pipelined): row chunks
for ch in 8 16 32 64; do
  python bench.py --no-cpu-baseline --steps 5 --warmup 3 --e2e-steps 5 --e2e-chunks $ch 2>/dev/null | python -c "
import json,sys; d=json.load(sys.stdin); e=d['e2e']; print('C5 chunks=$ch', e['value'], 'GB/s', e['ms_per_step'], 'ms', e['pcie'])"
done
for ch in 16 64; do
  python bench.py --config C3 --no-cpu-baseline --steps 5 --warmup 3 --e2e-steps 5 --e2e-chunks $ch 2>/dev/null | python -c "
import json,sys; d=json.load(sys.stdin); e=d['e2e']; print('C3 chunks=$ch', e['value'], 'GB/s', e['ms_per_step'], 'ms', e['pcie'])"
done
