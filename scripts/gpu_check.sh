#!/bin/bash
# parity + bench lines for every config (quick iteration loop)
mkdir -p gpurun_out
python -m pytest tests/ -q -m gpu -x 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
for c in C5 C1 C2 C3 C4; do
  python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
cat gpurun_out/pytest_gpu.txt
for c in C1 C2 C3 C4 C5; do python -c "
import json,sys
d=json.load(open('gpurun_out/bench_$c.json'))
print('$c', d['value'], 'GB/s', d['us_per_subgraph'], 'us', 'frac', d['roofline']['frac'], 'copy%', d['pct_of_copy_kernel'], d['config']['timing'], d['config']['template'], 'regs', d['config']['regs'], 'grid', d['config']['grid'], d['clocks'])
" 2>&1 | tail -1; done
