mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_runtime_gpu.py -q -x 2>&1 | tail -3
for c in C1 C2 C5; do python scripts/eager_overhead.py $c; done
python scripts/eager_overhead.py C1 512
for c in C1 C2; do python bench.py --config $c --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(d['config']['workload'][:3], d['us_per_subgraph'], d['eager_us_per_call'])"; done
