mkdir -p gpurun_out
python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "wide or slab or parity_reduced or fused or determinism" 2>&1 | tail -3 > gpurun_out/pytest_wide.txt
for c in 32768 131072; do
  python bench.py --config C5 --rows 4096 --cols $c --no-cpu-baseline --no-e2e --steps 20 > gpurun_out/b_wide_$c.json 2>&1
  python bench.py --config C5 --rows 4096 --cols $c --no-cpu-baseline --no-e2e --steps 20 --tune unroll=4 > gpurun_out/b_wide_${c}_u4.json 2>&1
done
python bench.py --config C5 --rows 16384 --cols 131072 --no-cpu-baseline --no-e2e --steps 10 > gpurun_out/b_wide_big.json 2>&1
