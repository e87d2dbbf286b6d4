#!/bin/bash
# One GPU session producing the round's evidence under gpurun_out/:
#   pytest -m gpu, the default bench line (C5) and every config, the reference
#   arm, the ncu launch list of the bench command itself, dram traffic per
#   launch, and one `ncu --set full` capture per HBM-bound config.
#   usage: bash scripts/gpu_round.sh [ROUND] [PARTS]   (PARTS: any of t b r l p; default all)
R=${1:-r02}; P=${2:-tbrlp}
mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > gpurun_out/gpu.txt
if [[ $P == *t* ]]; then python -m pytest tests/ -q -m gpu -p no:cacheprovider 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt; fi
if [[ $P == *b* ]]; then
  python bench.py > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err
  for c in C1 C2 C3 C4 C3v; do
    python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
  done
fi
if [[ $P == *r* ]]; then
  python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
fi
if [[ $P == *l* ]]; then
  # launch list of the bench command (serialised, cold-cache: compare shares)
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
     --log-file gpurun_out/launches_bench_C5.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 \
     > gpurun_out/ncu_bench_C5.out 2>&1
  for c in C1 C2 C3 C4 C5 C3v; do
    timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
       --log-file gpurun_out/launches_$c.csv python scripts/profile_run.py --config $c --iters 5 > /dev/null 2>&1
  done
fi
if [[ $P == *p* ]]; then
  for c in C3 C4 C5 C2 C3v; do
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:astitch_ -s 2 -c 1 \
       -o gpurun_out/prof_${R}_$c -f python scripts/profile_run.py --config $c --iters 3 > gpurun_out/ncu_$c.log 2>&1
  done
fi
ls -la gpurun_out
