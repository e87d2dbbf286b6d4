#!/bin/bash
# One GPU session: bench lines for every config, reference arm, ncu launch list
# and one full ncu capture per config.  Output under gpurun_out/.
set -x
mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt
python bench.py > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err
for c in C1 C2 C3 C4; do
  python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for c in C1 C2 C3 C4 C5; do
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
     --log-file gpurun_out/launches_$c.csv python scripts/profile_run.py --config $c --iters 5 > /dev/null 2>&1
done
for c in C3 C4 C5; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:astitch_ -s 2 -c 1 \
     -o gpurun_out/prof_$c -f python scripts/profile_run.py --config $c --iters 3 > gpurun_out/ncu_$c.log 2>&1
done
ls -la gpurun_out
