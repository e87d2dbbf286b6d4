#!/bin/bash
# usage: gpu_prof.sh CONFIG [FLAGS]
mkdir -p gpurun_out
c=$1; f=${2:-0}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:astitch_ -s 2 -c 1 \
   -o gpurun_out/prof_${c}_f$f -f python scripts/profile_run.py --config $c --iters 3 --flags $f > gpurun_out/ncu_${c}_f$f.log 2>&1
tail -3 gpurun_out/ncu_${c}_f$f.log
