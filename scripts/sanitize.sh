#!/bin/bash
# compute-sanitizer on reduced shapes of every template and round-2 code path
# (memcheck, racecheck, synccheck); output under gpurun_out/sanitize_*.txt
mkdir -p gpurun_out
run() {  # tool config rows cols [flags] [tune]
  local f=${5:-0} t=${6:-}
  local tag=$1_$2_$3x$4_f${f}${t:+_t}
  timeout 900 compute-sanitizer --tool $1 --error-exitcode 99 python scripts/profile_run.py --config $2 --rows $3 --cols $4 \
     --iters 1 --flags $f ${t:+--tune $t} > gpurun_out/sanitize_$tag.txt 2>&1
  echo "$1 $2 [$3,$4] flags=$f ${t:+tune=$t }exit=$? $(grep -E 'ERROR SUMMARY' gpurun_out/sanitize_$tag.txt | tail -1)"
}
for tool in ${TOOLS:-memcheck racecheck synccheck}; do
  run $tool C1 37 129                      # row team, ragged
  run $tool C3 8192 512                    # masked row team, oversubscribed grid
  run $tool C4 5003 36                     # TMA packed tiles, tail tile, oversubscribed grid
  run $tool C2 8192 768                    # one-wave row team, FHADD mixed-precision adds
  run $tool C5 4099 1024                   # global sweep + grid barrier
  run $tool C5 20000 1024 0 threads=1024,sync=1,prefetch=0   # long-sweep mapping: per-step block barrier
  run $tool C5 300 40000                   # column slabs (wide rows)
  run $tool fig7a 300 96                   # global sweep + second barrier + sweep 2
  run $tool bn 3000 96                     # three sweeps, fp64 column means (R7c)
  run $tool C4 3000 36 2                   # FORCE_GLOBAL: hi+lo ROWVEC buffers across barriers
  run $tool fig6a 50001 32                 # non-persistent row teams
  run $tool C5 4099 1024 0 tma=0           # static register global sweep (tma_sweep off)
  run $tool C5 997 4096                    # tma_sweep E=8, one team of 512 lanes
  run $tool C3 4099 512 0 tma_team=0       # masked register row teams (tma_team off)
  run $tool C1 5000 128 0 tma_team=1       # tma_team, unmasked rows, tail tile
done
