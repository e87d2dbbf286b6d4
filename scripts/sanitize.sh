#!/bin/bash
# compute-sanitizer on reduced shapes of every template (memcheck, racecheck,
# synccheck); output under gpurun_out/sanitize_*.txt
mkdir -p gpurun_out
run() {  # tool config rows cols
  timeout 600 compute-sanitizer --tool $1 --error-exitcode 99 python scripts/profile_run.py --config $2 --rows $3 --cols $4 --iters 1 \
     > gpurun_out/sanitize_$1_$2_$3x$4.txt 2>&1
  echo "$1 $2 [$3,$4] exit=$? $(grep -E 'ERROR SUMMARY' gpurun_out/sanitize_$1_$2_$3x$4.txt | tail -1)"
}
for tool in memcheck racecheck synccheck; do
  run $tool C1 37 129        # row team, ragged
  run $tool C3 8192 512      # masked row team
  run $tool C4 5003 36       # TMA packed tiles, tail tile
  run $tool C2 8192 768      # TMA team tiles
  run $tool C5 4099 1024     # global sweep + grid barrier
  run $tool fig7a 300 96     # global sweep + second barrier + sweep 2
done
