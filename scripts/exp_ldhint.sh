#!/bin/bash
# streaming-load qualifiers and vector width vs torch.add on C5's traffic
for h in default ".L1::no_allocate.L2::256B" ".L1::no_allocate.L2::128B" "none"; do
  echo "== LD_HINT $h"
  if [ "$h" = default ]; then python scripts/exp_c5_variants.py 2>&1 | grep -v torch.add; else ASTITCH_LD_HINT="$h" python scripts/exp_c5_variants.py 2>&1 | grep -v torch.add; fi
done
echo "== VEC_BYTES 32"; ASTITCH_VEC_BYTES=32 python scripts/exp_c5_variants.py 2>&1 | tail -5
echo "== VEC_BYTES 32 + L2::256B"; ASTITCH_VEC_BYTES=32 ASTITCH_LD_HINT=".L1::no_allocate.L2::256B" python scripts/exp_c5_variants.py 2>&1 | tail -5
