#!/bin/bash
# non-portable 16-CTA clusters for <= 9 long rows vs portable 8
timeout 900 python -m pytest tests/test_parity_gpu.py -q -k "row_stream or split" 2>&1 | tail -2
for shape in "fig6b 3 4000000" "C1 8 2000000" "C1 9 2000000" "C4 8 1000003"; do
  set -- $shape
  echo -n "$1 $2x$3 K16: "; bash scripts/bench_brief.sh $1 --no-e2e --rows $2 --cols $3
  echo -n "$1 $2x$3 K8: "; ASTITCH_PORTABLE_CLUSTERS=1 bash scripts/bench_brief.sh $1 --no-e2e --rows $2 --cols $3
done
python - <<'PY'
import sys; sys.path.insert(0,'.')
import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
from workloads import specs
for c,r,cc in [("fig6b",3,4000000),("C1",9,2000000)]:
    s=specs.get(c, rows=r, cols=cc)
    p=A.Plan(A.Graph.from_spec(s), s["rows"], s["cols"], device=0)
    d=p.describe(); print(c, r, cc, d["mapping"]["split"], d["mapping"]["grid"], d["kernels"][0])
PY
