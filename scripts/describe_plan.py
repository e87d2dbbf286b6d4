import sys, json
sys.path.insert(0, "/root/repo")
import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
from workloads import specs
dev = int(sys.argv[2]) if len(sys.argv) > 2 else 0
s = specs.get(sys.argv[1])
p = A.Plan(A.Graph.from_spec(s), s["rows"], s["cols"], device=dev)
d = p.describe()
print(sys.argv[1], json.dumps(d["kernels"]), json.dumps({k: d["mapping"][k] for k in ("team","threads","row_unroll","blocks_per_sm","reg_cap","grid")}))
