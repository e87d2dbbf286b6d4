"""Diagnose the fused exchange with virtual ranks on one GPU: per-rank kernel
start/end (CUDA events) to see whether the ranks' kernels overlap."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
from paper_conf_asplos_zhengyzlzzzlyzs22_b200.dist import PeerExchange, ShardedPlan
from tests.harness import device_inputs
from workloads import gen, specs

world = int(sys.argv[1]) if len(sys.argv) > 1 else 2
div = int(sys.argv[2]) if len(sys.argv) > 2 else world
spec = specs.get("C5", rows=3001, cols=1024)
x = gen.generate("C5", spec)
g = A.Graph.from_spec(spec)
sms = torch.cuda.get_device_properties(0).multi_processor_count
ranks = []
for r in range(world):
    sp = ShardedPlan(g, 3001, 1024, world, r, 0, sm_count=sms // div)
    b, n = sp.row_begin, sp.row_count
    xs = {k: (v[b:b + n] if getattr(v, "ndim", 0) == 2 else v) for k, v in x.items()}
    ranks.append([sp, device_inputs(dict(spec, rows=n), xs), sp.plan.alloc_outputs(), sp.plan.alloc_workspace(),
                  torch.cuda.Stream()])
for sp, *_ in ranks:
    sp.peer = PeerExchange(sp.plan)
for sp, *_ in ranks:
    for o, *_ in ranks:
        if o is not sp:
            sp.peer.link(o.rank, o.peer)
for sp, *_ in ranks:
    d = sp.plan.describe()
    print("rank", sp.rank, "grid", d["kernels"][0]["grid"], "occ", d["kernels"][0]["occupancy_blocks_per_sm"], "regs", d["kernels"][0]["regs"])
for it in range(2):
    torch.cuda.synchronize()
    evs = []
    t0 = time.time()
    for sp, ins, outs, ws, st in ranks:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        sp.run(ins, outs, ws=ws, stream=st)
        e1.record(st)
        evs.append((e0, e1))
    torch.cuda.synchronize()
    base = evs[0][0]
    for (e0, e1), (sp, *_) in zip(evs, ranks):
        print(f"it {it} rank {sp.rank}: start {base.elapsed_time(e0):.3f} ms end {base.elapsed_time(e1):.3f} ms timed_out {sp.peer.timed_out()}")
    print("wall", time.time() - t0)
    print("fused kernel grid", ranks[0][0].plan.describe())
