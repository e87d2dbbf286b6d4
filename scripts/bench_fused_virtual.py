"""Cost of the in-kernel exchange with virtual ranks on ONE GPU: C5 at full
size as g ranks (each plan sized for 148/g SMs, one stream per rank, the
ranks' cooperative kernels running concurrently) vs the unsharded plan on the
whole GPU.  Same total HBM traffic, so the difference is the exchange (+ the
split of the grid).  CUDA-event timing over K iterations after warm-up."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
from paper_conf_asplos_zhengyzlzzzlyzs22_b200.dist import PeerExchange, ShardedPlan
from workloads import specs

world = int(sys.argv[1]) if len(sys.argv) > 1 else 2
K = 20
spec = specs.get("C5")
R, C = spec["rows"], spec["cols"]
g = A.Graph.from_spec(spec)
dy = torch.randn(R, C, device="cuda").to(torch.bfloat16)
z = torch.randn(R, C, device="cuda").to(torch.bfloat16)
b = torch.randn(C, device="cuda")
sms = torch.cuda.get_device_properties(0).multi_processor_count

def timeit(fn):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(K):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / K * 1e3

full = A.Plan(g, R, C, device=0)
fo = full.alloc_outputs()
fws = full.alloc_workspace()
t_full = timeit(lambda: full.run([dy, z, b], fo, ws=fws))

ranks = []
for r in range(world):
    sp = ShardedPlan(g, R, C, world, r, 0, sm_count=sms // world)
    bb, n = sp.row_begin, sp.row_count
    ranks.append([sp, [dy[bb:bb + n], z[bb:bb + n], b], sp.plan.alloc_outputs(), sp.plan.alloc_workspace(),
                  torch.cuda.Stream()])
for sp, *_ in ranks:
    sp.peer = PeerExchange(sp.plan)
for sp, *_ in ranks:
    for o, *_ in ranks:
        if o is not sp:
            sp.peer.link(o.rank, o.peer)
cur = torch.cuda.current_stream()

def fused_step():
    ev = torch.cuda.Event()
    ev.record(cur)
    for sp, ins, outs, ws, st in ranks:
        st.wait_event(ev)
        sp.run(ins, outs, ws=ws, stream=st)
    for *_, st in ranks:
        e = torch.cuda.Event()
        e.record(st)
        cur.wait_event(e)

t_fused = timeit(fused_step)
ok = not any(sp.peer.timed_out() for sp, *_ in ranks)
same = all(torch.equal(ranks[0][2][1], rk[2][1]) for rk in ranks)
d1, d0 = ranks[0][2][1].double(), fo[1].double()
close = float((d1 - d0).abs().max() / d0.pow(2).mean().sqrt())
print(json.dumps({"world": world, "us_unsharded_one_kernel": round(t_full, 2), "us_fused_virtual_ranks": round(t_fused, 2),
                  "no_timeout": ok, "db_bitwise_equal_across_ranks": same, "db_max_abs_diff_over_rms_vs_unsharded": close}))
