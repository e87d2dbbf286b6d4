"""Fused sharded run, process plumbing (NEXT f1) on one GPU: two processes
(gloo world 2) each create their exchange buffer, all-gather the CUDA IPC
handles and map the other rank's buffer (PeerExchange.from_process_group).
The in-kernel exchange itself is covered by test_fused_exchange_virtual_ranks
(two processes' cooperative kernels would time-slice on one GPU without MPS,
so a cross-process run needs one GPU per rank)."""

import os
import socket

import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    import torch
    import torch.distributed as dist
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
        from paper_conf_asplos_zhengyzlzzzlyzs22_b200.dist import PeerExchange, ShardedPlan
        from workloads import specs
        spec = specs.get("C5", rows=4001, cols=256)
        sp = ShardedPlan(A.Graph.from_spec(spec), 4001, 256, world, rank, 0)
        x = PeerExchange.from_process_group(sp.plan)
        q.put((rank, len(x.ipc_handle), any(x.ipc_handle), x.timed_out()))
        dist.barrier()
    except Exception as e:  # pragma: no cover
        q.put((rank, "error", repr(e), None))
    finally:
        dist.destroy_process_group()


def test_peer_ipc_handles_open_across_processes():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    for rank, n, nonzero, timed_out in res:
        assert n == 64 and nonzero is True and timed_out is False, res
