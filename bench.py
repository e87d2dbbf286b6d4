#!/usr/bin/env python
"""Benchmark of the stitched-subgraph hot path (BASELINE.json metric:
stitched-subgraph achieved HBM GB/s (% of 8 TB/s) and us/subgraph at 1/2/4/8 B200).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--impl reference]

Default workload: C5 = BASELINE configs[4], the training bias-gradient subgraph
on [1,048,576, 1024] bf16 (dz = dy * gelu'(z); db = col_sum(dz);
b_new = b - 2^-7 db) — the config the metric is quoted on at 1/2/4/8 GPUs, run
as ONE stitched kernel with global stitching (grid barrier).  At N > 1 the
rows are sharded contiguously (strong scaling of the fixed problem) and the
column partials are exchanged inside the stitched kernel over peer memory
(`--exchange fused`, default) or with one NCCL allreduce + epilogue
(`--exchange nccl`, also the fallback when peer access is unavailable).

A "step" is one execution of the whole subgraph (one astitch_run /
astitch_run_sharded) over the resident synthetic inputs.  Timing: W warm-up
steps, then K steps between a barrier + synchronize on both sides, CUDA events
on the launching stream, max over ranks.  C5's inputs (4.3 GB) exceed L2
(126 MB); the small configs rotate input sets (>= 4x L2).
"""

from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

WORKLOAD_NAMES = {
    "C1": "softmax fp32 [32,128]",
    "C2": "BERT-base bias+residual+LayerNorm+GELU bf16 [4096,768]",
    "C3": "Transformer attention masked softmax bf16 [64*16*512,512], lengths 37-512",
    "C4": "DIEN row standardise fp32 [2,000,000,36]",
    "C5": "bias-GELU backward + bias-grad column reduce + in-kernel SGD step, bf16 [1,048,576,1024]",
    "C3v": "Transformer attention softmax bf16, packed varlen (64 batches x 16 heads x L_b rows of L_b, L_b 37-512)",
}
def spec_name(cfg):
    from workloads import specs
    return specs.ALL[cfg]["name"]


METRIC = "stitched-subgraph achieved HBM GB/s (% of 8 TB/s) and us/subgraph"


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def _traffic(cfg):
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            d = json.load(f)
        return d.get(cfg)
    except Exception:
        return None


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    def __init__(self, device: int):
        self.device = device
        self.samples = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device),
                 "--query-gpu=clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
                 "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc is not None:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        rows = [s for s in self.samples if len(s) >= 8]
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}

        def num(x):
            try:
                return float(x)
            except Exception:
                return None
        sm = sorted(v for v in (num(r[0]) for r in rows) if v is not None)
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            for n, v in zip(names, r[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": num(rows[0][1]),
                "reasons": sorted(reasons), "samples": len(rows),
                "power_w_max": max((num(r[2]) or 0) for r in rows)}


# ---------------------------------------------------------------------- inputs
def make_inputs(cfg, spec, row_start=0, row_count=None):
    from workloads import gen
    return gen.generate(cfg, spec, row_start=row_start, row_count=row_count)


def compulsory_bytes(spec, inputs, rows=None):
    """Each input read once + each output written once; a masked FULL input
    counts only its valid prefix."""
    import numpy as np
    R = spec["rows"] if rows is None else rows
    C = spec["cols"]
    es = {"F32": 4, "BF16": 2, "F16": 2, "I32": 4}
    mask = spec.get("mask")
    valid = None
    seg = spec.get("segments")
    if seg is not None:  # packed varlen: every element of every row is valid (no padding)
        valid = int(sum(r * c for r, c in zip(seg["seg_rows"], seg["seg_cols"])))
        kinds = {"FULL": valid, "ROWVEC": R, "COLVEC": C}
        b = sum(kinds[k] * es[dt] for _, k, dt in spec["inputs"] if k in kinds)
        b += 16 * len(seg["seg_rows"])
        b += sum(kinds[_out_kind(spec, n)] * es[dt] for n, dt in spec["outputs"])
        return b
    if mask is not None:
        L = np.clip(np.asarray(inputs[mask["lengths"]], dtype=np.int64), 0, C)
        rps = mask["rows_per_segment"]
        seg = np.arange(len(L))
        nrows = np.minimum(rps, np.maximum(0, R - seg * rps))
        valid = int((L * nrows).sum())
    b = 0
    for name, kind, dt in spec["inputs"]:
        if kind == "FULL":
            b += (valid if valid is not None else R * C) * es[dt]
        elif kind == "ROWVEC":
            b += R * es[dt]
        elif kind == "COLVEC":
            b += C * es[dt]
        elif kind == "LENGTHS":
            b += 4 * len(inputs[name])
    for name, dt in spec["outputs"]:
        kind = {"FULL": (R * C), "ROWVEC": R, "COLVEC": C}
        k = _out_kind(spec, name)
        b += kind[k] * es[dt]
    return b


def _out_kind(spec, name):
    kinds = {n: k for n, k, _ in spec["inputs"]}
    for op in spec["ops"]:
        n, t = op[0], op[1]
        if t == "const":
            kinds[n] = "SCALAR"
        elif t == "unary":
            kinds[n] = kinds[op[3]]
        elif t == "binary":
            ka, kb = kinds[op[3]], kinds[op[4]]
            kinds[n] = kb if ka == "SCALAR" else ka
        elif t == "reduce":
            kinds[n] = "ROWVEC" if op[3] == "ROW" else "COLVEC"
        else:
            kinds[n] = "FULL"
    return kinds[name]


# ---------------------------------------------------------------------- oracle on the host cores
def _cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def _shard_problem(cfg, spec, x, r0, n):
    """The same graph on rows [r0, r0 + n) of a dense spec (masked specs: r0 a
    multiple of rows_per_segment, lengths re-sliced)."""
    from workloads import specs
    sspec = specs.resized(spec, rows=n)
    sx = {}
    for name, kind, _ in spec["inputs"]:
        v = x[name]
        sx[name] = v[r0:r0 + n] if kind in ("FULL", "ROWVEC") else v
    m = spec.get("mask")
    if m is not None:
        rps = m["rows_per_segment"]
        assert r0 % rps == 0
        sspec["mask"] = dict(m, rows_per_segment=min(rps, n))
        sx[m["lengths"]] = x[m["lengths"]][r0 // rps: -(-(r0 + n) // rps)]
        if n < rps:  # one partial segment: its single length
            sx[m["lengths"]] = x[m["lengths"]][r0 // rps: r0 // rps + 1]
    return sspec, sx


def oracle_on_host_cores(cfg, spec, x, target_s=15.0, reps=1, rows_cap=None, skip=0, min_shard_rows=256,
                         full_rows=None):
    """The fp64 oracle as it stands (oracle.evaluate, unmodified) on every
    host core: the rows (the method's independent units) are cut into W
    contiguous shards, W = the cores this process may run on, and each shard
    is evaluated by its own forked process (numpy pinned to one thread), the
    same data-parallel split as the GPU path's row shards.  The sample is the
    whole problem when it fits ~target_s of wall time at the pilot-measured
    rate, else its first rows (a bounded sample, stated in the result).  Wall
    time = last shard end - first shard start, median over `reps`.
    Packed varlen specs shard whole segments."""
    import multiprocessing as mp
    import statistics
    from oracle import evaluate
    cores = len(os.sched_getaffinity(0))
    ragged = bool(spec.get("segments"))
    R = spec["rows"]
    # pilot: one small slice in this process (rows/s of one core)
    if ragged:
        from workloads import gen
        nseg = len(spec["segments"]["seg_rows"])
        psub = gen.ragged_subset(spec, [0])
        px = gen.generate(cfg, psub)
        t0 = time.perf_counter()
        evaluate(psub, px)
        rate = psub["segments"]["elems"] / max(time.perf_counter() - t0, 1e-6)   # elements / s
        total = spec["segments"]["elems"]
    else:
        unit = spec["mask"]["rows_per_segment"] if spec.get("mask") else 1
        pr = min(R, max(unit, 256 if unit == 1 else unit))
        psp, pxx = _shard_problem(cfg, spec, x, 0, pr)
        t0 = time.perf_counter()
        evaluate(psp, pxx, row_chunk=2048)
        rate = pr / max(time.perf_counter() - t0, 1e-6)                          # rows / s
        total = R
    budget = rate * cores * target_s
    W = cores
    if ragged:
        # whole segments, in order, until the element budget is reached
        segs, acc = [], 0
        for i, (r, c) in enumerate(zip(spec["segments"]["seg_rows"], spec["segments"]["seg_cols"])):
            if segs and acc + r * c > budget:
                break
            segs.append(i)
            acc += r * c
        W = min(W, len(segs))
        parts = [segs[k::W] for k in range(W)]
        sample = f"segments 0-{segs[-1]} of {nseg} ({acc} valid elements)"
    else:
        rows = int(min(R, max(unit, budget), rows_cap or R))
        rows = max(unit, rows // unit * unit) if unit > 1 else max(1, rows)
        W = max(1, min(W, rows // max(unit, min_shard_rows)))
        per = -(-rows // W)
        if unit > 1:
            per = -(-per // unit) * unit
        bounds = [(r0, min(per, rows - r0)) for r0 in range(0, rows, per)]
        W = len(bounds)
        FR = full_rows or R
        sample = f"rows 0-{rows - 1} of {FR}" + (" (whole problem)" if rows == FR else "") + f", {W} row shards"

    def work(k, bar, q):
        try:
            from threadpoolctl import threadpool_limits
            threadpool_limits(1)
        except Exception:
            pass
        if ragged:
            from workloads import gen
            sspec = gen.ragged_subset(spec, parts[k])
            sx = gen.generate(cfg, sspec, threads=1)
        else:
            sspec, sx = _shard_problem(cfg, spec, x, *bounds[k])
        nb = compulsory_bytes(sspec, sx)
        for _ in range(total_reps):
            bar.wait()
            a = time.time()
            evaluate(sspec, sx, row_chunk=2048) if not ragged else evaluate(sspec, sx)
            q.put((k, a, time.time(), nb))
        bar.wait()

    total_reps = reps + skip
    ctx = mp.get_context("fork")
    bar = ctx.Barrier(W)
    q = ctx.Queue()
    procs = [ctx.Process(target=work, args=(k, bar, q)) for k in range(W)]
    for pr_ in procs:
        pr_.start()
    reps += skip
    res = [q.get() for _ in range(W * reps)]
    for pr_ in procs:
        pr_.join()
    walls, nbytes = [], 0
    for r in range(skip, reps):
        chunk = res[r * W:(r + 1) * W]
        walls.append(max(c[2] for c in chunk) - min(c[1] for c in chunk))
    nbytes = sum(c[3] for c in res[:W])
    wall = statistics.median(walls)
    return {"value": round(nbytes / wall / 1e9, 4), "unit": "GB/s", "cores": W, "kind": "oracle",
            "sample": f"{sample}; unmodified numpy fp64 oracle, one process per core; "
                      f"{wall:.2f} s wall (median of {reps - skip})",
            "cpu_model": _cpu_model(), "host_cores": cores, "bytes": int(nbytes), "wall_s": round(wall, 3)}


# ---------------------------------------------------------------------- reference arm
def run_reference(args, rank, world):
    """--impl reference: the fp64 oracle as it stands, on the host cores (one
    process per core over row shards), each step a bounded sample of the same
    workload (~2 s of wall time), median over the timed steps."""
    if rank != 0:
        return None
    cfg = args.config
    spec = _full_spec(cfg, rows=args.rows, cols=args.cols)
    if spec.get("segments"):
        x = None
    else:
        # the rows a ~2 s step can cover on this host, generated once
        from workloads import specs
        cap = {"C1": 32, "C2": 4096, "C3": 524288, "C4": 2_000_000, "C5": 262144}.get(cfg, 65536)
        cap = min(cap, spec["rows"])
        if spec.get("mask"):
            cap = max(spec["mask"]["rows_per_segment"], cap // spec["mask"]["rows_per_segment"] * spec["mask"]["rows_per_segment"])
        sub = specs.resized(spec, rows=cap) if cap < spec["rows"] else spec
        x = make_inputs(cfg, sub)
    cpu = oracle_on_host_cores(cfg, spec if x is None else _sub_or_full(spec, x), x, target_s=2.0,
                               reps=args.steps, skip=args.warmup, full_rows=spec["rows"])
    gbs = cpu["value"]
    dt = cpu["wall_s"]
    return {
        "impl": "reference", "metric": METRIC, "value": gbs, "unit": "GB/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 3),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic",
        "config": {"workload": f"{cfg}: {WORKLOAD_NAMES.get(cfg, spec_name(cfg))}", "rows": spec["rows"], "cols": spec["cols"],
                   "parallelism": f"host oracle, {cpu['cores']} processes (rank 0)"},
        "cpu_baseline": cpu,
        "e2e": {"value": gbs, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }


def _sub_or_full(spec, x):
    """The spec restricted to the rows present in x (the generated prefix)."""
    from workloads import specs
    n = len(next(v for k, v in x.items() if getattr(v, "ndim", 0) == 2))
    return spec if n == spec["rows"] else specs.resized(spec, rows=n)


def _full_spec(cfg, rows=None, cols=None):
    """The workload spec; packed varlen specs get their seeded segment layout."""
    from workloads import gen, specs
    spec = specs.get(cfg, rows=rows, cols=cols)
    if spec.get("segments"):
        spec = gen.ragged_spec(spec, gen.CONFIG_SEEDS.get(cfg, 0))
    return spec


# ---------------------------------------------------------------------- main arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C5", help="C1..C5 (BASELINE configs) or another workloads.specs entry")
    ap.add_argument("--impl", default="astitch", choices=["astitch", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--e2e-chunks", type=int, default=16,
                    help="row chunks of the pipelined host path (H2D / kernel / D2H overlap); 1 = serial")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true", help="skip the host-buffer e2e leg (ablation sweeps)")
    ap.add_argument("--flags", type=int, default=0)
    ap.add_argument("--tune", default=None, help="planner overrides (astitch_plan_ex), e.g. bps=2,unroll=2")
    ap.add_argument("--exchange", default="fused", choices=["fused", "nccl"],
                    help="N>1 column reductions: in-kernel exchange over peer memory (fused) or ncclAllReduce + epilogue")
    ap.add_argument("--eager", action="store_true", help="time eager launches instead of a CUDA graph")
    ap.add_argument("--rows", type=int, default=None, help="override the config's rows (experiments)")
    ap.add_argument("--cols", type=int, default=None, help="override the config's cols (experiments)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        line = run_reference(args, rank, world)
        if line is not None:
            print(json.dumps(line), flush=True)
        return

    import numpy as np
    import torch
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
    from paper_conf_asplos_zhengyzlzzzlyzs22_b200.dist import Comm, ShardedPlan
    from tests.harness import to_torch
    from workloads import specs

    torch.cuda.set_device(local_rank)
    dev = local_rank
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", dev))

    cfg = args.config
    spec = _full_spec(cfg, rows=args.rows, cols=args.cols)
    ragged = bool(spec.get("segments"))
    if ragged and world > 1:
        # packed varlen: shard whole segments (independent problems, no
        # communication), contiguous ranges balanced by packed bytes
        from workloads import gen
        seg = spec["segments"]
        w = np.asarray(seg["seg_rows"], dtype=np.float64) * (np.asarray(seg["seg_cols"]) + 7) // 8 * 8
        cut = np.searchsorted(np.cumsum(w), np.sum(w) * np.arange(1, world) / world)
        bounds = [0] + [int(c) + 1 for c in cut] + [len(w)]
        spec = gen.ragged_subset(spec, list(range(bounds[rank], max(bounds[rank], bounds[rank + 1]))))
    R, C = spec["rows"], spec["cols"]
    graph = A.Graph.from_spec(spec)
    comm = Comm.from_process_group(dev) if world > 1 else None
    row_range = None
    if spec.get("mask") and world > 1:
        # masked batches: whole segments per rank, balanced by compulsory bytes
        from paper_conf_asplos_zhengyzlzzzlyzs22_b200.dist import mask_row_ranges
        from workloads import gen as _gen
        L = _gen.lengths_for(spec, _gen.CONFIG_SEEDS.get(cfg, 0))
        es = {"F32": 4, "BF16": 2, "F16": 2}
        ein = sum(es[d] for _, k, d in spec["inputs"] if k == "FULL")
        eout = sum(es[d] for n, d in spec["outputs"] if _out_kind(spec, n) == "FULL")
        row_range = mask_row_ranges(L, spec["mask"]["rows_per_segment"], C, R, world, ein, eout)[rank]
    sp = ShardedPlan(graph, R, C, 1 if ragged else world, 0 if ragged else rank, dev, comm=comm, flags=args.flags,
                     tune=args.tune, row_range=row_range)
    exchange = "none"
    if world > 1 and not ragged and sp.needs_exchange():
        exchange = "ncclAllReduce + epilogue"
        if args.exchange == "fused":
            from paper_conf_asplos_zhengyzlzzzlyzs22_b200.dist import PeerExchange
            try:
                sp.peer = PeerExchange.from_process_group(sp.plan)
                exchange = "in-kernel over peer memory (astitch_run_fused)"
            except Exception as e:  # pragma: no cover - needs a multi-GPU box
                print(f"[bench] fused exchange unavailable ({e}); using NCCL", file=sys.stderr)
                sp.peer = None
            # every rank must take the same path (a fused kernel waits for all peers)
            ok = torch.tensor([1.0 if sp.peer is not None else 0.0], device=f"cuda:{dev}")
            dist.all_reduce(ok, op=dist.ReduceOp.MIN)
            if float(ok.item()) < 1.0:
                sp.peer = None
                exchange = "ncclAllReduce + epilogue (peer mapping failed on a rank)"
    plan = sp.plan
    desc = plan.describe()
    r0, nr = sp.row_begin, sp.row_count

    # seeded inputs of this rank's row slice, resident in HBM
    t_gen = time.time()
    x = make_inputs(cfg, spec) if ragged else \
        make_inputs(cfg, spec, row_start=r0 if r0 % 8192 == 0 else 0, row_count=nr) if r0 % 8192 == 0 \
        else {k: v[r0:r0 + nr] if getattr(v, "ndim", 0) == 2 else v
              for k, v in make_inputs(cfg, spec).items()}
    if spec.get("mask") and world > 1:  # the rank's slice of the per-segment lengths
        rps = spec["mask"]["rows_per_segment"]
        assert r0 % rps == 0, "masked configs shard by whole segments"
        ln = spec["mask"]["lengths"]
        x[ln] = x[ln][r0 // rps: -(-(r0 + nr) // rps)]
    shard_spec = dict(spec, rows=nr)
    nbytes = compulsory_bytes(shard_spec, x, rows=nr)
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    nsets = 1 if nbytes >= 4 * l2 else min(1024, -(-4 * l2 // max(nbytes, 1)))
    dev_in = [[to_torch(x[n], d, None).to(f"cuda:{dev}") for n, _, d in spec["inputs"]] for _ in range(nsets)]
    dev_out = [plan.alloc_outputs() for _ in range(nsets)]
    ws = plan.alloc_workspace()
    gen_s = time.time() - t_gen
    stream = torch.cuda.current_stream()

    def step(i):
        sp.run(dev_in[i % nsets], dev_out[i % nsets], ws=ws)

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    if sp.peer is not None:
        exchange = check_fused_exchange(sp, dev_in[0], plan, ws, exchange)

    # copy-kernel ceiling on the same number of bytes (practical roofline),
    # timed like the step: K launches of the same-bytes copy kernel captured
    # in a CUDA graph over the same number of rotating buffer sets, so the
    # small configs' launch / ramp latency is in the ceiling too
    half = (nbytes // 2) // 16 * 16
    cbufs = [(torch.empty(half, dtype=torch.uint8, device=f"cuda:{dev}"),
              torch.empty(half, dtype=torch.uint8, device=f"cuda:{dev}")) for _ in range(nsets)]
    for i in range(3):
        A.bench_copy(dev, *cbufs[i % nsets], half)
    torch.cuda.synchronize()
    ce0, ce1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    try:
        cgraph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(cgraph):
            for i in range(args.steps):
                A.bench_copy(dev, *cbufs[i % nsets], half)
        cgraph.replay()
        torch.cuda.synchronize()
        ce0.record(stream)
        cgraph.replay()
        ce1.record(stream)
    except Exception:  # pragma: no cover
        torch.cuda.synchronize()
        ce0.record(stream)
        for i in range(args.steps):
            A.bench_copy(dev, *cbufs[i % nsets], half)
        ce1.record(stream)
    torch.cuda.synchronize()
    copy_us = ce0.elapsed_time(ce1) * 1e3 / args.steps
    copy_gbs = 2 * half / (copy_us * 1e-6) / 1e9
    del cbufs

    # K steps captured once into a CUDA graph (removes host launch overhead,
    # which otherwise dominates the us-scale configs); eager if capture fails
    graph = None
    if not args.eager:
        try:
            graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(graph):
                for i in range(args.steps):
                    step(i)
            graph.replay()
            torch.cuda.synchronize()
        except Exception as e:  # pragma: no cover
            print(f"[bench] graph capture failed ({e}); timing eagerly", file=sys.stderr)
            graph = None
            torch.cuda.synchronize()

    # ---- timed region
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(dev) as clk:
        e0.record(stream)
        if graph is not None:
            graph.replay()
        else:
            for i in range(args.steps):
                step(i)
        e1.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([ms], device=f"cuda:{dev}")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        tb = torch.tensor([float(nbytes)], device=f"cuda:{dev}", dtype=torch.float64)
        dist.all_reduce(tb)
        total_bytes = float(tb.item())
    else:
        total_bytes = float(nbytes)
    ms_step = ms / args.steps
    gbs = total_bytes / (ms_step * 1e-3) / 1e9

    # per-launch duration of the dominant kernel (the stitched kernel; at N=1
    # the step IS the one kernel; at N>1 time the rank-local stitched kernel)
    if world > 1:
        kin, kout = dev_in[0], dev_out[0]
        k0, k1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        for _ in range(3):
            plan.run(kin, kout, ws=ws)
        k0.record(stream)
        for _ in range(args.steps):
            plan.run(kin, kout, ws=ws)
        k1.record(stream)
        torch.cuda.synchronize()
        kern_ms = k0.elapsed_time(k1) / args.steps
    else:
        kern_ms = ms_step
    peak, peak_src = _peaks()
    achieved = nbytes / (kern_ms * 1e-3) / 1e9

    # C5's traffic mix (2 bf16 reads : 1 bf16 write) runs faster than a copy:
    # report torch.add over the same element count as the mix ceiling
    mix = None
    if cfg == "C5" and world == 1:
        n_el = nr * C
        xa = torch.empty(n_el, dtype=torch.bfloat16, device=f"cuda:{dev}").normal_()
        xb = torch.empty_like(xa).normal_()
        xc = torch.empty_like(xa)
        for _ in range(3):
            torch.add(xa, xb, out=xc)
        m0, m1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        m0.record(stream)
        for _ in range(5):
            torch.add(xa, xb, out=xc)
        m1.record(stream)
        torch.cuda.synchronize()
        mix_gbs = 3 * 2 * n_el * 5 / (m0.elapsed_time(m1) * 1e-3) / 1e9
        mix = {"gbs": round(mix_gbs, 1), "frac": round(achieved / mix_gbs, 4),
               "how": "torch.add bf16 over the same element count (2 reads : 1 write, C5's mix)"}
        del xa, xb, xc
        torch.cuda.empty_cache()

    # eager per-call latency (no CUDA graph; host launch cost included):
    # back-to-back pre-marshalled astitch_run calls (Plan.bind), rank-local
    eager_us = None
    if world == 1:
        fns = [plan.bind(dev_in[i], dev_out[i], ws=ws) for i in range(min(nsets, args.steps))]
        for f in fns[:3]:
            f()
        torch.cuda.synchronize()
        q0, q1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        q0.record(stream)
        for i in range(args.steps):
            fns[i % len(fns)]()
        q1.record(stream)
        torch.cuda.synchronize()
        eager_us = q0.elapsed_time(q1) * 1e3 / args.steps
        del fns

    # ---- e2e through the C ABI with pinned HOST buffers (H2D + kernel + D2H)
    host_in = [to_torch(x[n], d, None).pin_memory() for n, _, d in spec["inputs"]]
    host_out = [torch.empty(t.shape, dtype=t.dtype).pin_memory() for t in dev_out[0]]
    h2d = sum(t.numel() * t.element_size() for t in host_in)
    d2h = sum(t.numel() * t.element_size() for t in host_out)
    if world > 1:
        e2e_run = None
    if args.no_e2e:
        args.e2e_steps = 0
    for _ in range(2 if args.e2e_steps else 0):
        plan.run_host(host_in, host_out, dev_in[0], dev_out[0], ws=ws, chunks=args.e2e_chunks) if world == 1 else \
            _sharded_host(sp, host_in, host_out, dev_in[0], dev_out[0], ws)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    h0, h1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    h0.record(stream)
    for _ in range(args.e2e_steps):
        if world == 1:
            plan.run_host(host_in, host_out, dev_in[0], dev_out[0], ws=ws, chunks=args.e2e_chunks)
        else:
            _sharded_host(sp, host_in, host_out, dev_in[0], dev_out[0], ws)
    h1.record(stream)
    torch.cuda.synchronize()
    e2e_ms = h0.elapsed_time(h1) / max(args.e2e_steps, 1)
    if world > 1:
        t = torch.tensor([e2e_ms], device=f"cuda:{dev}")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())
    e2e_gbs = total_bytes / (e2e_ms * 1e-3) / 1e9 if args.e2e_steps else None
    # the PCIe floor of that step: the same H2D bytes alone, the same D2H bytes alone
    link = None
    if args.e2e_steps:
        def _copy_ms(pairs):
            c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            c0.record(stream)
            for dst_, src_ in pairs:
                dst_.copy_(src_, non_blocking=True)
            c1.record(stream)
            torch.cuda.synchronize()
            return c0.elapsed_time(c1)
        _copy_ms(list(zip(dev_in[0], host_in)))
        h2d_ms = _copy_ms(list(zip(dev_in[0], host_in)))
        d2h_ms = _copy_ms(list(zip(host_out, dev_out[0])))
        # both directions at once (what the pipelined step overlaps)
        side = torch.cuda.Stream(device=f"cuda:{dev}")
        b0, b1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        b0.record(stream)
        side.wait_event(b0)
        for dst_, src_ in zip(dev_in[0], host_in):
            dst_.copy_(src_, non_blocking=True)
        with torch.cuda.stream(side):
            for dst_, src_ in zip(host_out, dev_out[0]):
                dst_.copy_(src_, non_blocking=True)
        stream.wait_stream(side)
        b1.record(stream)
        torch.cuda.synchronize()
        bidir_ms = b0.elapsed_time(b1)
        floor = max(h2d_ms, d2h_ms, bidir_ms)
        link = {"h2d_gbs": round(h2d / (h2d_ms * 1e-3) / 1e9, 2), "d2h_gbs": round(d2h / (d2h_ms * 1e-3) / 1e9, 2),
                "bidir_ms": round(bidir_ms, 3), "floor_ms": round(floor, 3),
                "frac_of_floor": round(floor / e2e_ms, 4)}

    # ---- oracle on the host cores (rank 0, N=1): the whole problem (or a
    # bounded sample of its rows) over one process per host core
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = oracle_on_host_cores(cfg, spec, x, target_s=15.0, reps=3 if cfg in ("C1", "C2") else 1)

    if rank == 0:
        clocks = clk.summary()
        line = {
            "metric": METRIC, "value": round(gbs, 2), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 6),
            "higher_is_better": True, "scaling": "strong" if world > 1 else "strong",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"{cfg}: {WORKLOAD_NAMES.get(cfg, spec_name(cfg))}", "rows": R, "cols": C, "global_batch": R,
                       "io_dtype": "bf16" if any(d == "BF16" for _, _, d in spec["inputs"]) else "f32",
                       "parallelism": f"dp{world} contiguous row shards" + (f", column totals exchanged {exchange}" if exchange != "none" else ""),
                       "l2": ("inputs > L2 (%.2f GB per rank vs %d MB L2)" % (nbytes / 1e9, l2 // 2**20)) if nsets == 1
                       else f"{nsets} rotating input sets >= 4x L2",
                       "timing": "cuda_graph_replay" if graph is not None else "eager",
                       "template": desc["mapping"]["template"] + ("/tma_sweep" if desc["mapping"].get("tma_sweep") else "")
                                   + ("/tma_team" if desc["mapping"].get("tma_team") else ""),
                       "grid": desc["kernels"][0]["grid"],
                       "threads": desc["mapping"]["threads"], "regs": desc["kernels"][0]["regs"],
                       "tuning": desc.get("tuning") or None, "flags": args.flags or None},
            "us_per_subgraph": round(ms_step * 1e3, 3),
            "eager_us_per_call": round(eager_us, 3) if eager_us is not None else None,
            "pct_of_8TBps": round(100.0 * gbs / world / 8000.0, 2),
            "compulsory_bytes_per_step": int(total_bytes),
            "copy_kernel_gbs": round(copy_gbs, 1),
            "copy_kernel_us": round(copy_us, 3),
            "pct_of_copy_kernel": round(100.0 * achieved / copy_gbs, 2),
            "roofline": {"bound": "hbm", "achieved": round(achieved, 2), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "traffic": _traffic(cfg),
                         "peak_source": peak_src, "kernel": desc["kernels"][0]["name"],
                         "kernel_us": round(kern_ms * 1e3, 3),
                         "algorithmic_bytes_per_launch": int(nbytes), "mix_ceiling": mix},
            "e2e": None if e2e_gbs is None else {"value": round(e2e_gbs, 3), "unit": "GB/s", "h2d_bytes_per_step": int(h2d),
                    "d2h_bytes_per_step": int(d2h), "ms_per_step": round(e2e_ms, 3),
                    "api": "astitch_run_host_pipelined" if (world == 1 and args.e2e_chunks > 1) else
                           ("astitch_run_host" if world == 1 else "astitch_run_sharded_host"),
                    "chunks": args.e2e_chunks if world == 1 else 1, "pcie": link},
            "gpu_launches": int(args.steps * sp.kernels_per_run()),
            "clocks": clocks,
            "cpu_baseline": cpu,
            "input_gen_s": round(gen_s, 1),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def check_fused_exchange(sp, inputs, plan, ws, exchange):
    """N>1 safety net for the in-kernel exchange: run the step once fused and
    once through ncclAllReduce + epilogue on the same inputs and compare every
    output (the fused combine sums the ranks in a fixed order, NCCL in its own:
    equal within fp32 reassociation).  A bounded-wait timeout or a mismatch on
    any rank switches every rank to the NCCL exchange."""
    import torch
    import torch.distributed as dist
    out_f, out_n = plan.alloc_outputs(), plan.alloc_outputs()
    sp.run(inputs, out_f, ws=ws)
    torch.cuda.synchronize()
    bad = 1.0 if sp.peer.timed_out() else 0.0
    peer, sp.peer = sp.peer, None
    sp.run(inputs, out_n, ws=ws)
    torch.cuda.synchronize()
    sp.peer = peer
    for a, b in zip(out_f, out_n):
        a, b = a.float(), b.float()
        scale = float(b.pow(2).mean().sqrt()) if b.numel() else 0.0
        if not bool(torch.isfinite(a).all()) or float((a - b).abs().max()) > 1e-5 * max(scale, 1e-30) + 1e-30:
            bad = 1.0
    flag = torch.tensor([bad], device=out_f[0].device)
    dist.all_reduce(flag, op=dist.ReduceOp.MAX)
    if float(flag.item()) > 0:
        print("[bench] fused exchange failed its check against NCCL; using NCCL", file=sys.stderr)
        sp.peer = None
        return "ncclAllReduce + epilogue (fused exchange failed its check)"
    return exchange + ", checked against NCCL"


def _sharded_host(sp, host_in, host_out, dev_in, dev_out, ws):
    """Sharded e2e step through the C ABI (astitch_run_sharded_host): H2D of
    this rank's inputs, the fused / NCCL sharded run, D2H of its outputs."""
    sp.run_host(host_in, host_out, dev_in, dev_out, ws=ws)


if __name__ == "__main__":
    main()
