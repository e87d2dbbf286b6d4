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


# ---------------------------------------------------------------------- reference arm
def run_reference(args, rank, world):
    """--impl reference: the fp64 oracle as it stands, on the host cores, on a
    bounded row sample of the same workload (each step one sample)."""
    if rank != 0:
        return None
    import numpy as np  # noqa: F401
    from oracle import evaluate
    from workloads import specs
    cfg = args.config
    spec_full = _full_spec(cfg)
    if spec_full.get("segments"):  # packed varlen: a bounded subset of whole segments
        from workloads import gen
        spec = gen.ragged_subset(spec_full, list(range(4)))
        x = make_inputs(cfg, spec)
        return _reference_line(args, world, cfg, spec, spec_full, x)
    sample_rows = {"C1": 32, "C2": 4096, "C3": 8192, "C4": 200_000, "C5": 16384}.get(cfg, 4096)
    spec = specs.get(cfg, rows=min(sample_rows, spec_full["rows"]))
    if spec.get("mask"):
        spec["mask"]["rows_per_segment"] = min(spec["mask"]["rows_per_segment"], spec["rows"])
    x = make_inputs(cfg, spec)
    return _reference_line(args, world, cfg, spec, spec_full, x)


def _full_spec(cfg, rows=None, cols=None):
    """The workload spec; packed varlen specs get their seeded segment layout."""
    from workloads import gen, specs
    spec = specs.get(cfg, rows=rows, cols=cols)
    if spec.get("segments"):
        spec = gen.ragged_spec(spec, gen.CONFIG_SEEDS.get(cfg, 0))
    return spec


def _reference_line(args, world, cfg, spec, spec_full, x):
    from oracle import evaluate
    nbytes = compulsory_bytes(spec, x)
    for _ in range(args.warmup):
        evaluate(spec, x)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        evaluate(spec, x)
    dt = (time.perf_counter() - t0) / args.steps
    gbs = nbytes / dt / 1e9
    sample = f"{spec['rows']} of {spec_full['rows']} rows x {spec['cols']} cols per step"
    if spec.get("segments"):
        sample = (f"segments 0-{len(spec['segments']['seg_rows']) - 1} of {len(spec_full['segments']['seg_rows'])} "
                  f"({spec['rows']} of {spec_full['rows']} packed rows) per step")
    return {
        "impl": "reference", "metric": METRIC, "value": round(gbs, 4), "unit": "GB/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 3),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic",
        "config": {"workload": f"{cfg}: {WORKLOAD_NAMES.get(cfg, spec_name(cfg))}", "rows": spec["rows"], "cols": spec["cols"],
                   "parallelism": "host oracle (rank 0)"},
        "cpu_baseline": {"value": round(gbs, 4), "unit": "GB/s", "cores": 1, "kind": "oracle", "sample": sample},
        "e2e": {"value": round(gbs, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }


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
    sp = ShardedPlan(graph, R, C, 1 if ragged else world, 0 if ragged else rank, dev, comm=comm, flags=args.flags, tune=args.tune)
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

    # copy-kernel ceiling on the same number of bytes (practical roofline)
    half = (nbytes // 2) // 16 * 16
    src = torch.empty(half, dtype=torch.uint8, device=f"cuda:{dev}")
    dst = torch.empty_like(src)
    for _ in range(3):
        A.bench_copy(dev, src, dst, half)
    ce0, ce1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ce0.record(stream)
    for _ in range(10):
        A.bench_copy(dev, src, dst, half)
    ce1.record(stream)
    torch.cuda.synchronize()
    copy_gbs = 2 * half * 10 / (ce0.elapsed_time(ce1) * 1e-3) / 1e9
    del src, dst

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

    # ---- oracle on the host cores: bounded sample of the same workload (rank 0, N=1)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        from oracle import evaluate
        if ragged:  # whole segments 0-7 (bit-identical to the full problem's)
            from workloads import gen
            sspec = gen.ragged_subset(spec, list(range(min(8, len(spec["segments"]["seg_rows"])))))
            sx = make_inputs(cfg, sspec)
        else:
            srows = {"C1": 32, "C2": 4096, "C3": 8192, "C4": 400_000, "C5": 131_072}.get(cfg, 4096)
            sspec = specs.get(cfg, rows=min(srows, R))
            if sspec.get("mask"):
                sspec["mask"]["rows_per_segment"] = min(sspec["mask"]["rows_per_segment"], sspec["rows"])
            sx = {k: (v[: sspec["rows"]] if getattr(v, "ndim", 0) == 2 else v) for k, v in x.items()}
            if sspec.get("mask"):
                sx[sspec["mask"]["lengths"]] = x[spec["mask"]["lengths"]][: -(-sspec["rows"] // sspec["mask"]["rows_per_segment"])]
        reps = 3 if cfg in ("C1", "C2") else 1
        t0 = time.perf_counter()
        for _ in range(reps):
            evaluate(sspec, sx)
        cdt = (time.perf_counter() - t0) / reps
        cb = compulsory_bytes(sspec, sx)
        cpu = {"value": round(cb / cdt / 1e9, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": f"{sspec['rows']} of {R} rows x {C} cols (numpy fp64, {cdt:.2f} s)"}

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
                       "template": desc["mapping"]["template"], "grid": desc["kernels"][0]["grid"],
                       "threads": desc["mapping"]["threads"], "regs": desc["kernels"][0]["regs"],
                       "tuning": desc.get("tuning") or None, "flags": args.flags or None},
            "us_per_subgraph": round(ms_step * 1e3, 3),
            "eager_us_per_call": round(eager_us, 3) if eager_us is not None else None,
            "pct_of_8TBps": round(100.0 * gbs / world / 8000.0, 2),
            "compulsory_bytes_per_step": int(total_bytes),
            "copy_kernel_gbs": round(copy_gbs, 1),
            "pct_of_copy_kernel": round(100.0 * achieved / copy_gbs, 2),
            "roofline": {"bound": "hbm", "achieved": round(achieved, 2), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "traffic": _traffic(cfg),
                         "peak_source": peak_src, "kernel": desc["kernels"][0]["name"],
                         "kernel_us": round(kern_ms * 1e3, 3),
                         "algorithmic_bytes_per_launch": int(nbytes), "mix_ceiling": mix},
            "e2e": None if e2e_gbs is None else {"value": round(e2e_gbs, 3), "unit": "GB/s", "h2d_bytes_per_step": int(h2d),
                    "d2h_bytes_per_step": int(d2h), "ms_per_step": round(e2e_ms, 3),
                    "api": "astitch_run_host_pipelined" if (world == 1 and args.e2e_chunks > 1) else
                           ("astitch_run_host" if world == 1 else "torch H2D/D2H + astitch_run_sharded"),
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
    """Sharded e2e step: H2D of this rank's inputs, astitch_run_sharded, D2H."""
    for h, d in zip(host_in, dev_in):
        d.copy_(h, non_blocking=True)
    sp.run(dev_in, dev_out, ws=ws)
    for h, d in zip(host_out, dev_out):
        h.copy_(d, non_blocking=True)


if __name__ == "__main__":
    main()
