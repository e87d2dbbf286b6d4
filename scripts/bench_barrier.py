#!/usr/bin/env python
"""Global-barrier micro-benchmark on B200 (the paper's Table 6).

A cooperative kernel containing only grid barriers (astitch_bench_barrier).
For each grid size we time (CUDA events, after warm-up) a kernel with one
barrier (the paper's "kernel consisting of only a global barrier") and the
per-barrier cost from kernels with 1 and 101 barriers.  Prints one JSON line.

    python scripts/bench_barrier.py > profiles/r01_barrier.json
"""

import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A

    dev = 0
    torch.cuda.set_device(dev)
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    ws = torch.zeros(64, dtype=torch.int32, device="cuda")  # 256 B, zeroed once
    s = torch.cuda.current_stream()

    def timed(blocks, threads, iters, reps=50):
        for _ in range(5):
            A.bench_barrier(dev, blocks, threads, iters, ws)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(reps):
            A.bench_barrier(dev, blocks, threads, iters, ws)
        e1.record(s)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) * 1e3 / reps  # us per kernel

    rows = []
    configs = [(b, 1024) for b in (20, 40, 60, 80, 100, 120, 140, 160, sms, 2 * sms)]
    configs += [(b, 256) for b in (sms, 2 * sms, 4 * sms, 8 * sms)]
    for blocks, threads in configs:
        try:
            t1 = timed(blocks, threads, 1)
            t101 = timed(blocks, threads, 101)
        except Exception as e:  # e.g. cooperative launch too large
            rows.append({"blocks": blocks, "threads": threads, "error": str(e)[:120]})
            continue
        rows.append({"blocks": blocks, "threads": threads, "kernel_us_1_barrier": round(t1, 3),
                     "per_barrier_us": round((t101 - t1) / 100, 3)})
    print(json.dumps({"what": "grid barrier micro-benchmark (Table 6 on B200)", "sms": sms,
                      "paper_v100_us": {"20": 2.53, "40": 2.53, "60": 2.59, "80": 2.59, "100": 2.66,
                                        "120": 2.66, "140": 2.69, "160": 2.72},
                      "rows": rows}))


if __name__ == "__main__":
    main()
