"""B200-native AStitch: memory-intensive subgraphs as ONE stitched kernel.

Public API (thin ctypes binding of include/astitch.h, libastitch.so):

    g = Graph.from_spec(spec)                 # or Graph().input/unary/binary/reduce/broadcast/output
    p = Plan(g, rows, cols, device=0)         # astitch_plan: classify -> dominants -> mapping -> NVRTC sm_100a
    p.run(inputs, outputs)                    # astitch_run on the current CUDA stream
    p.describe()                              # schemes, mapping, grid, registers, kernel count

Multi-GPU row sharding lives in ``.dist``.
"""

from ._lib import (FLAG_FORCE_GLOBAL, FLAG_LAUNCH_CHECK, FLAG_NO_COMPILE, FLAG_NO_PACK,  # noqa: F401
                   FLAG_FORCE_SPLIT, FLAG_NO_PREFETCH, FLAG_NO_SPLIT, FLAG_NO_TMA,
                   FLAG_STRICT_SINGLE_KERNEL, FLAG_NO_PDL, FLAG_DEBUG_BARRIER, LIB_PATH,
                   AstitchError)
from .api import (Graph, Plan, bench_barrier, bench_copy, plan, segments_layout, set_cache_dir,  # noqa: F401
                  shard_rows)

__version__ = "0.2.0"
