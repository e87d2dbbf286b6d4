"""fp64 op-by-op CPU oracle (TEST INFRASTRUCTURE ONLY; see evaluator.py header).

Importable only from tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs.  Parity status of every function is in
DESIGN.md Sec. "Oracle pins"."""
from .evaluator import evaluate, evaluate_columns, evaluate_rows, widen  # noqa: F401
