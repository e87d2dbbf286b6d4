"""Seeded synthetic inputs for the workload specs (shared by the CUDA path's
tests/bench and by the oracle; holds none of the method's arithmetic).

Recipe (stated again in DESIGN.md Sec. "Input recipe"):

* Every FULL tensor is drawn in row chunks of ``CHUNK_ROWS`` rows.  Chunk ``k`` of
  input ``i`` uses its own generator
  ``PCG64(SeedSequence(seed, spawn_key=(i, k)))``, so the bits of a row never
  depend on how many rows were requested or on the thread count: a reduced-row
  problem is exactly the prefix of the full-size one.
* ROWVEC / COLVEC / LENGTHS tensors use ``spawn_key=(i, 1 << 20)``.
* Gaussians are drawn as float32 ``standard_normal`` and scaled in fp32.
* bf16 tensors are the round-to-nearest-even of those fp32 values, returned as
  their raw ``uint16`` bit patterns (numpy has no bfloat16).  Both the GPU path
  and the oracle consume exactly these bits.
* Per-config distributions follow SURVEY.md Sec. 8(d) (shapes of the paper's
  BERT / Transformer / DIEN / training workloads, Table 2).
"""

from __future__ import annotations

import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np

CHUNK_ROWS = 8192
_VEC_KEY = 1 << 20

CONFIG_SEEDS = {"C1": 1, "C2": 2, "C3": 3, "C3v": 3, "C4": 4, "C5": 5, "C5int": 6,
                "fig5": 7, "fig7a": 8, "fig6a": 9, "fig6b": 10}


def f32_to_bf16_bits(a: np.ndarray) -> np.ndarray:
    """fp32 -> bf16 round-to-nearest-even, returned as uint16 bits (finite inputs)."""
    u = np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)
    return ((u + np.uint32(0x7FFF) + ((u >> np.uint32(16)) & np.uint32(1))) >> np.uint32(16)).astype(np.uint16)


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    """Exact widening of bf16 bits to fp32."""
    return (np.asarray(b, dtype=np.uint16).astype(np.uint32) << np.uint32(16)).view(np.float32)


def _gen(seed: int, i: int, k: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(np.random.SeedSequence(seed, spawn_key=(i, k))))


def _encode(a: np.ndarray, dtype: str) -> np.ndarray:
    if dtype == "F32":
        return np.ascontiguousarray(a, dtype=np.float32)
    if dtype == "BF16":
        return f32_to_bf16_bits(a)
    if dtype == "F16":
        return np.ascontiguousarray(a, dtype=np.float16)
    if dtype == "I32":
        return np.ascontiguousarray(a, dtype=np.int32)
    raise ValueError(dtype)


# --- per-config FULL-chunk draws: (generator, nrows, ncols, input name) -> fp32
def _full_chunk(cfg: str, name: str, g: np.random.Generator, n: int, c: int) -> np.ndarray:
    if cfg in ("C3", "C3v"):              # q.k logits with d=64: N(0, 8^2); x0.125 -> N(0,1)
        return g.standard_normal((n, c), dtype=np.float32) * np.float32(8.0)
    if cfg == "C4":                       # x[r,:] = mu_r + sigma_r * N(0,1)
        mu = g.uniform(-2.0, 2.0, n).astype(np.float32)
        sg = g.uniform(0.5, 2.0, n).astype(np.float32)
        z = g.standard_normal((n, c), dtype=np.float32)
        return mu[:, None] + sg[:, None] * z
    if cfg == "C5int":                    # small integers: exact products and sums
        return g.integers(-2, 3, (n, c)).astype(np.float32)
    return g.standard_normal((n, c), dtype=np.float32)


def _vec(cfg: str, name: str, g: np.random.Generator, n: int) -> np.ndarray:
    if cfg == "C2":
        if name == "gamma":
            return np.float32(1.0) + g.standard_normal(n, dtype=np.float32) * np.float32(0.1)
        return g.standard_normal(n, dtype=np.float32) * np.float32(0.1)
    if cfg == "fig7a" and name == "p2":
        return g.uniform(1.0, 2.0, n).astype(np.float32)
    return g.standard_normal(n, dtype=np.float32)


def lengths_for(spec: dict, seed: int) -> np.ndarray:
    """C3 key lengths: L ~ integers[37, 512], first = 37, last = 512."""
    rps = spec["mask"]["rows_per_segment"]
    nseg = -(-spec["rows"] // rps)
    i = [n for n, _, _ in spec["inputs"]].index(spec["mask"]["lengths"])
    g = _gen(seed, i, _VEC_KEY)
    lo, hi = min(37, spec["cols"]), spec["cols"]
    L = g.integers(lo, hi + 1, nseg)
    if nseg >= 1:
        L[0] = lo
    if nseg >= 2:
        L[-1] = hi
    return L.astype(np.int32)


def ragged_spec(spec: dict, seed: int, lengths=None) -> dict:
    """Fill in a packed varlen spec (``"segments"`` entry): batch b has
    ``heads * L_b`` rows of ``L_b`` columns, L_b drawn like C3's key lengths
    (integers[min_len, cols], first = min_len, last = cols) unless given.
    Adds seg_rows / seg_cols / elems and sets rows; the layout is the canonical
    one of include/astitch.h (pitch = L rounded up to 8 elements, segments back
    to back), described by :func:`segment_table`."""
    import copy
    s = copy.deepcopy(spec)
    seg = s["segments"]
    if "seg_rows" not in seg:
        C = int(s["cols"])
        if lengths is None:
            i = [n for n, _, _ in s["inputs"]].index(seg["table"])
            g = _gen(seed, i, _VEC_KEY)
            lo = min(int(seg.get("min_len", 1)), C)
            L = g.integers(lo, C + 1, int(seg["batches"]))
            if len(L) >= 1:
                L[0] = lo
            if len(L) >= 2:
                L[-1] = C
        else:
            L = np.asarray(lengths, dtype=np.int64)
        seg["seg_cols"] = [int(x) for x in L]
        seg["seg_rows"] = [int(seg["heads"]) * int(x) for x in L]
    seg["elems"] = int(table_elems(seg["seg_rows"], seg["seg_cols"]))
    s["rows"] = int(sum(seg["seg_rows"]))
    return s


def ragged_subset(spec: dict, seg_ids) -> dict:
    """A filled packed varlen spec restricted to the segments ``seg_ids`` (in
    order), repacked back to back.  The segments keep their generator keys
    (``seg_keys``), so their data are bit-identical to the full problem's (row
    shards by whole batches; sampled parity at full size)."""
    import copy
    s = copy.deepcopy(spec)
    seg = s["segments"]
    keys = seg.get("seg_keys", list(range(len(seg["seg_rows"]))))
    ids = [int(i) for i in seg_ids]
    seg["seg_rows"] = [seg["seg_rows"][i] for i in ids]
    seg["seg_cols"] = [seg["seg_cols"][i] for i in ids]
    seg["seg_keys"] = [keys[i] for i in ids]
    seg["elems"] = int(table_elems(seg["seg_rows"], seg["seg_cols"]))
    s["rows"] = int(sum(seg["seg_rows"]))
    return s


def segment_table(seg_rows, seg_cols) -> np.ndarray:
    """int32 [nseg, 4] {row_start, cols, pitch, offset / 8}: segments packed back
    to back, row pitch = cols rounded up to a multiple of 8 elements."""
    r = np.asarray(seg_rows, dtype=np.int64)
    c = np.asarray(seg_cols, dtype=np.int64)
    pitch = (c + 7) // 8 * 8
    row_start = np.concatenate([[0], np.cumsum(r)[:-1]])
    off = np.concatenate([[0], np.cumsum(r * pitch)[:-1]])
    return np.stack([row_start, c, pitch, off // 8], axis=1).astype(np.int32)


def table_elems(seg_rows, seg_cols) -> int:
    r = np.asarray(seg_rows, dtype=np.int64)
    c = np.asarray(seg_cols, dtype=np.int64)
    return int((r * ((c + 7) // 8 * 8)).sum())


def _generate_ragged(cfg: str, spec: dict, seed: int, threads: int) -> dict:
    seg = spec["segments"]
    table = segment_table(seg["seg_rows"], seg["seg_cols"])
    elems = seg["elems"]
    out = {}
    for i, (name, kind, dtype) in enumerate(spec["inputs"]):
        if kind == "SEGMENTS":
            out[name] = table
        elif kind == "COLVEC":
            out[name] = _encode(_vec(cfg, name, _gen(seed, i, _VEC_KEY), spec["cols"]), dtype)
        elif kind == "ROWVEC":
            out[name] = _encode(_vec(cfg, name, _gen(seed, i, _VEC_KEY), spec["rows"]), dtype)
        elif kind == "FULL":
            res = np.zeros(elems, dtype={"F32": np.float32, "BF16": np.uint16, "F16": np.float16}[dtype])

            keys = seg.get("seg_keys", list(range(len(seg["seg_rows"]))))

            def work(b, i=i, name=name, dtype=dtype, res=res, keys=keys):
                nr, nc, pitch, off8 = (int(seg["seg_rows"][b]), int(table[b, 1]), int(table[b, 2]),
                                       int(table[b, 3]))
                if nr == 0:
                    return
                a = _full_chunk(cfg, name, _gen(seed, i, int(keys[b])), nr, nc)
                res[off8 * 8: off8 * 8 + nr * pitch].reshape(nr, pitch)[:, :nc] = _encode(a, dtype)

            with ThreadPoolExecutor(max(1, threads)) as ex:
                list(ex.map(work, range(len(seg["seg_rows"]))))
            out[name] = res
        else:
            raise ValueError(kind)
    return out


def generate(cfg: str, spec: dict, seed: int | None = None, threads: int | None = None,
             row_start: int = 0, row_count: int | None = None) -> dict:
    """Inputs for ``spec`` (config family ``cfg``) as numpy arrays keyed by name.

    ``row_start``/``row_count`` select a row window of the FULL/ROWVEC inputs
    (used to draw bounded samples of the full-size problem); the window must be
    chunk-aligned at its start.
    """
    if seed is None:
        seed = CONFIG_SEEDS.get(cfg, 0)
    if spec.get("segments"):  # packed varlen: per-segment draws (generator key = segment index)
        assert row_start == 0 and row_count is None and "seg_rows" in spec["segments"], \
            "call ragged_spec first; no row windows on packed layouts"
        return _generate_ragged(cfg, spec, seed, threads or min(32, os.cpu_count() or 1))
    R, C = spec["rows"], spec["cols"]
    if row_count is None:
        row_count = R - row_start
    assert row_start % CHUNK_ROWS == 0 or row_start == 0
    threads = threads or min(32, os.cpu_count() or 1)
    out = {}
    for i, (name, kind, dtype) in enumerate(spec["inputs"]):
        if kind == "LENGTHS":
            out[name] = lengths_for(spec, seed)
        elif kind == "COLVEC":
            out[name] = _encode(_vec(cfg, name, _gen(seed, i, _VEC_KEY), C), dtype)
        elif kind == "ROWVEC":
            full = _vec(cfg, name, _gen(seed, i, _VEC_KEY), R)
            out[name] = _encode(full[row_start:row_start + row_count], dtype)
        elif kind == "FULL":
            k0 = row_start // CHUNK_ROWS
            nchunks = -(-row_count // CHUNK_ROWS)
            res = np.empty((row_count, C), dtype={"F32": np.float32, "BF16": np.uint16,
                                                   "F16": np.float16}[dtype])

            def work(j, i=i, name=name, dtype=dtype):
                n = min(CHUNK_ROWS, row_count - j * CHUNK_ROWS)
                a = _full_chunk(cfg, name, _gen(seed, i, k0 + j), n, C)
                res[j * CHUNK_ROWS: j * CHUNK_ROWS + n] = _encode(a, dtype)

            if nchunks <= 2 or threads <= 1:
                for j in range(nchunks):
                    work(j)
            else:
                with ThreadPoolExecutor(threads) as ex:
                    list(ex.map(work, range(nchunks)))
            out[name] = res
        else:
            raise ValueError(kind)
    return out
