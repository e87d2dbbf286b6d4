"""GPU parity of packed varlen rows (astitch_graph_segments):
the stitched row-team kernel over a segment table against the fp64 oracle's
per-segment evaluation, element by element on the valid elements, plus the
guarantee that nothing outside a row's 16-byte chunks is written."""

import numpy as np
import pytest

from oracle import evaluate
from tests.harness import check_close, from_torch, spec_tol, to_torch
from workloads import gen, specs

pytestmark = pytest.mark.gpu



def _spec(lengths, heads=2, base="C3v", seg_rows=None):
    s = specs.get(base)
    s["segments"]["heads"] = heads
    if seg_rows is not None:
        s["segments"]["seg_rows"] = list(seg_rows)
        s["segments"]["seg_cols"] = list(lengths)
    return gen.ragged_spec(s, 3, lengths=list(lengths))


def _valid_index(spec, x, E):
    """(valid element indices, written-tail indices = cols..ceil_E(cols) of each row)."""
    t = x[spec["segments"]["table"]]
    R = spec["rows"]
    valid, tail = [], []
    for s in range(t.shape[0]):
        r0, c, pitch, off = int(t[s, 0]), int(t[s, 1]), int(t[s, 2]), 8 * int(t[s, 3])
        r1 = int(t[s + 1, 0]) if s + 1 < t.shape[0] else R
        rows = np.arange(r1 - r0)[:, None] * pitch + off
        valid.append((rows + np.arange(c)[None, :]).ravel())
        ce = -(-c // E) * E
        tail.append((rows + np.arange(c, ce)[None, :]).ravel())
    return np.concatenate(valid), np.concatenate(tail)


def _run(spec, x, fill, tune=None):
    import torch
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
    g = A.Graph.from_spec(spec)
    plan = A.Plan(g, spec["rows"], spec["cols"], device=torch.cuda.current_device(), tune=tune)
    ins = [to_torch(x[n], d) for n, _, d in spec["inputs"]]
    outs = plan.alloc_outputs()
    for o in outs:
        o.view(torch.uint8).fill_(fill)
    plan.run(ins, outs)
    torch.cuda.synchronize()
    return plan, outs


def _check(spec, x, E=8, tune=None):
    import torch
    plan, outs = _run(spec, x, 0xFF, tune=tune)
    ref = evaluate(spec, x)
    valid, tail = _valid_index(spec, x, E)
    for (name, dt), o in zip(spec["outputs"], outs):
        r = ref[name]
        if r.shape == (spec["segments"]["elems"],):
            g = from_torch(o)
            check_close(g[valid], r[valid], dt, spec_tol(spec), name=f"{spec['name']}:{name}")
            assert np.all(g[tail] == 0.0), "partial chunk tail must be written as 0"
            # every element outside the written chunks keeps the fill pattern
            raw = o.view(torch.uint8).cpu().numpy().reshape(o.numel(), -1)
            untouched = np.ones(o.numel(), dtype=bool)
            untouched[valid] = False
            untouched[tail] = False
            assert np.all(raw[untouched] == 0xFF), "wrote outside a row's chunks"
        else:
            check_close(from_torch(o), r, dt, spec_tol(spec), name=f"{spec['name']}:{name}")
    return plan


@pytest.mark.parametrize("lengths,heads", [([37, 1, 8, 9, 64, 511, 512, 200], 2),
                                           ([512] * 3, 4), ([1, 2, 3, 4, 5, 6, 7], 3),
                                           ([100, 300, 37], 40)])
def test_ragged_softmax_parity(lengths, heads):
    spec = _spec(lengths, heads)
    x = gen.generate("C3v", spec)
    plan = _check(spec, x)
    assert plan.describe()["kernel_count"] == 1


def test_ragged_empty_segments():
    """Segments with zero rows between non-empty ones (row_start repeats)."""
    spec = _spec([64, 9, 300, 17], seg_rows=[5, 0, 7, 0])
    x = gen.generate("C3v", spec)
    _check(spec, x)


def test_ragged_layernorm_f32_and_rowvec_output():
    """fp32 I/O (16-byte chunks of 4 elements inside an 8-element pitch) and a
    ROWVEC output: L2 row normalisation over variable-length rows."""
    base = {
        "name": "ragged_l2norm_f32", "rows": None, "cols": 256,
        "inputs": [("x", "FULL", "F32"), ("S", "SEGMENTS", "I32")], "mask": None,
        "segments": {"table": "S", "batches": 6, "heads": 5, "min_len": 3},
        "ops": [("sq", "binary", "MUL", "x", "x"), ("ss", "reduce", "SUM", "ROW", "sq"),
                ("eps", "const", 1e-6), ("se", "binary", "ADD", "ss", "eps"),
                ("r", "unary", "RSQRT", "se"), ("rb", "broadcast", "ROW", "r"),
                ("o", "binary", "MUL", "x", "rb"), ("mx", "reduce", "RMAX", "ROW", "o")],
        "outputs": [("o", "F32"), ("ss", "F32"), ("mx", "F32")],
    }
    spec = gen.ragged_spec(base, 11, lengths=[3, 4, 5, 13, 255, 256])
    x = gen.generate("fig6a", spec)
    _check(spec, x, E=4)


def test_ragged_full_c3v_sampled_segments():
    """Full C3v (64 batches x 16 heads, lengths 37..512 from C3's seed): the
    GPU runs the whole packed problem; the oracle checks segments 0, 1, 31, 63
    (repacked subsets keep their bits)."""
    import torch
    spec = gen.ragged_spec(specs.get("C3v"), 3)
    x = gen.generate("C3v", spec)
    plan, outs = _run(spec, x, 0)
    got = from_torch(outs[0])
    t = x["S"]
    ids = [0, 1, 31, 63]
    sub = gen.ragged_subset(spec, ids)
    xs = gen.generate("C3v", sub)
    ref = evaluate(sub, xs)["p"]
    ts = xs["S"]
    for j, b in enumerate(ids):
        nr, c = spec["segments"]["seg_rows"][b], spec["segments"]["seg_cols"][b]
        g = got[8 * t[b, 3]: 8 * t[b, 3] + nr * t[b, 2]].reshape(nr, t[b, 2])[:, :c]
        r = ref[8 * ts[j, 3]: 8 * ts[j, 3] + nr * ts[j, 2]].reshape(nr, ts[j, 2])[:, :c]
        check_close(g, r, "BF16", spec_tol(spec), name=f"C3v seg {b}")
    del torch
