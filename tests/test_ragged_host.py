"""Packed varlen rows (astitch_graph_segments, the paper's
irregular shapes P:L157-L159) on the host: the oracle's per-segment evaluation
pinned against the masked dense formulation and closed forms, the canonical
segment-table layout of the C helper, and the planner / codegen decisions."""

import numpy as np
import pytest

import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
from oracle import evaluate
from workloads import gen, specs


def _spec(lengths, heads=2, base="C3v"):
    s = specs.get(base)
    s["segments"]["heads"] = heads
    return gen.ragged_spec(s, 3, lengths=list(lengths))


def test_segment_table_canonical_layout():
    rows, cols = [3, 0, 5, 2], [37, 9, 8, 1]
    t = gen.segment_table(rows, cols)
    # row starts, lengths, pitch = ceil8(cols), offsets back to back (in units of 8)
    assert t[:, 0].tolist() == [0, 3, 3, 8]
    assert t[:, 1].tolist() == cols
    assert t[:, 2].tolist() == [40, 16, 8, 8]
    assert (t[:, 3] * 8).tolist() == [0, 120, 120, 160]
    assert gen.table_elems(rows, cols) == 176
    # the C-ABI helper computes the same canonical table
    ct, crows, celems = A.segments_layout(rows, cols)
    assert np.array_equal(np.array(ct), t) and crows == 10 and celems == 176
    with pytest.raises(A.AstitchError):
        A.segments_layout([1], [0])
    with pytest.raises(A.AstitchError):
        A.segments_layout([-1], [4])


def test_oracle_ragged_equals_masked_dense():
    """A packed varlen segment of length L is the masked dense problem restricted
    to its valid prefix (two independent code paths of the oracle: per-segment
    sub-problems vs the key-padding mask)."""
    L = [37, 5, 64, 1]
    heads = 3
    sv = _spec(L, heads=heads)
    xv = gen.generate("C3v", sv)
    got = evaluate(sv, xv)["p"]
    t = xv["S"]
    for b, Lb in enumerate(L):
        r0, pitch, off = t[b, 0], t[b, 2], 8 * t[b, 3]
        nr = heads * Lb
        dense = np.zeros((nr, 64), dtype=np.uint16)
        dense[:, :Lb] = xv["s"][off: off + nr * pitch].reshape(nr, pitch)[:, :Lb]
        m = specs.get("C3", rows=nr, cols=64)
        m["mask"]["rows_per_segment"] = nr
        ref = evaluate(m, {"s": dense, "L": np.array([Lb], dtype=np.int32)})["p"]
        seg = got[off: off + nr * pitch].reshape(nr, pitch)
        np.testing.assert_allclose(seg[:, :Lb], ref[:, :Lb], rtol=1e-15, atol=0)
        assert np.all(seg[:, Lb:] == 0.0)              # pitch padding stays 0
        np.testing.assert_allclose(seg[:, :Lb].sum(axis=1), 1.0, rtol=1e-13)  # softmax rows sum to 1
        del r0


def test_oracle_ragged_single_column_rows_are_one():
    """cols_s = 1: softmax of one element is exactly 1."""
    sv = _spec([1, 1], heads=4)
    out = evaluate(sv, gen.generate("C3v", sv))["p"]
    t = gen.segment_table(sv["segments"]["seg_rows"], sv["segments"]["seg_cols"])
    for b in range(2):
        off, pitch = 8 * t[b, 3], t[b, 2]
        seg = out[off: off + 4 * pitch].reshape(4, pitch)
        assert np.all(seg[:, 0] == 1.0) and np.all(seg[:, 1:] == 0.0)


def test_ragged_subset_keeps_segment_bits():
    sv = _spec([37, 5, 64, 1, 20], heads=2)
    x = gen.generate("C3v", sv)
    sub = gen.ragged_subset(sv, [3, 1])
    xs = gen.generate("C3v", sub)
    t, ts = x["S"], xs["S"]
    for j, b in enumerate([3, 1]):
        nr = sv["segments"]["seg_rows"][b]
        a = x["s"][8 * t[b, 3]: 8 * t[b, 3] + nr * t[b, 2]]
        c = xs["s"][8 * ts[j, 3]: 8 * ts[j, 3] + nr * ts[j, 2]]
        assert np.array_equal(a, c)


def _plan(spec, flags=A.FLAG_NO_COMPILE, **kw):
    g = A.Graph.from_spec(spec)
    return A.Plan(g, spec["rows"], spec["cols"], device=-1, flags=flags, **kw)


def test_planner_ragged_row_team_and_describe():
    sv = gen.ragged_spec(specs.get("C3v"), 3)
    assert sv["rows"] == 16 * sum(sv["segments"]["seg_cols"])
    p = _plan(sv)
    d = p.describe()
    assert d["mapping"]["template"] == "row_team" and d["mapping"]["team"] == 8
    assert d["ragged"] == {"nseg": 64, "elems": sv["segments"]["elems"]}
    src = p.source(0)
    assert "as::seg_find<NSEG>(SG" in src and "constexpr int KF = " in src
    assert "// chunks of the row only (packed)" in src     # no writes past a row
    assert "= (-AS_INF);" in src                            # mask absorption still applies
    assert p.io_shape("FULL") == (sv["segments"]["elems"],)


def test_planner_ragged_unsupported_combinations():
    sv = _spec([8, 16], heads=1)
    with pytest.raises(A.AstitchError):
        _plan(sv, flags=A.FLAG_NO_COMPILE | A.FLAG_FORCE_GLOBAL)
    with pytest.raises(A.AstitchError):
        _plan(sv, shard_rank=0, shard_world=2)
    # a column reduction over packed rows is rejected
    col = dict(sv)
    col["ops"] = [("cs", "reduce", "SUM", "COL", "s")]
    col["outputs"] = [("cs", "F32")]
    with pytest.raises(A.AstitchError):
        _plan(col)
    g = A.Graph()
    g.segments(2, 64)
    with pytest.raises(A.AstitchError):
        g.lengths(4)                                        # one mask mechanism per graph


def test_ragged_kernel_compiles_for_sm100a():
    sv = gen.ragged_spec(specs.get("C3v"), 3)
    p = _plan(sv, flags=0)
    d = p.describe()
    # a spill of a few registers (<= 32 bytes) is accepted rather than halving
    # the occupancy (runtime.cpp, assume-relax-apply)
    assert p.cubin(0)[:4] == b"\x7fELF" and d["kernels"][0]["spill_bytes"] <= 32
    assert d["mapping"]["grid"] >= 2 * 148
