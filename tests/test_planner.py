"""Planner golden tests (host only): op classes, dominant candidates, groups,
schemes (Table 1 / Sec. 4.3), the thread-mapping selector (Sec. 3.3)
and the generated kernels (NVRTC sm_100a compile, no GPU needed)."""

import pytest

import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
from workloads import specs


def describe(cfg, rows=None, cols=None, flags=A.FLAG_NO_COMPILE, **kw):
    spec = specs.get(cfg, rows=rows, cols=cols)
    g = A.Graph.from_spec(spec)
    p = A.Plan(g, spec["rows"], spec["cols"], device=-1, flags=flags, **kw)
    d = p.describe()
    ops = {name: d["ops"][vid] for name, vid in g.names.items()}
    return d, ops, p


def test_c1_softmax_regional_one_group():
    d, ops, _ = describe("C1")
    assert ops["m"]["class"] == "reduce_row" and ops["m"]["scheme"] == "regional"
    assert ops["s"]["scheme"] == "regional"
    assert ops["e"]["class"] == "heavy_ew" and ops["e"]["scheme"] == "local"
    assert ops["y"]["scheme"] == "independent" and ops["y"]["candidate"]
    assert len(d["groups"]) == 1
    assert ops["m"]["dominant"] and ops["s"]["sub_dominant"] and ops["y"]["sub_dominant"]
    assert d["mapping"]["template"] == "row_team"


def test_c2_layernorm_heavy_rowvec_candidate():
    d, ops, _ = describe("C2")
    # rsqrt on the per-row variance is heavy EW followed by a broadcast (Fig. 5 pattern)
    assert ops["rstd"]["class"] == "heavy_ew" and ops["rstd"]["candidate"]
    assert ops["rstd"]["scheme"] == "regional"
    assert ops["hs"]["scheme"] == "regional" and ops["vs"]["scheme"] == "regional"
    assert ops["o"]["class"] == "heavy_ew"
    assert len(d["groups"]) == 1
    m = d["mapping"]
    assert m["template"] == "row_team" and m["team"] == 32 and m["chunks_per_lane"] == 3 and m["vec_elems"] == 8
    assert m["lane_util"] == 1.0


def test_c3_mask_row_team_absorbed():
    d, ops, p = describe("C3")
    m = d["mapping"]
    # masked rows: finer chunks (T=16 x 4 chunks of 8 bf16) for chunk-uniform skipping
    assert m["template"] == "row_team" and m["team"] == 16 and m["chunks_per_lane"] == 4
    assert ops["m"]["scheme"] == "regional" and ops["z"]["scheme"] == "regional"
    src = p.source(0)
    # mask absorption: invalid logits take -inf, reductions carry no selects
    assert "= (-AS_INF);" in src
    assert "r_ = r_ * 0x1p-3f;" in src          # max(0.125 x) = 0.125 max(x) hoist
    assert "as::ex2_2(as::fma2(" in src         # exp(kx - m) fused to ex2(fma)


def test_c4_many_tiny_rows_packed():
    d, _, _ = describe("C4")
    m = d["mapping"]
    assert m["template"] == "packed_tile"
    assert m["team"] == 1 and m["chunks_per_lane"] == 9
    assert m["lds128_conflict_ways"] == 1          # 144-byte rows: conflict-free LDS.128
    assert m["smem_bytes"] > 0 and m["stages"] >= 3
    # ablation NO_TMA falls back to a row team
    d2, _, _ = describe("C4", flags=A.FLAG_NO_COMPILE | A.FLAG_NO_TMA)
    assert d2["mapping"]["template"] == "row_team"


def test_c5_global_scheme_and_barrier():
    d, ops, _ = describe("C5")
    assert d["mapping"]["template"] == "global_sweep"
    assert ops["db"]["class"] == "reduce_col" and ops["db"]["scheme"] == "global" and ops["db"]["dominant"]
    assert ops["b_new"]["post_barrier"] and not ops["dz"]["post_barrier"]
    assert ops["g"]["class"] == "heavy_ew" and ops["g"]["scheme"] == "local"
    assert ops["dz"]["scheme"] == "local"            # consumed by the reduce before the barrier
    assert d["global_fulls"] == [] and not d["needs_sweep2"]
    assert d["workspace"]["total"] > 0
    assert d["mapping"]["grid"] <= d["mapping"]["blocks_per_sm"] * 148


def test_fig5_heavy_producer_once_per_row():
    d, ops, p = describe("fig5")
    assert ops["pw"]["candidate"] and ops["pw"]["scheme"] == "regional"
    src = p.source(0)
    # power is computed on the row scalar (once per row), not per element
    assert "const float s" in src and "(s" in src


def test_fig7a_schemes_match_paper():
    """regional for reduce.1, global for power.1 and reduce.2,
    independent for multiply.1, local for the others; final dominants reduce.1
    and reduce.2, sub-dominants power.1 and multiply.1.  The paper's
    global scheme buffers power.1 in HBM: the plan with recomputation off
    (remat=0)."""
    d, ops, _ = describe("fig7a", tune="remat=0")
    assert d["global_fulls"] == [ops["power1"]["id"]] and "recomputed_at" not in ops["power1"]
    assert ops["reduce1"]["scheme"] == "regional"
    assert ops["power1"]["scheme"] == "global"
    assert ops["reduce2"]["scheme"] == "global"
    assert ops["multiply1"]["scheme"] == "independent"
    for n in ("divide1", "add1", "broadcast1", "broadcast2"):
        assert ops[n]["scheme"] == "local", n
    assert ops["reduce1"]["dominant"] and ops["reduce2"]["dominant"]
    assert ops["power1"]["sub_dominant"] and ops["multiply1"]["sub_dominant"]
    assert len(d["groups"]) == 2
    assert d["needs_sweep2"] and d["kernel_count"] == 1


def test_fig7a_power1_recomputed_not_buffered():
    """Reading R22 (default plan): power.1 still crosses the barrier (global
    scheme), but the level-1 sweep re-reads x (4 B / element) and recomputes
    add.1 and power.1 instead of writing and re-reading an fp32 buffer (8 B);
    only the row scalar divide.1 is buffered (R floats + its lo part)."""
    d, ops, _ = describe("fig7a")
    assert ops["power1"]["scheme"] == "global" and ops["power1"]["recomputed_at"] == [1]
    assert ops["add1"]["recomputed_at"] == [1] and ops["add1"]["scheme"] == "local"
    assert d["global_fulls"] == [ops["divide1"]["id"]] and ops["divide1"]["scheme"] == "global"
    assert ops["reduce1"]["scheme"] == "regional" and ops["multiply1"]["scheme"] == "independent"
    # BatchNorm: the centred x of the variance level is recomputed for the
    # normalising sweep (level 2), no FULL buffer at all
    d, ops, _ = describe("bn", rows=100_000, cols=256)
    assert d["global_fulls"] == [] and ops["xc"]["recomputed_at"] == [2]
    # two fp32 inputs (8 B) cost as much as the buffer: buffered
    spec = {"name": "two_in", "rows": 5000, "cols": 64, "inputs": [("x", "FULL", "F32"), ("y", "FULL", "F32")],
            "mask": None, "ops": [("xy", "binary", "MUL", "x", "y"), ("s", "reduce", "SUM", "COL", "xy"),
                                  ("sb", "broadcast", "COL", "s"), ("o", "binary", "SUB", "xy", "sb")],
            "outputs": [("o", "F32")]}
    g = A.Graph.from_spec(spec)
    d = A.Plan(g, 5000, 64, device=-1, flags=A.FLAG_NO_COMPILE).describe()
    assert d["global_fulls"] == [g.names["xy"]]
    spec["inputs"] = [("x", "FULL", "BF16"), ("y", "FULL", "BF16")]
    g = A.Graph.from_spec(spec)
    d = A.Plan(g, 5000, 64, device=-1, flags=A.FLAG_NO_COMPILE).describe()
    assert d["global_fulls"] == [] and d["ops"][g.names["xy"]]["recomputed_at"] == [1]


def test_fig6_selector_branches():
    d, _, _ = describe("fig6a")              # <750000,32>: pack many rows per block
    m = d["mapping"]
    assert m["team"] < 32 and m["rows_per_block"] > 32
    # light rows: one row group per CTA on a non-persistent grid (the block
    # scheduler orders the sweep); heavier rows: a persistent one-wave grid
    assert m["nonpersistent"] and m["grid"] * m["rows_per_block"] >= 750_000 and m["vertical_trips"] == 1
    d, _, _ = describe("C3")      # masked rows: tma_team, 16-row tiles, one wave of ring CTAs
    m = d["mapping"]
    assert m["tma_team"] and m["tma_rows"] == 16 and m["tma_stages"] == 4 and not m["nonpersistent"]
    assert m["threads"] == m["rows_per_block"] * m["team"] + 32 and m["grid"] == 148 * m["blocks_per_sm"]
    d, _, _ = describe("C2", rows=65536)   # heavy unmasked rows: one persistent wave
    assert d["mapping"]["grid"] <= d["mapping"]["blocks_per_sm"] * 148
    # <64,30000>: the paper's shape rule holds, but 120 KB rows are below the
    # measured B200 threshold (reading R15) -> one block team per row
    d, _, _ = describe("fig6b")
    assert d["mapping"]["template"] == "row_team" and d["mapping"]["team"] == 1024
    d, _, _ = describe("fig6b", flags=A.FLAG_NO_COMPILE | A.FLAG_FORCE_SPLIT)
    assert d["mapping"]["template"] == "split_row" and "split rule holds" in d["mapping"]["reason"]
    # cluster of K CTAs: the largest power of two with rows * K <= SMs (one wave)
    assert d["mapping"]["split"] == 2 and d["mapping"]["grid"] % 2 == 0
    d, _, _ = describe("fig6b", cols=300_000)  # 1.2 MB rows: split by default (streamed over a cluster)
    assert d["mapping"]["template"] == "row_stream" and d["mapping"]["split"] == 2
    assert d["mapping"]["grid"] == 128
    d, _, _ = describe("fig6b", cols=300_000, flags=A.FLAG_NO_COMPILE | A.FLAG_NO_SPLIT)
    # no splitting: a 1024-lane block would need 293 values per lane -> streamed by one block
    assert d["mapping"]["template"] == "row_stream" and d["mapping"]["split"] == 1


@pytest.mark.parametrize("cfg", ["C2", "C3", "C4"])
def test_mapping_independent_of_rows(cfg):
    """Reading R13: a row's reduction tree depends only on C, so shards are
    bitwise equal to the unsharded run."""
    a, _, _ = describe(cfg)
    b, _, _ = describe(cfg, rows=8192 + 17)
    for k in ("template", "team", "chunks_per_lane", "vec_elems"):
        assert a["mapping"][k] == b["mapping"][k], k


def test_remote_stitching_one_kernel():
    """Two independent subgraphs in one stitch op (remote stitching):
    separate groups, one kernel, outputs of both are independent."""
    d, ops, p = describe("remote")
    assert len(d["groups"]) == 2
    assert ops["m"]["group"] != ops["ys"]["group"]
    assert d["kernel_count"] == 1 and d["mapping"]["template"] in ("row_team", "packed_tile")


def test_batchnorm_two_barrier_levels():
    """Dependent column reductions (BatchNorm: mean, then variance): levels
    1 and 2, the centred values read again after the 2nd barrier (global:
    buffered in HBM with remat=0, recomputed from x by default, R22), one
    kernel."""
    d, ops, p = describe("bn", tune="remat=0")
    assert ops["s1"]["class"] == "reduce_col" and ops["s2"]["class"] == "reduce_col"
    assert ops["s1"]["scheme"] == "global" and ops["s2"]["scheme"] == "global"
    assert ops["xc"]["scheme"] == "global"                 # read again after the 2nd barrier
    assert len(d["global_fulls"]) == 1
    d, ops, p = describe("bn")
    assert ops["xc"]["scheme"] == "global" and d["global_fulls"] == []
    assert d["kernel_count"] == 1 and d["mapping"]["template"] == "global_sweep"
    # per level: partials -> barrier -> finalise -> barrier (publish) -> next sweep
    assert p.source(0).count("as::grid_barrier(bar);") == 4


def test_force_global_ablation_demotes_row_reductions():
    """FORCE_GLOBAL (regional -> global demotion; the Table 4 mirror):
    every row reduction is stored to HBM and read back after a grid barrier."""
    d, ops, p = describe("C1", flags=A.FLAG_NO_COMPILE | A.FLAG_FORCE_GLOBAL)
    assert ops["m"]["scheme"] == "global" and ops["s"]["scheme"] == "global"
    assert d["mapping"]["template"] == "global_sweep" and d["kernel_count"] == 1
    # softmax: max | exp + sum | divide -> 3 sweeps, 2 barriers; e buffered in HBM
    assert p.source(0).count("as::grid_barrier(bar);") == 2
    assert set(d["global_fulls"]) == {ops[n]["id"] for n in ("m", "e", "s")}
    d2, ops2, p2 = describe("C2", flags=A.FLAG_NO_COMPILE | A.FLAG_FORCE_GLOBAL)
    assert p2.source(0).count("as::grid_barrier(bar);") == 2   # mean | variance | normalise
    d3, _, _ = describe("C1")
    assert d3["mapping"]["template"] == "row_team"
    with pytest.raises(A.AstitchError):
        describe("C1", flags=A.FLAG_NO_COMPILE | A.FLAG_FORCE_GLOBAL, shard_rank=0, shard_world=2)


DOUBLE_SOFTMAX = {
    "name": "double_softmax", "rows": 1000, "cols": 200,
    "inputs": [("x", "FULL", "F32")], "mask": None,
    "ops": [("m1", "reduce", "RMAX", "ROW", "x"), ("m1b", "broadcast", "ROW", "m1"),
            ("d1", "binary", "SUB", "x", "m1b"), ("e1", "unary", "EXP", "d1"),
            ("s1", "reduce", "SUM", "ROW", "e1"), ("s1b", "broadcast", "ROW", "s1"),
            ("y1", "binary", "DIV", "e1", "s1b"),
            ("m2", "reduce", "RMAX", "ROW", "y1"), ("m2b", "broadcast", "ROW", "m2"),
            ("d2", "binary", "SUB", "y1", "m2b"), ("e2", "unary", "EXP", "d2"),
            ("s2", "reduce", "SUM", "ROW", "e2"), ("s2b", "broadcast", "ROW", "s2"),
            ("y2", "binary", "DIV", "e2", "s2b")],
    "outputs": [("y2", "F32")],
}


def test_global_buffer_reuse_by_liveness():
    """a6 memory reuse: FORCE_GLOBAL double softmax buffers m1, e1, s1,
    y1, m2, e2, s2 in HBM across 4 barriers; a buffer whose last reader is an
    earlier sweep is taken over (m2 <- m1, e2 <- e1, s2 <- s1): 4 buffers, not 7."""
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A2
    g = A2.Graph.from_spec(DOUBLE_SOFTMAX)
    p = A2.Plan(g, 1000, 200, device=-1, flags=A.FLAG_NO_COMPILE | A.FLAG_FORCE_GLOBAL)
    d = p.describe()
    assert len(d["global_fulls"]) == 7 and d["global_buffers"] == 4
    assert p.source(0).count("as::grid_barrier(bar);") == 4
    # FULL buffers hold R x C floats, ROWVEC buffers R floats
    # 2 FULL buffers (R x C) + 2 ROWVEC buffers (2 R each: value + R7b lo part)
    assert d["workspace"]["total"] - d["workspace"]["globals"] <= (2 * 1000 * 200 + 2 * 2 * 1000) * 4 + 4 * 256


def test_no_pack_ablation():
    d, _, _ = describe("fig6a", flags=A.FLAG_NO_COMPILE | A.FLAG_NO_PACK)
    assert d["mapping"]["team"] == 32


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3", "C4", "C5", "fig5", "fig7a", "fig6a", "fig6b"])
def test_generated_kernels_compile_for_sm100a(cfg):
    """NVRTC compiles every generated kernel for sm_100a on the host (no GPU)."""
    d, _, p = describe(cfg, flags=0)
    cub = p.cubin(0)
    assert len(cub) > 1000 and cub[:4] == b"\x7fELF"
    k = d["kernels"][0]
    # a one-wave row team may keep a small spill at its target occupancy (C2:
    # 40 bytes at 7 blocks/SM, measured faster than spill-free at 4)
    allowed = 64 if d["mapping"].get("single_wave_bps", 0) > 0 else 32
    assert k["spill_bytes"] <= allowed, k
    assert k["name"].startswith("astitch_")


def test_sharded_plan_has_epilogue_kernels():
    d, _, _ = describe("C5", rows=131072, flags=0, shard_rank=1, shard_world=8)
    assert d["kernel_count"] == 1 and d["shard_kernels"] == 2
    d, _, _ = describe("fig7a", flags=0, shard_rank=0, shard_world=2)
    assert d["shard_kernels"] == 3


def test_row_stream_for_rows_beyond_registers():
    """A row too long for a team's registers is streamed in column tiles (one
    pass per row-reduction level: softmax = max | sum | output = 3 passes)."""
    d, _, p = describe("C1", rows=16, cols=2_000_000)
    m = d["mapping"]
    assert m["template"] == "row_stream" and m["split"] == 8 and m["chunks_per_lane"] * m["vec_elems"] == 32
    src = p.source(0)
    assert src.count("// ---- pass ") == 3
    d, _, _ = describe("C1")                       # short rows stay in registers
    assert d["mapping"]["template"] == "row_team"
    d, _, _ = describe("C4", rows=100_000, cols=200_000)  # many long rows: block per row, no cluster
    assert d["mapping"]["template"] == "row_stream" and d["mapping"]["split"] == 1


def test_one_wave_row_teams_and_store_cap():
    """Launch heuristics measured on B200: rows that need <= 28
    warps per SM get one wave of 4-warp blocks (C2: 4096 rows -> 1024 blocks
    of 128 threads, 7 per SM, every row its own team); row teams that write
    whole rows keep ~48 KB of row stores per SM (C3: 3 blocks of 256);
    read-mostly rows keep the full occupancy (fig6a)."""
    d, _, _ = describe("C2")
    m = d["mapping"]
    assert m["single_wave_bps"] == 7 and m["threads"] == 128 and m["grid"] == 1024
    assert m["vertical_trips"] == 1
    d, _, _ = describe("C2", rows=300)                     # 2 warps per SM: default blocks
    assert d["mapping"]["single_wave_bps"] == 0
    d, _, _ = describe("C3")      # 3 resident blocks of 256 per SM, an oversubscribed grid
    assert d["mapping"]["blocks_per_sm"] == 3 and d["mapping"]["grid"] >= 3 * 148
    d, _, _ = describe("fig6a")
    assert d["mapping"]["blocks_per_sm"] == 8


def test_cluster_size_fills_one_wave():
    """Few long rows: K = largest power of two <= 8 with R * K <= SMs; rows
    <= 9 ask for non-portable clusters of 16 (validated when the kernel loads
    on a GPU, else back to 8)."""
    for rows, k in ((64, 2), (16, 8), (37, 4), (38, 2), (100, 1), (3, 16), (9, 16), (10, 8)):
        d, _, _ = describe("C1", rows=rows, cols=2_000_000)
        m = d["mapping"]
        assert m["template"] == "row_stream" and m["split"] == k, (rows, m["split"])
        assert rows * m["split"] <= 148 or m["split"] == 1


def _many_inputs_spec(n, cols, rows=100_000, dt="F32"):
    """n short-row FULL inputs summed, then a row-centred output (row reduce)."""
    ins = [(f"x{i}", "FULL", dt) for i in range(n)]
    ops, prev = [], "x0"
    for i in range(1, n):
        ops.append((f"a{i}", "binary", "ADD", prev, f"x{i}"))
        prev = f"a{i}"
    ops += [("s", "reduce", "SUM", "ROW", prev), ("sb", "broadcast", "ROW", "s"), ("y", "binary", "SUB", prev, "sb")]
    return {"name": f"many{n}", "rows": rows, "cols": cols, "inputs": ins, "mask": None, "ops": ops,
            "outputs": [("y", dt)]}


@pytest.mark.parametrize("n", [2, 3, 7, 12, 16])
@pytest.mark.parametrize("cols", [36, 100, 120])
def test_smem_overflow_demotion(n, cols):
    """a6 / P:L288: no plan ever asks for more shared memory than a B200 block
    can have (227 KB opt-in); a staged tile that would overflow is demoted
    (fewer stages / rows) or abandoned for a register row team, and the plan
    says so in describe()["demotions"].  Round 1 planned 442-1475 KB here."""
    s = _many_inputs_spec(n, cols)
    d = A.Plan(A.Graph.from_spec(s), s["rows"], cols, device=-1, flags=A.FLAG_NO_COMPILE).describe()
    m = d["mapping"]
    assert m["smem_bytes"] <= 227 * 1024
    if m["template"] == "packed_tile":
        assert m["smem_bytes"] <= 100 * 1024           # >= 2 blocks per SM
    if n >= 7:
        assert m["template"] == "row_team" and m["smem_bytes"] == 0
        assert any("row team" in x for x in d["demotions"])
    assert d["kernel_count"] == 1


def test_global_sweep_block_combine_fits_smem():
    """The global sweep's block combine (teams x columns x 4 B, x2 for fp64
    hi/lo partials) is demoted to fewer teams per block instead of
    overflowing shared memory."""
    for name, rows, cols in (("C5", 4096, 1024), ("bn", 3000, 4096), ("bn", 3000, 8192), ("C5", 4096, 16384)):
        s = specs.get(name, rows=rows, cols=cols)
        d = A.Plan(A.Graph.from_spec(s), rows, cols, device=-1, flags=A.FLAG_NO_COMPILE).describe()
        m = d["mapping"]
        if m["tma_sweep"]:  # the bulk-copy ring fills one CTA's shared memory (the combine reuses it)
            assert m["smem_bytes"] <= 227 * 1024 - 8 * 1024 and m["blocks_per_sm"] == 1, (name, cols, m)
            continue
        assert m["smem_bytes"] <= 96 * 1024, (name, cols, m)
        assert m["rows_per_block"] == 1 or m["smem_bytes"] > 0


def test_group_mappings_follow_their_dominants():
    """Step 2: every group's schedule is its dominant's; Fig. 7(a)
    has a row-reduce group (level 0) and a column-reduce group (level 1);
    an element-wise-only group adopts its producer's mapping."""
    d, _, _ = describe("fig7a")
    gm = d["group_mappings"]
    kinds = sorted((x["level"], x["schedule"].split(":")[0]) for x in gm)
    assert kinds == [(0, "row reduce"), (1, "column reduce")]
    ew = {"name": "ew", "rows": 100, "cols": 64, "inputs": [("x", "FULL", "F32")], "mask": None,
          "ops": [("e", "unary", "EXP", "x"), ("n", "unary", "NEG", "e")], "outputs": [("n", "F32")]}
    p = A.Plan(A.Graph.from_spec(ew), 100, 64, device=-1, flags=A.FLAG_NO_COMPILE)
    assert all("element-wise only" in x["schedule"] or "dominant" in x for x in p.describe()["group_mappings"])


def test_tma_sweep_selection():
    """tma_sweep (R23) for one-sweep element-wise + column-reduction graphs
    (C5 and its shapes); not for row reductions (fig7a), dependent column
    levels (BatchNorm), masks, or when switched off (tuning tma=0, NO_TMA)."""
    def m(name, rows=1 << 20, cols=None, **kw):
        s = specs.get(name, rows=rows, cols=cols)
        return A.Plan(A.Graph.from_spec(s), rows, s["cols"], device=-1, flags=kw.get("flags", A.FLAG_NO_COMPILE),
                      tune=kw.get("tune")).describe()["mapping"]
    c5 = m("C5")
    assert c5["tma_sweep"] and c5["vec_elems"] == 4 and c5["team"] == 256 and c5["rows_per_block"] == 1
    assert c5["threads"] == 288 and c5["tma_stages"] == 3 and c5["tma_rows"] == 16
    assert c5["smem_bytes"] == 3 * 16 * 4096 and c5["grid"] == 148
    assert m("C5", cols=512)["rows_per_block"] == 2                  # >= 8 compute warps
    assert m("C5", cols=4096)["vec_elems"] == 8                      # > 512 lanes of 4 columns
    assert not m("C5", cols=100)["tma_sweep"]                        # lanes not a multiple of a warp
    assert not m("C5", cols=16384)["tma_sweep"]                      # column slabs instead
    assert not m("C5", tune="tma=0")["tma_sweep"]
    assert not m("C5", flags=A.FLAG_NO_COMPILE | A.FLAG_NO_TMA)["tma_sweep"]
    assert not m("fig7a")["tma_sweep"]                               # row reductions
    assert not m("bn", rows=3000, cols=128)["tma_sweep"]             # short sweep (< 16 tiles per CTA)
    assert m("bn", rows=1 << 20, cols=1024)["tma_sweep"]             # long BatchNorm: 3 levels, precise bins
    assert m("C5", rows=7, tune="tma=1")["grid"] == 1                # never more CTAs than tiles
