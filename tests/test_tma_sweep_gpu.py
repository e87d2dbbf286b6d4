"""GPU tests of the tma_sweep global sweep (reading R23): address-ordered
dynamic row tiles staged by bulk copies, column sums in exact binned
accumulators.  The tile order changes from run to run and with the grid size;
the column totals must not (bitwise), and must match the fp64 oracle under the
DESIGN.md rule, including non-finite and extreme-range columns.
"""

import numpy as np
import pytest

from oracle import evaluate
from tests.harness import check_close, run_gpu, spec_tol
from workloads import gen, specs

pytestmark = pytest.mark.gpu


def _plan(spec, **kw):
    """Plans default to tune tma=1: the planner takes tma_sweep by itself for
    long sweeps only (>= 16 tiles per CTA); these tests use small shapes."""
    import torch
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
    kw.setdefault("tune", "tma=1")
    return A.Plan(A.Graph.from_spec(spec), spec["rows"], spec["cols"], device=torch.cuda.current_device(), **kw)


def test_tma_sweep_chosen_for_c5():
    spec = specs.get("C5", rows=1 << 20)
    m = _plan(spec, tune=None).describe()["mapping"]
    assert m["tma_sweep"] and m["template"] == "global_sweep"
    assert m["threads"] == m["rows_per_block"] * m["team"] + 32   # + the producer warp
    assert m["blocks_per_sm"] == 1 and m["smem_bytes"] == m["tma_stages"] * m["tma_rows"] * 2 * 1024 * 2


@pytest.mark.parametrize("rows", [1, 17, 20011])
def test_tma_sweep_order_independent_bitwise(rows):
    """Grids of 148, 37 and 5 CTAs take the tiles in different orders and
    groupings; the binned totals are identical bit for bit, and so is dz."""
    spec = specs.get("C5", rows=rows)
    x = gen.generate("C5", spec)
    ref = evaluate(spec, x)
    outs = []
    for sms in (0, 37, 5):
        p = _plan(spec, sm_count=sms)
        assert p.describe()["mapping"]["tma_sweep"]
        got = run_gpu(spec, x, plan=p)
        for name, dt in spec["outputs"]:
            check_close(got[name], ref[name], dt, spec_tol(spec), name=f"C5[{rows}] sms={sms}:{name}")
        outs.append(got)
    for got in outs[1:]:
        for k in got:
            assert np.array_equal(got[k], outs[0][k]), k


def test_tma_sweep_static_sweep_still_correct():
    """tune tma=0 keeps the register global sweep (static row ownership)."""
    spec = specs.get("C5", rows=3005)
    x = gen.generate("C5", spec)
    ref = evaluate(spec, x)
    p = _plan(spec, tune="tma=0")
    assert not p.describe()["mapping"]["tma_sweep"]
    got = run_gpu(spec, x, plan=p)
    for name, dt in spec["outputs"]:
        check_close(got[name], ref[name], dt, spec_tol(spec), name=name)


COLSUM = {
    "name": "colsum_edge", "rows": 2003, "cols": 256,
    "inputs": [("x", "FULL", "F32")], "mask": None,
    "ops": [("s", "reduce", "SUM", "COL", "x"), ("m", "reduce", "RMAX", "COL", "x")],
    "outputs": [("s", "F32"), ("m", "F32")],
}


def test_tma_sweep_extreme_columns():
    """Non-finite deposits (R12 / R23: +inf, +inf and -inf -> NaN, NaN),
    huge dynamic range, exact cancellation, zeros and subnormals."""
    rng = np.random.default_rng(23)
    R, C = COLSUM["rows"], COLSUM["cols"]
    x = rng.standard_normal((R, C)).astype(np.float32)
    x[:, 0] = 1.0
    x[1234, 0] = 1.0e30                      # window jumps to 2^100 late in the sweep
    x[5, 1] = 3.0e38; x[6, 1] = -3.0e38       # cancels exactly; the rest is truncated below 2^96
    x[100, 2] = np.inf
    x[3, 3] = np.inf; x[2000, 3] = -np.inf    # -> NaN
    x[77, 4] = np.nan
    x[:, 5] = 0.0
    x[:, 6] = np.float32(1e-40)               # subnormal deposits
    x[:, 7] = np.where(np.arange(R) % 2 == 0, 1.0 + 2.0 ** -20, -1.0).astype(np.float32)
    x[:, 8] = -np.abs(x[:, 8]) * 1e-30        # tiny, all negative
    x[:, 9] = np.float32(2.0 ** 60) * np.sign(x[:, 9])
    xin = {"x": x}
    p = _plan(COLSUM)
    assert p.describe()["mapping"]["tma_sweep"]
    got = run_gpu(COLSUM, xin, plan=p)
    ref = evaluate(COLSUM, xin)
    assert np.isposinf(got["s"][2]) and np.isnan(got["s"][3]) and np.isnan(got["s"][4])
    assert np.isnan(got["m"][4]) and np.isposinf(got["m"][2])
    assert got["s"][5] == 0.0
    # exact cases: column 7 = (R // 2 + 1) * 2^-20 exactly, column 0 = 1e30 + (R - 1)
    assert got["s"][7] == np.float32(ref["s"][7])
    assert got["s"][0] == np.float32(ref["s"][0])
    assert got["s"][9] == np.float32(ref["s"][9])
    for name, dt in COLSUM["outputs"]:
        check_close(got[name], ref[name], dt, spec_tol(COLSUM), name=name)
    # columns 1 and 8 compared on their own scale (not floored by the RMS of the huge columns)
    assert abs(got["s"][8] - ref["s"][8]) <= 1e-5 * abs(ref["s"][8])
    # column 1: +-3e38 cancel exactly; the standard-normal rest is truncated
    # at the window of 3e38 (2^128 -> bins from 2^64): the total is 0
    assert got["s"][1] == 0.0 and abs(ref["s"][1]) < 1e3


@pytest.mark.parametrize("cols,dt", [(2048, "BF16"), (4096, "BF16"), (512, "F32"), (384, "F32")])
def test_tma_sweep_shapes(cols, dt):
    """E = 4 / 8 lanes, one team (T = 512) or several, fp32 and bf16 rows."""
    spec = specs.get("C5", rows=997, cols=cols)
    if dt == "F32":
        spec["inputs"] = [(n, k, "F32" if k == "FULL" else d) for n, k, d in spec["inputs"]]
        spec["outputs"] = [(n, "F32") for n, _ in spec["outputs"]]
    x = gen.generate("C5", spec)
    ref = evaluate(spec, x)
    p = _plan(spec)
    assert p.describe()["mapping"]["tma_sweep"], p.describe()["mapping"]["reason"]
    got = run_gpu(spec, x, plan=p)
    for name, d in spec["outputs"]:
        check_close(got[name], ref[name], d, spec_tol(spec), name=f"{cols}:{name}")
    again = run_gpu(spec, x, plan=_plan(spec, sm_count=11))
    for k in got:
        assert np.array_equal(got[k], again[k]), k


# ---------------------------------------------------------------- tma_team
@pytest.mark.parametrize("cfg,rows,cols,tune", [
    ("C3", 3 * 256 + 7, None, "tma_team=1"), ("C3", 2048, None, "tma_team=1,tma_teams=32"),
    ("C3", 1000, None, "tma_team=1,tma_rows=16,tma_stages=2"),
    ("C3", 1000, None, "tma_team=1,tma_rows=16,tma_stages=4"),
    ("C1", None, None, "tma_team=1"), ("C1", 50000, 128, "tma_team=1"),
    ("C2", 300, 256, "tma_team=1"), ("C4", 20003, 36, "tma_team=1")])
def test_tma_team_parity(cfg, rows, cols, tune):
    """Row teams fed by the producer warp (one bulk copy per row's valid
    prefix, address-ordered tiles) match the oracle, run after run."""
    spec = specs.get(cfg, rows=rows, cols=cols)
    if spec.get("mask"):
        spec["mask"]["rows_per_segment"] = 256
    if spec.get("segments"):
        spec["segments"]["heads"] = 2
        spec = gen.ragged_spec(spec, 3)
    x = gen.generate(cfg, spec)
    p = _plan(spec, tune=tune)
    m = p.describe()["mapping"]
    if m["template"] == "row_team":
        assert m["tma_team"], m["reason"]
    got = run_gpu(spec, x, plan=p)
    ref = evaluate(spec, x)
    for name, dt in spec["outputs"]:
        check_close(got[name], ref[name], dt, spec_tol(spec), name=f"{cfg}:{name}")
    again = run_gpu(spec, x, plan=p)
    for k in got:
        assert np.array_equal(got[k], again[k]), k


@pytest.mark.parametrize("lengths,heads", [([37, 1, 8, 9, 64, 511, 512, 200], 2), ([100, 300, 37], 40)])
def test_tma_team_ragged(lengths, heads):
    from tests.test_ragged_gpu import _check, _spec
    spec = _spec(lengths, heads=heads)
    x = gen.generate("C3v", spec)
    plan = _check(spec, x, tune="tma_team=1")
    assert plan.describe()["mapping"]["tma_team"]


@pytest.mark.parametrize("seed,rows,cols,rowwise,flags", [(4039, 4606, 256, True, 0), (4161, 24271, 128, False, 64)])
def test_tma_team_colvec_outputs_fuzz_seeds(seed, rows, cols, rowwise, flags):
    """Graph-fuzz regressions (round 2, `--tma --wide`): a masked row plan
    with COLVEC outputs (tanh(cv - cv), sqrt(|cv| + 1)) under tma_team left
    them unwritten until the pre-barrier column outputs were emitted there."""
    from workloads.random_graphs import random_graph
    spec = random_graph(seed, rows, cols, wide=True, rowwise=rowwise)
    x = gen.generate("fig6a", spec)
    got, plan = run_gpu(spec, x, return_plan=True, flags=flags)
    assert plan.describe()["mapping"]["tma_team"]
    ref = evaluate(spec, x)
    for name, dt in spec["outputs"]:
        check_close(got[name], ref[name], dt, spec_tol(spec), name=name, atol=1e-5)


@pytest.mark.parametrize("seed,rows,cols", [(704, 5000, 512), (1004, 20011, 256), (1190, 37, 1024)])
def test_tma_sweep_barrier_levels(seed, rows, cols):
    """tma_sweep over dependent barrier levels (a value read after a column
    reduction's barrier, buffered in HBM or recomputed): the same ring and
    mbarriers carry on across levels (the sentinel's stage released, a proxy
    fence before the next level's bulk copies), one tile counter per level."""
    from workloads.random_graphs import random_graph
    spec = random_graph(seed, rows, cols, rowwise=False)
    x = gen.generate("fig6a", spec)
    got, plan = run_gpu(spec, x, return_plan=True, tune="tma=1")
    d = plan.describe()
    assert d["mapping"]["tma_sweep"]
    ref = evaluate(spec, x)
    for name, dt in spec["outputs"]:
        check_close(got[name], ref[name], dt, spec_tol(spec), name=name, atol=1e-5)
    again = run_gpu(spec, x, plan=plan)
    for k in got:
        assert np.array_equal(got[k], again[k]), k


@pytest.mark.parametrize("rows,cols", [(3, 1024), (777, 128), (20000, 256), (5, 4096)])
@pytest.mark.parametrize("mean", [0.0, 1000.0, -3.0e4])
def test_tma_sweep_precise_bins_batchnorm(rows, cols, mean):
    """BatchNorm under tma_sweep: the column mean is a precise sum (R7c) whose
    fp64 tile partials go to 4 x 16-bit bins (>= 48 bits): means up to 3e6x
    the spread hold the fp32 1e-5 rule, and the totals are identical for
    grids of 148 and 7 CTAs."""
    spec = specs.get("bn", rows=rows, cols=cols)
    x = gen.generate("bn", spec)
    x["x"] = (mean + 0.01 * x["x"].astype(np.float64)).astype(np.float32)
    ref = evaluate(spec, x)
    outs = []
    for sms in (0, 7):
        p = _plan(spec, sm_count=sms)
        assert p.describe()["mapping"]["tma_sweep"]
        got = run_gpu(spec, x, plan=p)
        for name, dt in spec["outputs"]:
            check_close(got[name], ref[name], dt, spec_tol(spec), name=f"bn[{rows},{cols}] mean={mean}:{name}")
        outs.append(got)
    for k in outs[0]:
        assert np.array_equal(outs[0][k], outs[1][k]), k
