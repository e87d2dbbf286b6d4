"""Shared test helpers: move seeded inputs to the GPU, run a plan through the
C-ABI binding, and compare with the oracle under the tolerance rule of
DESIGN.md (readings R1/R2):

    |g - r| <= tol * max(|r|, s) + 1/2 ulp_out(r) + FLT_MIN     for every element

with s = RMS(r) over the output tensor (floor against cancellation near 0),
1/2 ulp_out the unavoidable rounding of the stored output (0 for fp32), and
tol = 1e-5 for fp32-I/O configs, 2e-3 for bf16/fp16 I/O (BASELINE north_star).
"""

from __future__ import annotations

import numpy as np

TOL_F32 = 1e-5
TOL_BF16 = 2e-3
FLT_MIN = 1.1754943508222875e-38   # smallest normal fp32


def spec_tol(spec: dict) -> float:
    dts = {d for _, k, d in spec["inputs"] if k != "LENGTHS"} | {d for _, d in spec["outputs"]}
    return TOL_F32 if dts <= {"F32"} else TOL_BF16


def half_ulp(ref: np.ndarray, dtype: str) -> np.ndarray:
    if dtype == "F32":
        return np.zeros_like(ref)
    mant = 7 if dtype == "BF16" else 10
    a = np.abs(ref)
    e = np.floor(np.log2(np.where(a > 0, a, 1.0)))
    return np.where(a > 0, np.exp2(e - mant - 1), 0.0)


def check_close(gpu: np.ndarray, ref: np.ndarray, dtype: str, tol: float, name: str = "", atol: float = 0.0) -> dict:
    gpu = np.asarray(gpu, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    assert gpu.shape == ref.shape, (name, gpu.shape, ref.shape)
    # values beyond the output format's range are +-inf once stored (IEEE
    # round-to-nearest overflow: |r| >= 65520 for f16)
    if dtype == "F16":
        ref = np.where(np.abs(ref) >= 65520.0, np.copysign(np.inf, ref), ref)
    # non-finite reference values (e.g. -inf = max over a fully masked row,
    # reading R14) must be reproduced exactly; the rule applies to the rest
    nf = ~np.isfinite(ref)
    if nf.any():
        same = (gpu[nf] == ref[nf]) | (np.isnan(gpu[nf]) & np.isnan(ref[nf]))
        assert same.all(), f"{name}: non-finite reference values not reproduced"
        gpu = np.where(nf, 0.0, gpu)
        ref = np.where(nf, 0.0, ref)
    assert np.isfinite(gpu).all(), f"{name}: non-finite GPU values"
    s = float(np.sqrt(np.mean(ref * ref))) if ref.size else 0.0
    err = np.abs(gpu - ref)
    # + FLT_MIN: subnormal fp32 results may flush to zero (the kernels'
    # MUFU ops are .ftz; reading R21)
    bound = tol * np.maximum(np.abs(ref), s) + half_ulp(ref, dtype) + FLT_MIN + atol
    bad = err > bound
    info = {"max_abs_err": float(err.max()) if err.size else 0.0,
            "max_rel_err_floored": float((err / np.maximum(np.maximum(np.abs(ref), s), 1e-300)).max()) if err.size else 0.0,
            "rms_ref": s, "violations": int(bad.sum())}
    if bad.any():
        idx = np.unravel_index(np.argmax(err - bound), err.shape)
        raise AssertionError(f"{name}: {int(bad.sum())} elements out of tolerance (tol={tol}); worst at {idx}: "
                             f"gpu={gpu[idx]!r} ref={ref[idx]!r} bound={bound[idx]!r}; {info}")
    return info


# ------------------------------------------------------------------ torch side

def to_torch(arr: np.ndarray, dtype: str, device="cuda"):
    import torch
    if dtype == "BF16":
        t = torch.from_numpy(np.ascontiguousarray(arr)).view(torch.bfloat16)
    elif dtype == "F16":
        t = torch.from_numpy(np.ascontiguousarray(arr))
    elif dtype == "I32":
        t = torch.from_numpy(np.ascontiguousarray(arr, dtype=np.int32))
    else:
        t = torch.from_numpy(np.ascontiguousarray(arr, dtype=np.float32))
    return t.to(device) if device is not None else t


def from_torch(t) -> np.ndarray:
    import torch
    return t.detach().to(torch.float64).cpu().numpy()


def device_inputs(spec: dict, inputs: dict, device="cuda"):
    return [to_torch(inputs[n], d, device) for n, _, d in spec["inputs"]]


def run_gpu(spec: dict, inputs: dict, flags: int = 0, plan=None, return_plan=False, tune=None):
    """Plan (unless given) and run `spec` on cuda:0; returns {output: np.float64}."""
    import torch
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
    if plan is None:
        g = A.Graph.from_spec(spec)
        plan = A.Plan(g, spec["rows"], spec["cols"], device=torch.cuda.current_device(), flags=flags, tune=tune)
    ins = device_inputs(spec, inputs)
    outs = plan.alloc_outputs()
    if spec.get("segments"):  # packed rows: elements past a row's 16-byte chunks are never written
        for o in outs:
            o.zero_()
    plan.run(ins, outs)
    torch.cuda.synchronize()
    res = {n: from_torch(t) for (n, _), t in zip(spec["outputs"], outs)}
    if return_plan:
        return res, plan
    return res


def virtual_allreduce(shards):
    """Test stand-in for astitch_run_sharded's collective when every rank's
    plan runs on one GPU: shards = [(ShardedPlan, workspace)], combined in
    rank order in place -- fp32 sum for SUM slots, int32 max of the order keys
    for RMAX slots (include/astitch.h, astitch_plan_colpart)."""
    import torch
    sp0 = shards[0][0]
    off0, cnt = sp0.colpart()
    if not cnt:
        return
    ops = sp0.colpart_ops()
    C = cnt // len(ops)
    for sp, _ in shards:
        assert sp.colpart()[1] == cnt and sp.colpart_ops() == ops
    for q, op in enumerate(ops):
        dt = torch.int32 if op == "max" else torch.float32
        parts = []
        for sp, ws in shards:
            off = sp.colpart()[0] + 4 * q * C     # each rank's own offset (depends on its grid)
            parts.append(ws[off: off + 4 * C].view(dt))
        total = parts[0].clone()
        for p_ in parts[1:]:
            total = torch.maximum(total, p_) if op == "max" else total + p_
        for p_ in parts:
            p_.copy_(total)
