"""bench.py contract on the host: the reference arm (the fp64 oracle on the
host cores) prints one JSON line with the driver's keys; ranks other than 0
print nothing and exit 0."""

import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env_extra=None):
    env = dict(os.environ)
    env.update(env_extra or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                          env=env, cwd=ROOT, timeout=600)


def test_reference_arm_json_line():
    r = _run(["--impl", "reference", "--config", "C1", "--steps", "2", "--warmup", "3"])
    assert r.returncode == 0, r.stderr
    lines = [ln for ln in r.stdout.splitlines() if ln.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["unit"] == "GB/s" and d["value"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["config"]["workload"].startswith("C1")


def test_reference_arm_other_ranks_silent():
    r = _run(["--impl", "reference", "--config", "C1", "--steps", "1"],
             {"WORLD_SIZE": "2", "RANK": "1", "LOCAL_RANK": "1"})
    assert r.returncode == 0, r.stderr
    assert r.stdout.strip() == ""


def test_reference_arm_uses_host_cores_and_records_cpu():
    """SURVEY 8(d) oracle timing: one unmodified-oracle process per host core
    over row shards; the line records the core count and the CPU model."""
    r = _run(["--impl", "reference", "--config", "C4", "--steps", "2", "--warmup", "3"])
    assert r.returncode == 0, r.stderr
    d = json.loads([ln for ln in r.stdout.splitlines() if ln.strip()][-1])
    cb = d["cpu_baseline"]
    assert cb["cores"] >= 1 and cb["host_cores"] >= cb["cores"] and cb["cpu_model"]
    assert "row shards" in cb["sample"] and cb["value"] > 0
