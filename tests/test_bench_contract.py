"""bench.py's JSON-line contract, exercised on CPU through the reference arm
(the oracle timed on a bounded sample) — the GPU arm shares the config,
metric and unit code."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args, env=None):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args],
                         capture_output=True, text=True, cwd=ROOT, timeout=600,
                         env={**os.environ, **(env or {})})
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.strip()]
    return lines


@pytest.mark.parametrize("workload", ["C1", "NS"])
def test_reference_arm_prints_one_contract_line(workload):
    lines = _run("--impl", "reference", "--steps", "3", "--warmup", "1", "--workload", workload,
                 "--ref-seconds", "4")
    assert len(lines) == 1
    j = json.loads(lines[0])
    assert j["impl"] == "reference"
    assert j["metric"] == "particle-dim updates/sec and % of HBM roofline at 1/2/4/8 B200"
    assert j["unit"] == "particle-dim updates/s" and j["higher_is_better"] is True
    assert j["steps"] == 3 and j["warmup"] == 1 and j["n_gpus"] == 1
    assert j["value"] > 0 and j["ms_per_step"] > 0
    assert j["dtype"] == "f32" and j["vs_baseline"] is None
    assert j["config"]["workload"].startswith({"C1": "C1-", "NS": "northstar"}[workload])
    cb = j["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] == 1 and cb["value"] == j["value"]
    e2e = j["e2e"]
    assert e2e["value"] == j["value"] and e2e["h2d_bytes_per_step"] == 0


def test_reference_arm_non_zero_rank_is_silent():
    lines = _run("--impl", "reference", "--steps", "1", "--warmup", "0", "--workload", "C1",
                 env={"RANK": "1", "WORLD_SIZE": "2"})
    assert lines == []
