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


def _torchrun(nproc, *args, env=None):
    import socket
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    out = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                          f"--nproc-per-node={nproc}", "--master-addr", "127.0.0.1",
                          "--master-port", str(port), os.path.join(ROOT, "bench.py"), *args],
                         capture_output=True, text=True, cwd=ROOT, timeout=900,
                         env={**os.environ, **(env or {})})
    assert out.returncode == 0, out.stderr[-3000:]
    return [ln for ln in out.stdout.splitlines() if ln.strip().startswith("{")]


@pytest.mark.gpu
def test_gpu_arm_one_rank_contract_line():
    lines = _run("--steps", "50", "--warmup", "3", "--workload", "C2", "--cpu-seconds", "1")
    assert len(lines) == 1
    j = json.loads(lines[0])
    assert j["n_gpus"] == 1 and j["steps"] == 50 and j["warmup"] == 3
    assert j["gpu_launches"] >= 1 and j["value"] > 0  # C2 runs the resident kernel: 1 launch
    r = j["roofline"]
    assert r["bound"] == "hbm" and 0 < r["frac"] < 1.2 and r["unit"] == "GB/s"
    assert j["cpu_baseline"]["kind"] == "oracle" and j["cpu_baseline"]["cores"] >= 1
    e2e = j["e2e"]
    assert e2e["value"] > 0 and e2e["h2d_bytes_per_step"] > 0 and e2e["d2h_bytes_per_step"] > 0
    assert j["clocks"] is None or "sm_mhz" in j["clocks"]


@pytest.mark.gpu
@pytest.mark.parametrize("mode", ["sync", "async"])
def test_gpu_arm_two_ranks_share_one_gpu(mode):
    """The N > 1 path of bench.py (torchrun, barrier + max over ranks, peer
    exchange, e2e through set_state) with both ranks on GPU 0 (PSO_SHARE_GPU)."""
    lines = _torchrun(2, "--gpus", "2", "--steps", "30", "--warmup", "3", "--workload", "C2",
                      env={"PSO_SHARE_GPU": "1", "PSO_GBEST": mode})
    assert len(lines) == 1  # rank 0 only
    j = json.loads(lines[0])
    assert j["n_gpus"] == 2 and j["scaling"] == "strong" and j["cpu_baseline"] is None
    c = j["config"]
    assert c["gbest_exchange"] == "nvlink-peer-stores" and c["gbest_mode"] == mode
    assert c["shared_gpu_harness_test"] is True
    assert j["value"] > 0 and j["e2e"]["value"] > 0


@pytest.mark.gpu
def test_gpu_arm_self_launches_ranks():
    """`python bench.py --gpus N` without torchrun launches the N ranks itself
    (the driver's SCALE run may call it either way) and still prints one line;
    here 3 ranks share GPU 0 (PSO_SHARE_GPU harness), NS_R8-sized swarm split 3 ways."""
    lines = _run("--gpus", "3", "--steps", "20", "--warmup", "3", "--workload", "NS_R8",
                 env={"PSO_SHARE_GPU": "1"})
    lines = [ln for ln in lines if ln.startswith("{")]
    assert len(lines) == 1
    j = json.loads(lines[0])
    assert j["n_gpus"] == 3 and j["value"] > 0 and j["gpu_launches"] >= 20
    assert j["config"]["gbest_exchange"] == "nvlink-peer-stores"


def test_self_launch_reference_arm_prints_once():
    lines = _run("--impl", "reference", "--gpus", "2", "--steps", "2", "--warmup", "1",
                 "--workload", "C1", "--ref-seconds", "3")
    lines = [ln for ln in lines if ln.startswith("{")]
    assert len(lines) == 1 and json.loads(lines[0])["impl"] == "reference"


def test_reference_arm_under_torchrun_prints_once():
    lines = _torchrun(2, "--impl", "reference", "--gpus", "2", "--steps", "2", "--warmup", "1",
                      "--workload", "C1", "--ref-seconds", "3")
    assert len(lines) == 1 and json.loads(lines[0])["impl"] == "reference"
