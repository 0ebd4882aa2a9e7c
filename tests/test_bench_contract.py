"""bench.py keeps the driver's contract: one JSON line with the required keys
(CPU reference arm here; the GPU arm is checked with -m gpu)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
REQUIRED = ["metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
            "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config"]


def run_bench(*args, env=None, timeout=600):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args],
                         capture_output=True, text=True, timeout=timeout, cwd=ROOT,
                         env={**os.environ, **(env or {})})
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    return json.loads(lines[0])


def test_reference_arm_json_line():
    d = run_bench("--impl", "reference", "--config", "1", "--steps", "2", "--warmup", "1")
    for k in REQUIRED:
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert "first" in d["cpu_baseline"]["sample"] and d["cpu_baseline"]["value"] == d["value"]
    assert d["config"]["workload"].startswith("config1")


def test_reference_arm_other_ranks_exit_quietly():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                          "--config", "1", "--steps", "1", "--warmup", "1"],
                         capture_output=True, text=True, timeout=300, cwd=ROOT,
                         env={**os.environ, "RANK": "1", "WORLD_SIZE": "2"})
    assert out.returncode == 0 and out.stdout.strip() == ""


@pytest.mark.gpu
def test_gpu_arm_json_line():
    d = run_bench("--config", "1", "--steps", "3", "--warmup", "3", "--e2e-steps", "1")
    for k in REQUIRED + ["roofline", "clocks", "e2e", "gpu_launches", "cpu_baseline"]:
        assert k in d, k
    r = d["roofline"]
    assert r["bound"] == "hbm" and 0 < r["frac"] < 1 and r["peak"] > 1000
    o = d["onchip_roofline"]
    assert o["bound"] == "alu" and 0 < o["frac"] < 1 and o["peak"] > 1e12
    assert o["events_per_residue"]["hits"] > 0 and o["method_ops_per_residue"] > 10
    assert d["gpu_launches"] == 3
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle"


@pytest.mark.gpu
@pytest.mark.parametrize("gather,port", [("p2p", 29571), ("nccl", 29572)])
def test_gpu_arm_two_ranks_one_gpu(gather, port):
    """The N > 1 path of bench.py under torchrun (2 ranks sharing the one GPU,
    gloo host collectives): rank 0 alone prints one line with n_gpus 2 and
    the gather it timed (the fused peer append or the NCCL-style gather)."""
    out = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                          "--nproc-per-node", "2", "--master-addr", "127.0.0.1",
                          "--master-port", str(port), os.path.join(ROOT, "bench.py"),
                          "--gpus", "2", "--config", "1", "--steps", "3", "--warmup", "3",
                          "--no-e2e", "--no-cpu-baseline", "--gather", gather],
                         capture_output=True, text=True, timeout=600, cwd=ROOT,
                         env={**os.environ, "BLASTP_DIST_BACKEND": "gloo"})
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0
    assert d["config"]["gather"].startswith("p2p" if gather == "p2p" else "NCCL")
